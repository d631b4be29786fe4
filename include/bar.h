/*
 * bar.h — C ABI of libbar.so: block-asynchronous relaxation async-(k) for A x = b on B200.
 *
 * The method is H. Anzt, S. Tomov, J. Dongarra, V. Heuveline, "A Block-Asynchronous
 * Relaxation Method for Graphics Processing Units" (/root/reference/PAPER.md; cited
 * as P:<line> with the section / equation / algorithm it falls in):
 *   - Jacobi, eq. 2 (§2.1):  x_i^{m+1} = (b_i - sum_{j!=i} a_ij x_j^m) / a_ii
 *   - async-(k), Algorithm 1 (§3.3) and eq. 4: rows are split into
 *     subdomains J_l of R consecutive rows, one per thread block; each block reads x "as it
 *     stands" in global memory, computes the off-block part s_i = b_i - sum_{j notin J_l} a_ij x_j
 *     once, runs k local Jacobi sweeps on its own components with the off-block values frozen
 *     (P:147), and writes x_J back, with no synchronisation between blocks (eq. 3).
 *   - sync-block-(k): the same two-stage sweep with every block reading the same x^(m)
 *     (deterministic block-Jacobi; reading R3), the parity mode.
 *   - the l2 residual ||b - A x||_2, fused into every sweep.
 *
 * No torch types cross this boundary: plain pointers and sizes only.
 *
 * Pointers. Matrix arrays given to bar_create_csr may be host or device memory (detected
 * with cudaPointerGetAttributes) and are COPIED into a library-owned layout; the caller keeps
 * ownership. b, x0, x given to bar_solve / bar_residual may be device memory on the matrix's
 * device (the fast path) or host memory (then the library stages them through device
 * buffers inside the call — the end-to-end path). The caller must not free them during a call.
 *
 * Streams. Every call is ordered on `cuda_stream` (a cudaStream_t; NULL = legacy default
 * stream) and returns only after its work on that stream is complete (it has to fill `info`).
 *
 * Errors. Every entry point returns a bar_status and never aborts or exits. The text of the
 * last error on the calling thread is available from bar_last_error(). Not converging within
 * max_global_iters is NOT an error (BAR_OK with info.converged = 0).
 *
 * Threads. A bar_matrix may be used by one thread at a time (its workspace is reused); different
 * matrices may be used from different threads at once.
 */
#ifndef BAR_H
#define BAR_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct bar_matrix_s *bar_matrix; /* opaque, library-owned */

typedef enum {
    BAR_MODE_ASYNC = 0,      /* async-(k): in-place, no inter-block sync (Alg. 1, eq. 4)      */
    BAR_MODE_SYNC_BLOCK = 1, /* sync-block-(k): block-Jacobi, k local sweeps, x double-buffered */
    BAR_MODE_JACOBI = 2      /* synchronous Jacobi (eq. 2)                                     */
} bar_mode;

typedef enum {
    BAR_OK = 0,
    BAR_ERR_INVALID_ARG = 1, /* NULL handle/pointer, n < 1, k < 1, tol < 0 or NaN, R out of range ... */
    BAR_ERR_BAD_CSR = 2,     /* rowptr[0] != 0, rowptr not monotone, rowptr[n] != nnz, col out of
                                [0, n), columns not strictly increasing, missing diagonal           */
    BAR_ERR_ZERO_DIAG = 3,   /* a_ii == 0                                                         */
    BAR_ERR_NONFINITE = 4,   /* a value is Inf/NaN (matrix, or b / x0 at solve time)              */
    BAR_ERR_DIVERGED = 5,    /* rel. residual became non-finite or > 1e30 (rho(B) > 1)     */
    BAR_ERR_CUDA = 6,        /* CUDA runtime failure; see bar_last_error()                        */
    BAR_ERR_NCCL = 7,        /* NCCL failure (multi-GPU)                                          */
    BAR_ERR_OOM = 8          /* device allocation failed                                          */
} bar_status;

/* Largest subdomain size R accepted (two fp64 copies of the block's x live in shared memory). */
#define BAR_MAX_ROWS_PER_BLOCK 8192

typedef struct {
    int64_t iters;          /* global iterations m of the returned x = x^(m) (sync modes: exactly
                               the oracle's count; async: completed global iterations)           */
    double rel_res;         /* ||b - A x||_2 / ||b||_2 of the RETURNED x, computed exactly       */
    int32_t converged;      /* rel_res <= tol                                                     */
    int64_t cta_iters_min;  /* async persistent kernel: min / max per-block global iteration      */
    int64_t cta_iters_max;  /*   counts (= iters otherwise)                                       */
    double model_bytes_per_iter; /* nnz*(8+4) + n*(8+8+8+4): the contract bytes of one iteration */
    int64_t kernel_launches;     /* kernels this call launched (all of them libbar's own)         */
    double sweep_kernel_ms;      /* device time of the block-sweep launches that did work, from CUDA
                                    events recorded on cuda_stream around each launch (excludes
                                    residual/setup kernels and launches queued after a stop)     */
    double sweep_kernel_iters;   /* global iterations those launches performed (one per launch; the
                                    single-launch async kernel: subdomain sweeps claimed / q), so
                                    sweep_kernel_ms / sweep_kernel_iters = device ms per iteration */
} bar_solve_info;

typedef struct {
    int64_t n, nnz;               /* matrix size and stored entries                              */
    int32_t rows_per_block;       /* R                                                            */
    int64_t num_subdomains;       /* q = ceil(n / R)                                              */
    int64_t layout_entries;       /* stored entries incl. padding of the sliced layout            */
    int64_t local_entries;        /* entries with a column inside their row's subdomain (incl. diag) */
    double model_bytes_per_iter;  /* nnz*(8+4) + n*(8+8+8+4)                                      */
    int32_t device;
    const char *last_sweep_kernel; /* static name of the sweep kernel the latest bar_solve /
                                      bar_sweep launch on this handle used ("none" before any);
                                      a diagnostic for profiling and the bench's roofline line  */
    int32_t coded;                /* 1: the layout also holds 1-byte column codes + per-subdomain
                                     offset dictionaries (read by the two-blocks-per-SM sweep)   */
    double layout_bytes_per_iter; /* compulsory HBM bytes of one sweep of THIS layout: values (8 B),
                                     columns (1 B coded / 4 B) per stored entry incl. padding,
                                     b + x read + x write (24 B) per row, slice metadata and
                                     dictionaries (excludes re-reads of off-block x)            */
} bar_matrix_info;

/*
 * bar_create_csr — validate a CSR matrix and copy it into the library layout.
 *   n            rows = columns (>= 1)
 *   nnz          stored entries (= rowptr[n]; < 2^31)
 *   rowptr       int32[n+1], rowptr[0] = 0, non-decreasing
 *   col          int32[nnz], 0 <= col < n, strictly increasing within each row, diagonal present
 *   val          double[nnz], finite, a_ii != 0
 *   rows_per_block  R, subdomain size (1 <= R <= BAR_MAX_ROWS_PER_BLOCK); J_l = [l R, min(n,(l+1) R))
 *   device       CUDA device ordinal for the layout and all later calls
 *   out          receives the handle (set to NULL on failure)
 * Errors: BAR_ERR_INVALID_ARG, BAR_ERR_BAD_CSR, BAR_ERR_ZERO_DIAG, BAR_ERR_NONFINITE,
 *         BAR_ERR_CUDA, BAR_ERR_OOM.
 */
bar_status bar_create_csr(int64_t n, int64_t nnz, const int32_t *rowptr, const int32_t *col,
                          const double *val, int32_t rows_per_block, int device, bar_matrix *out);

/*
 * bar_solve — iterate from x0 until ||b - A x^(m)||_2 / ||b||_2 <= tol or m = max_global_iters.
 *   b, x0        double[n] (device or host); x0 == NULL means x0 = 0
 *   x            double[n] output (device or host); may alias x0
 *   k            local Jacobi sweeps per global iteration (async / sync-block; ignored for
 *                Jacobi), >= 1 — the paper's async-(k)
 *   max_global_iters  >= 0
 *   tol          >= 0 (0 = run exactly max_global_iters iterations unless the residual is 0)
 *   mode         BAR_MODE_ASYNC / BAR_MODE_SYNC_BLOCK / BAR_MODE_JACOBI
 *   cuda_stream  cudaStream_t or NULL
 *   info         nullable
 * Stopping rule (reading R6): x^(0) is checked first; the sync modes return the
 * first x^(m) with rel_res <= tol (bitwise the oracle's m up to the order of the residual sum);
 * async returns the first iterate whose fused residual estimate AND exact confirming residual
 * are <= tol. b = 0 returns x = 0, iters = 0, converged. With x0 == NULL the exact residual of
 * x^(0) = 0 is ||b|| / ||b|| (one read of b, no SpMV).
 * Async kernels: large systems run one launch per global iteration; systems whose
 * subdomains all fit on the device at once run ONE launch for all iterations, and a repeated call
 * with the same pointers, k, max_global_iters and tol replays that solve from a CUDA graph the
 * handle captured on the first such call (the contents behind the pointers may change).
 * Errors: BAR_ERR_INVALID_ARG, BAR_ERR_NONFINITE (b or x0), BAR_ERR_DIVERGED, BAR_ERR_CUDA,
 *         BAR_ERR_OOM. On BAR_ERR_DIVERGED x holds the last iterate.
 */
bar_status bar_solve(bar_matrix A, const double *b, const double *x0, double *x, int32_t k,
                     int64_t max_global_iters, double tol, bar_mode mode, void *cuda_stream,
                     bar_solve_info *info);

/*
 * bar_solve_ex — bar_solve with the options of SURVEY §8(f)'s next rows (opts may be NULL):
 *   tau        N3, τ-scaled relaxation: every update x <- x + tau (v - x), i.e. the
 *              iteration matrix B = I - tau D^-1 A (tau = 2/(lambda_1 + lambda_n) of D^-1 A makes
 *              Jacobi converge for SPD systems with rho(B) > 1, like s1rmt3m1). 1 = the paper's methods.
 *   fail_mask  N1, failure injection (§4.5): n bytes (host or device), nonzero = the
 *              component "fails": it keeps its value in global iterations m (1-based: the m-th
 *              global iteration produces x^(m)) with fail_start <= m < fail_stop; fail_stop < 0 =
 *              never recovers. NULL = no failures.
 *   res_history  HOST double[max_global_iters + 1] (nullable): sync modes rel_res(x^(m)) for
 *              m = 0..iters (exact up to the summation order); async the fused per-iteration
 *              estimate (x as each block saw it). Entries past iters are left untouched.
 *   async_single_launch  -1 the handle's choice (bar_tuning.single_launch), 0 one launch per
 *              global iteration, 1 the fully asynchronous single-launch kernel (falls back
 *              silently where it does not apply). Options tau != 1, fail_mask and res_history
 *              imply 0.
 */
typedef struct {
    double tau;
    const uint8_t *fail_mask;
    int64_t fail_start, fail_stop;
    double *res_history;
    int32_t async_single_launch;
} bar_solve_opts;

bar_status bar_solve_ex(bar_matrix A, const double *b, const double *x0, double *x, int32_t k,
                        int64_t max_global_iters, double tol, bar_mode mode, void *cuda_stream,
                        bar_solve_info *info, const bar_solve_opts *opts);

/*
 * bar_residual — res_norm2 = ||b - A x||_2 (and b_norm2 = ||b||_2 if non-NULL), computed on the
 * device with a fixed-order (deterministic) reduction. b, x device or host.
 * Errors: BAR_ERR_INVALID_ARG, BAR_ERR_CUDA, BAR_ERR_OOM.
 */
bar_status bar_residual(bar_matrix A, const double *b, const double *x, void *cuda_stream,
                        double *res_norm2, double *b_norm2);

/*
 * bar_sweep — run exactly `nsweeps` global iterations of `mode` from the current x, with no
 * convergence control and no host synchronisation (stream-ordered; returns after enqueueing).
 * Sync modes ping-pong between x and a library buffer and leave x^(nsweeps) in x; async updates
 * x in place. For callers that drive their own loop and for per-launch kernel timing.
 *   b, x   DEVICE double[n] on the matrix's device; k >= 1; nsweeps >= 0.
 * Errors: BAR_ERR_INVALID_ARG (also for host pointers), BAR_ERR_CUDA, BAR_ERR_OOM.
 */
bar_status bar_sweep(bar_matrix A, const double *b, double *x, int32_t k, int64_t nsweeps, bar_mode mode,
                     void *cuda_stream);

/* bar_matrix_get_info — sizes and the contract bytes per global iteration of a handle. */
bar_status bar_matrix_get_info(bar_matrix A, bar_matrix_info *info);

/*
 * bar_tuning — explicit per-handle overrides of the library's kernel and schedule choices
 * (DESIGN.md §5). The library reads NO environment variables: every choice that is not the
 * default is made here, on one handle, by the caller (profiling, A/B runs, and the tests that
 * force each kernel path). All-zero = the defaults. Choices that do not apply to a layout fall
 * back silently to the next kernel in the dispatch order; sync-block and Jacobi
 * iterates do not depend on any field here (bitwise), async iterates depend on the schedule.
 */
typedef struct {
    int32_t kernel;         /* 0 auto; force a fallback family: 1 k_block (shared-memory staged),
                               2 k_reg, 3 k_reg_tma, 4 k_block_pers                              */
    int32_t duo;            /* 0 auto, 1 two-blocks-per-SM kernel wherever it fits, -1 never      */
    int32_t pipe;           /* 0 auto, 1 two-ahead pipelined kernel wherever it fits, -1 never    */
    int32_t coded;          /* 0 auto = 1: coded columns when the layout has them, off-block x
                               gathered entry by entry; 2 staged gathers (each subdomain's off-block
                               x intervals copied to shared memory first, where the layout has
                               them); -1 int32 columns                                            */
    int32_t async_order;    /* per-launch async subdomain order: 0 auto (contiguous chunks per
                               block, R15), 1 chunks, 2 round robin, 3 fronts: `fronts` contiguous
                               ranges, each swept round robin by its share of the blocks         */
    int32_t async_queue;    /* 0 static claims, 1 device work-queue claims (k_block_stage)       */
    int32_t resident;       /* 0 auto, -1 never use the block-owns-subdomain single-launch kernel */
    int32_t lead;           /* k_block_resident: max sweeps a block may lead the last completed
                               global iteration (0 = default 48, the residual ring's bound; 1..48) */
    int32_t ghost_prefetch; /* L2 bulk prefetch of the gather ranges: 0 auto (R >= 512), 1, -1   */
    int32_t graph;          /* single-launch async: 0 capture + replay as a CUDA graph, -1 never  */
    int32_t single_launch;  /* async: 0 auto (one launch for all iterations when one iteration
                               moves < 256 MB), 1 always where it applies, -1 never              */
    int32_t jacobi_rowwise; /* 1: Jacobi by the row-wise kernel even where the staged kernels apply */
    int32_t grid_cap;       /* > 0: at most this many persistent blocks                          */
    int32_t warps;          /* k_block: warps per block (0 auto)                                 */
    int32_t halo;           /* multi-GPU sync / collective exchange: 0 NCCL grouped send/recv,
                               1 one ncclAllGather per iteration                                 */
    int32_t peer;           /* multi-GPU async: 0 peer memory when mapped, -1 the collective path */
    int32_t fronts;         /* async_order = 3: number of fronts (0 = 8)                          */
    int32_t stage_bx;       /* k_block_duo: 0 stage b_J and x_J with the slab (bulk copies) where
                               that keeps the blocks per SM, -1 per-row loads                    */
    int32_t lazy_publish;   /* k_block_resident: 0 non-blocking residual publication — a tagged
                               word per block (partial + iteration in one relaxed store) in the
                               256-thread variant up to 256 blocks, else a ring of partials + a
                               release counter; 1 always the counter; 2 tagged wherever warp 0 can
                               hold the words; -1 one blocking atomic per block and iteration     */
    int32_t slab_prefetch;  /* k_block_duo: 1 L2 bulk prefetch of the slab two subdomains ahead
                               (a second slab buffer in L2), 0 off                               */
    int32_t overlap;        /* multi-GPU collective path: 0 sweep the interior subdomains (no ghost
                               reads) on a second stream while the halo exchange runs, then the
                               boundary ones; -1 one sweep after the exchange                    */
    int32_t unroll_off;     /* k_block_duo, coded columns: 0 phase 1 unrolled where a row has <= 4
                               off-block entries (both rows' gathers in flight), -1 the generic
                               loop                                                              */
    int32_t fuse_residual;  /* k_block_resident: 0 the confirming residual computed at the end of
                               the single launch (grid barrier), -1 a separate residual kernel    */
    int32_t gather_ahead;   /* k_block_resident (rows of > 12 local entries, 256 threads): 0 the
                               next iteration's off-block x loaded right after the write-back,
                               -1 at the start of the sweep                                      */
} bar_tuning;

/* bar_set_tuning — replace the handle's tuning (NULL = defaults). Not thread-safe with a
 * concurrent call on the same handle. Errors: BAR_ERR_INVALID_ARG. */
bar_status bar_set_tuning(bar_matrix A, const bar_tuning *tuning);

/* bar_destroy — free the handle and its device memory (NULL-safe). */
void bar_destroy(bar_matrix A);

/* ===================== multi-GPU: row-partitioned solve =====================
 * One process per GPU. Rank r owns the contiguous rows [row_begin, row_end) of the global
 * system — the paper's "blocks addressed to the different devices, again split into ... blocks
 * of rows ... assigned to the different thread blocks" (§3.4). row_begin must be a
 * multiple of rows_per_block, so subdomains never straddle ranks and the per-row arithmetic
 * is identical to the one-GPU solve (sync-block / Jacobi iterates are bitwise independent of
 * the number of ranks). Columns a rank reads but does not own are its "ghosts". Local numbering
 * is order-preserving: [ghosts below row_begin | owned rows | ghosts above], stored relative to
 * the owned block (ghosts below are negative), so a row's entries keep their global order.
 *
 * Two ways a rank reads its ghosts, replacing the paper's AMC / DC / DK host- or master-GPU
 * transfers:
 *   collective    sync-block and Jacobi (and async when peer memory is unavailable): once per
 *                 global iteration, NCCL grouped send/recv over NVLink (bar_tuning.halo = 0) or
 *                 one ncclAllGather (halo = 1) refreshes the ghost slots; the per-rank residual
 *                 sums are all-gathered and added in rank order, so every rank takes the same
 *                 stopping decision from the same bits.
 *   peer memory   async (the default when every rank can map every other rank's memory; north
 *                 star: "an async mode reads peers' x over NVLink P2P with no barrier"; the paper's
 *                 DK idea, without a master GPU): before each local sweep a rank PULLS its
 *                 ghosts from the owners' live iterates (relaxed system-scope loads: x "as it
 *                 stands", eq. 3) and pushes its residual partial into every rank's board (a small
 *                 array in each rank's memory, mapped through CUDA IPC). No collective and no
 *                 barrier while iterating: a rank whose estimate meets tol writes a tagged stop
 *                 request into every board, and the ranks meet only for the exact confirming
 *                 residual (two board barriers: device-side release/acquire waits, 20 s timeout
 *                 -> BAR_ERR_NCCL instead of a hang). info.iters = min over ranks of the global
 *                 iterations each ran; info.cta_iters_max = the max.
 */

/*
 * bar_create_csr_dist — §8(b)'s multi-GPU entry point: this rank's share of a row-partitioned
 * matrix, planned inside the library. Collective: every rank of the group calls it.
 *   n_global        rows of the global system
 *   row_begin/end   this rank's rows (row_begin a multiple of rows_per_block; the ranks' ranges
 *                   contiguous and ascending in rank order, together [0, n_global))
 *   nnz_local, rowptr, col, val   the local rows in CSR with GLOBAL column ids (rowptr relative,
 *                   rowptr[0] = 0), host or device memory, copied
 *   rows_per_block  R; device: this rank's GPU
 *   nccl_unique_id  128 bytes from bar_nccl_unique_id on rank 0, given to every rank (required)
 *   rank, nranks    this rank and the group size
 * Inside: ncclCommInitRank; an all-gather of every rank's row range, ghost count and device, and
 * of the ghost lists; the exchange plan and local numbering; the local layout; and, when every
 * rank can reach every other rank's memory (cudaDeviceCanAccessPeer, agreed by a min
 * all-reduce), an all-gather of CUDA IPC handles that maps every rank's iterate and board.
 * The returned handle works with bar_solve / bar_residual (collective: b, x0, x are this rank's
 * rows; every rank calls with the same k, limits and mode), bar_matrix_get_info (local sizes),
 * bar_set_tuning, bar_sweep (local launches on this rank's rows, no exchange: kernel timing) and
 * bar_destroy (frees the communicator). bar_solve_ex options tau, fail_mask and res_history are
 * not supported on it (BAR_ERR_INVALID_ARG).
 * Errors: as bar_create_csr, plus BAR_ERR_NCCL; BAR_ERR_INVALID_ARG for a bad partition.
 */
bar_status bar_create_csr_dist(int64_t n_global, int64_t row_begin, int64_t row_end, int64_t nnz_local,
                               const int32_t *rowptr, const int32_t *col, const double *val, int32_t rows_per_block,
                               int device, const void *nccl_unique_id, int rank, int nranks, bar_matrix *out);

/* bar_nccl_unique_id — rank 0 creates the NCCL id (128 bytes) that every rank passes to
 * bar_create_csr_dist / bar_dist_create (broadcast it by any means). BAR_ERR_NCCL without NCCL. */
bar_status bar_nccl_unique_id(void *id128);

/* ---- lower-level building blocks (explicit plans; tests, in-process loopback groups) -------- */
typedef struct bar_dist_s *bar_dist; /* opaque, one per rank */

/* Planning, host only (no GPU needed):
 *   bar_dist_ghosts    sorted distinct ghost columns of the local rows: the n_ghost_lo ones
 *                      below row_begin, then the n_ghost_hi ones at or above row_end. Call with
 *                      ghosts = NULL for the counts. rowptr is relative (rowptr[0] = 0), col global.
 *   bar_dist_localize  col_local[e] = col[e] - row_begin for owned columns, -n_ghost_lo + j for
 *                      the j-th ghost below, (row_end - row_begin) + j for the j-th ghost above.
 *   bar_dist_plan      from every rank's row range (row_ranges[2p], [2p+1]), ghost count and
 *                      ghost list (ghosts_all: the lists concatenated in rank order): this rank's
 *                      recv_counts[p] (its ghosts owned by p; consecutive in ghost order),
 *                      send_counts[p] and send_idx (owned local rows p needs, in p's ghost order,
 *                      concatenated by p; NULL to get the counts first) and ghost_src_idx[j]
 *                      (owner-local row of ghost j, for bar_dist_enable_p2p; nullable).
 */
bar_status bar_dist_ghosts(int64_t row_begin, int64_t row_end, int64_t nnz_local, const int32_t *rowptr,
                           const int32_t *col, int64_t *n_ghost_lo, int64_t *n_ghost_hi, int32_t *ghosts);
bar_status bar_dist_localize(int64_t row_begin, int64_t row_end, int64_t nnz_local, const int32_t *rowptr,
                             const int32_t *col, int64_t n_ghost_lo, int64_t n_ghost_hi, const int32_t *ghosts,
                             int32_t *col_local);
bar_status bar_dist_plan(int nranks, int rank, const int64_t *row_ranges, const int64_t *ghost_counts,
                         const int32_t *ghosts_all, int64_t *recv_counts, int64_t *send_counts, int32_t *send_idx,
                         int32_t *ghost_src_idx);

/*
 * bar_dist_create — this rank's share from an explicit plan: the local CSR (n_local = row_end -
 * row_begin rows, col_local from bar_dist_localize, values), the plan (bar_dist_plan), and the
 * transport.
 *   nccl_id   128-byte ncclUniqueId (an NCCL communicator for the collective path), or NULL: no
 *             communicator — then either link the ranks of one process into a LOOPBACK group
 *             (bar_dist_link_loopback; several ranks on one device, device copies as the exchange,
 *             driven by bar_dist_solve_loopback — the partitioned path on a single GPU), or, for
 *             separate processes, enable peer memory (bar_dist_enable_p2p with IPC handles): then
 *             only the async mode is available.
 *   send_idx  int32[sum send_counts] local row indices; send/recv_counts int64[nranks].
 * Arrays may be host or device memory and are copied. Errors as bar_create_csr, plus
 * BAR_ERR_NCCL, BAR_ERR_INVALID_ARG (row_begin not a multiple of R, inconsistent counts).
 */
bar_status bar_dist_create(int64_t n_global, int64_t row_begin, int64_t row_end, int64_t nnz_local,
                           const int32_t *rowptr, const int32_t *col_local, const double *val, int64_t n_ghost_lo,
                           int64_t n_ghost_hi, int nranks, int rank, const int64_t *recv_counts,
                           const int64_t *send_counts, const int32_t *send_idx, int32_t rows_per_block, int device,
                           const void *nccl_id, bar_dist *out);

/* bar_dist_link_loopback — connect the loopback ranks of one process (ranks[r] has rank r). */
bar_status bar_dist_link_loopback(bar_dist *ranks, int nranks);

/*
 * bar_dist_solve — the solve of one rank (every rank calls it with the same k, limits and mode):
 * b, x0, x are this rank's owned rows (device or host, as bar_solve). Collective path per global
 * iteration: halo exchange, one block sweep of the local subdomains, all-gather of the per-rank
 * [sum r^2, sum b^2] and a rank-ordered sum. Async over peer memory: see above. Async without
 * peer memory: blocks of a rank run asynchronously (async-(k) within the GPU) and read the
 * ghosts of the latest collective exchange.
 */
bar_status bar_dist_solve(bar_dist D, const double *b, const double *x0, double *x, int32_t k,
                          int64_t max_global_iters, double tol, bar_mode mode, void *cuda_stream,
                          bar_solve_info *info);

/* bar_dist_solve_loopback — the same solve for all loopback ranks of this process, on one
 * stream, with device-to-device copies as the exchange. b[r], x0[r], x[r] are rank r's rows. */
bar_status bar_dist_solve_loopback(bar_dist *ranks, int nranks, const double *const *b, const double *const *x0,
                                   double *const *x, int32_t k, int64_t max_global_iters, double tol,
                                   bar_mode mode, void *cuda_stream, bar_solve_info *info);

/*
 * Peer memory for the async mode (bar_create_csr_dist does this itself):
 *   bar_dist_p2p_handles  128 bytes: CUDA IPC handles of this rank's iterate and board (publish
 *                         them to the group), and *own_offset (its owned-block offset, in doubles).
 *   bar_dist_enable_p2p   ghost_src_idx[j] = owner-local row of ghost j (ghost order); handles =
 *                         nranks * 128 bytes and own_offsets = nranks offsets gathered from every
 *                         rank, or both NULL for linked loopback ranks (same process) and 1-rank groups.
 */
bar_status bar_dist_p2p_handles(bar_dist D, void *handles128, int64_t *own_offset);
bar_status bar_dist_enable_p2p(bar_dist D, const int32_t *ghost_src_idx, const void *handles,
                               const int64_t *own_offsets);

/* bar_dist_sweep — measurement entry point: enqueue exactly nsweeps launches of this rank's local
 * block-sweep kernel on its current iterate (no halo exchange, no convergence control, no sync;
 * ghost values are whatever the last exchange left). Local, not collective. */
bar_status bar_dist_sweep(bar_dist D, int32_t k, int64_t nsweeps, bar_mode mode, void *cuda_stream);

/* bar_dist_set_tuning — bar_set_tuning of the rank's local handle (kernel choice, halo mode). */
bar_status bar_dist_set_tuning(bar_dist D, const bar_tuning *tuning);

/* bar_dist_destroy — free one rank's share (NULL-safe; also destroys its NCCL communicator). */
void bar_dist_destroy(bar_dist D);

/* bar_last_error — text of the last failure on the calling thread ("" if none). */
const char *bar_last_error(void);

/* bar_build_id — identity of this build: "src:<16 hex> sm_100a", the hex being a SHA-256 over the
 * library's sources (csrc/*.cu, *.cuh, include/bar.h) and its nvcc flags, fixed at build time
 * (tools/build.py). Unlike a hash of the .so (nvcc output is not byte-reproducible) it is the same
 * for every build of the same sources; measurements stamped with it (profiles/traffic_*.json) are
 * used only by a library with the same id. Static string, never NULL. */
const char *bar_build_id(void);

#ifdef __cplusplus
}
#endif

#endif /* BAR_H */
