// bar_internal.cuh — library-private types shared by the libbar.so translation units.
//
// Device layout of a matrix ("split sliced-ELL"):
//   * rows are grouped into subdomains J_l = [l*R, min(n,(l+1)*R)) (eq. 4's TS..TE);
//   * each subdomain is cut into slices of 32 consecutive rows (one warp, lane = row);
//     slice s = l*SPB + j (SPB = ceil(R/32)) holds rows TS + 32 j + lane;
//   * a slice stores its rows' entries column-major (entry e of lane t at ptr[s] + 32 e + t),
//     first the `wo` OFF-BLOCK entries (global column) and then the `wl` LOCAL entries (column
//     inside J_l, stored as the local index col - TS, the diagonal always the first local entry
//     e = wo); shorter rows are padded with value 0 and a harmless column (their own row).
// So one warp-wide load of entry e is a single coalesced 256 B (values) / 128 B (columns)
// transaction, the local/off-block split of Alg. 1 costs nothing at run time,
// and the diagonal (for D^-1) is found without a search.
#pragma once

#include <cmath>

#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <string>

#include <nvtx3/nvToolsExt.h>

#include "bar.h"

namespace bar {

// NVTX range for the phases of a call (SURVEY §5 tracing): visible in nsys / ncu timelines;
// header-only NVTX3, a no-op unless a tool is attached.
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange &) = delete;
    NvtxRange &operator=(const NvtxRange &) = delete;
};

constexpr int kSlice = 32;  // rows per slice = warp width

// Device-resident solver state (one per matrix handle), updated by the last block of each
// launch (fixed-order final reduction). Read back by the host once per chunk of launches.
struct DevState {
    unsigned int counter;   // last-block ticket
    int stop;               // kernels return immediately when set
    int diverged;
    int aborted;            // k_block_resident: blocks were not co-resident (a block waited > ~2 ms
                            // for lagging ones); every block stopped, the host continues with
                            // per-launch kernels from the current iterate (R12)
    long long iter;         // launches that executed (sync: m of the latest x^(m) produced)
    long long conv_iter;    // sync: m with rel_res(x^(m)) <= tol
    double bnorm;           // ||b||_2
    double tol;
    double last_rel;        // latest fused relative residual
    double exact_rel;       // latest standalone residual (bar_residual / confirmation)
    double exact_ss;        // its sum of squares
    unsigned long long work;// async work queue: next claim (subdomain w mod q of iteration w / q)
    long long iters_done;   // async persistent: completed global iterations
    long long stop_iter;    // async persistent: iteration whose residual estimate met tol
    unsigned long long work_resume;  // async persistent: first unclaimed w when the queue closed
    // async persistent: per-iteration accumulators (ring of kSlots iterations)
    unsigned int done[64];  // subdomains of iteration m finished (slot m % 64)
    double ss[64];          // sum of r_i^2 of those subdomains (x as it stood)
    double bs[64];          // sum of b_i^2
    double init_rel;        // single-launch async: exact rel_res of x^(0) (k_init_check)
    unsigned long long res_sweeps;  // k_block_resident: subdomain sweeps done (all launches)
    unsigned long long t_first, t_last;  // single-launch kernels: %globaltimer (ns) of the first
                                         // block start and the last block exit (graph replays
                                         // cannot time their kernel with host-visible events)
    // k_block_resident's fused exact residual of the returned iterate (KP::fuse_residual): blocks
    // arrived at the final grid barrier, reduction ticket, and whether exact_rel was produced
    unsigned int fuse_arrive, fuse_ticket;
    int exact_fused;
    unsigned int epoch;     // bumped by every state reset / resume: tags k_block_resident's tagged
                            // residual publication (stale ring words of earlier launches never match)
};
constexpr int kSlots = 64;

// Host: size of the next chunk of per-launch sweeps queued before the host reads the state.
// Doubling (8, 16, ..., 256), or, once two fused estimates (iteration it, rel) are known, the
// launches the observed per-iteration rate needs to reach tol plus a margin of 2: the chunk that
// reaches tol then does not queue up to 255 launches that return at once (each a full-grid
// launch, and in the collective multi-GPU path a halo exchange and an all-gather) and needs no
// extra host round trip. Deterministic in (it, rel), so ranks holding the same agreed state size
// their chunks identically.
struct ChunkSizer {
    long long it = -1;
    double rel = 0.0;
    int64_t next(int64_t c, long long it_now, double rel_now, double tol) {
        int64_t nc = c * 2 < 256 ? c * 2 : 256;
        if (it >= 0 && it_now > it && rel > 0.0 && rel_now > 0.0 && rel_now < rel && tol > 0.0 &&
            std::isfinite(rel_now)) {
            const double rate = std::pow(rel_now / rel, 1.0 / (double)(it_now - it));
            const double need = std::ceil(std::log(tol / rel_now) / std::log(rate));
            // (need + 2 <= KernelTimer::kMax: every launch of a chunk gets its timer events)
            if (rate > 0.0 && rate < 1.0 && need >= 0.0 && need < 256.0) nc = std::min<int64_t>((int64_t)need + 2, 256);
        }
        it = it_now;
        rel = rel_now;
        return nc;
    }
};

struct Layout {
    int64_t n = 0, nnz = 0;
    int32_t R = 0;
    int32_t spb = 0;            // slices per (full) subdomain
    int64_t q = 0;              // subdomains
    int64_t nslices = 0;
    int64_t entries = 0;        // padded entries
    int64_t local_entries = 0;
    int max_wl = 0, max_wo = 0;
    int max_w = 0;              // widest slice: max over slices of wl + wo
    int sms = 148;              // SMs of the device (persistent grids)
    // device arrays
    double *val = nullptr;      // [entries]
    int32_t *col = nullptr;     // [entries]
    int64_t *sptr = nullptr;    // [nslices+1] entry offset of each slice
    int32_t *sw = nullptr;      // [nslices]   wl | (wo << 16)
    // [q][kGhostRanges] (first column, count) of x ranges holding most of subdomain l's
    // off-block columns (count 0 = unused): bulk L2 prefetch targets for the a3 gathers
    int32_t *gr = nullptr;
    // Coded columns (built when every subdomain has <= kDictMax distinct column offsets d = col - row,
    // as stencil / FE matrices do; else NULL): codes[e] indexes the dictionary of entry e's
    // subdomain, dict[dptr[l] .. dptr[l+1]) (16-byte padded), so a column costs 1 byte of HBM
    // traffic instead of 4 in the kernels that read them (k_block_duo).
    uint8_t *codes = nullptr;   // [entries]
    int32_t *dict = nullptr;    // [dptr[q]]
    int32_t *dptr = nullptr;    // [q + 1]
    int64_t dict_entries = 0;
    // Staged gathers (coded layouts whose every subdomain's off-block columns lie in <= kMaxIv
    // x intervals of total length <= 4 R; else xs_len = 0): iv[l] = kMaxIv x (lo, len, base, 0)
    // and sdict (dictionary of shared-memory index offsets, layout.cu k_codes); xs_len = the
    // largest interval buffer (>= R) in doubles
    int32_t *sdict = nullptr;   // [dptr[q]]
    int32_t *iv = nullptr;      // [q][kMaxIv][4]
    int64_t xs_len = 0;
    bar_tuning tune{};          // explicit kernel / schedule overrides (bar_set_tuning); zero = defaults
    mutable int64_t rw_grid = -1;  // cached rowwise_grid (occupancy queries cost API round trips)
    mutable const char *last_kernel = "none";  // name of the most recently launched sweep kernel
};
constexpr int kGhostRanges = 4;
constexpr int kDictMax = 256;
constexpr int kMaxIv = 4;

// Device time of the sweep-kernel launches of one solve, taken with CUDA events on the
// launching stream around each launch (the bench's live per-launch duration inside its timed
// region). Launches queued after a stop request return at once and are not counted.
struct KernelTimer {
    static constexpr int kMax = 256;  // >= the largest chunk of launches between host reads
    cudaEvent_t ev[2 * kMax] = {};
    int64_t m[kMax] = {};             // global iteration index of recorded launch i
    int used = 0;
    double ms = 0.0, iters = 0.0;     // accumulated over the current solve
};

// The first pass of a single-launch async solve (x^(0) residual, device-side x^(0) check, the
// solve, the confirming residual, the state read-back) captured as a CUDA graph and replayed when
// the same call repeats: one graph launch instead of five API launches per solve.
struct SolveGraph {
    cudaStream_t cap = nullptr;      // capture stream (library-private)
    cudaGraphExec_t exec = nullptr;
    bool unsupported = false;        // the key's call has no single-launch kernel: do not capture
    const char *kernel = "none";     // the sweep kernel the graph launches (Layout::last_kernel at capture)
    const double *b = nullptr, *x0 = nullptr;
    double *x = nullptr;
    int32_t k = 0;
    int64_t max_iters = 0;
    double tol = 0.0;
};

struct Workspace {
    KernelTimer timer;
    SolveGraph graph;
    double *xbuf = nullptr;     // n: second iterate buffer (sync modes)
    double *stage_b = nullptr;  // n: device staging of host b (end-to-end path)
    double *stage_x = nullptr;  // n: device staging of host x0/x
    double *partials = nullptr; // per-block partial sums of squares
    uint8_t *frozen = nullptr;  // N1 failure mask (device copy, n bytes)
    double *ring = nullptr;     // [kSlots][q] residual partials of k_block_resident's lazy publication
    double *bsum_arr = nullptr; // [q]
    int64_t npartials = 0;
    DevState *state = nullptr;  // device
    DevState *h_state = nullptr;// pinned host mirror
};

}  // namespace bar

struct bar_matrix_s {
    int device = 0;
    bar::Layout L;
    bar::Workspace W;
    struct bar_dist_s *dist = nullptr;  // set on handles from bar_create_csr_dist (one rank's share)
};

namespace bar {

void set_error(const std::string &msg);
bar_status cuda_fail(cudaError_t e, const char *what);

// RAII: switch to a handle's device for the duration of a call.
struct DeviceGuard {
    int prev = -1;
    bool ok = true;
    explicit DeviceGuard(int dev) {
        if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
        if (prev != dev) ok = cudaSetDevice(dev) == cudaSuccess;
    }
    ~DeviceGuard() {
        int cur = -1;
        if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
    }
};

// api.cu helpers
bool is_device_ptr(const void *p);
bar_status ensure_workspace(bar_matrix A);
bar_status ensure_buf(double **p, int64_t n);
double model_bytes(const Layout &L);
bool use_async_multi(const Layout &L);
bar_status read_state(bar_matrix A, cudaStream_t st);
// KernelTimer: bracket one sweep launch of global iteration m; after the stream has synchronised,
// add the launches with m <= bound (each worth `iters_each` global iterations) and reset.
void timer_reset(KernelTimer &T);
bar_status timer_begin(KernelTimer &T, int64_t m, cudaStream_t st);
bar_status timer_end(KernelTimer &T, cudaStream_t st);
bar_status timer_collect(KernelTimer &T, int64_t bound, double iters_each);
void timer_free(KernelTimer &T);

#define BAR_CUDA(call)                                              \
    do {                                                            \
        cudaError_t _e = (call);                                    \
        if (_e != cudaSuccess) return ::bar::cuda_fail(_e, #call);  \
    } while (0)

// Handles from bar_create_csr_dist (dist.cu): the collective solve / residual of one rank.
bar_status dist_solve_handle(bar_matrix A, const double *b, const double *x0, double *x, int32_t k,
                             int64_t max_global_iters, double tol, bar_mode mode, cudaStream_t st, bar_solve_info *info);
bar_status dist_residual_handle(bar_matrix A, const double *b, const double *x, cudaStream_t st, double *res_norm2,
                                double *b_norm2);
void dist_destroy_handle(bar_matrix A);
bar_status dist_sweep_handle(bar_matrix A, const double *b, double *x, int32_t k, int64_t nsweeps, bar_mode mode,
                             cudaStream_t st);

// Layout construction (layout.cu). rowptr/col/val are DEVICE pointers.
// Columns in [col_lo, col_hi) (default [0, n)); row i's diagonal is column i.
bar_status build_layout(Layout &L, int64_t n, int64_t nnz, const int32_t *d_rowptr, const int32_t *d_col,
                        const double *d_val, int32_t R, cudaStream_t st, int64_t col_lo = 0, int64_t col_hi = -1);
void free_layout(Layout &L);

// Kernel launchers (sweep.cu). All pointers are device pointers.
struct SweepArgs {
    const Layout *L;
    const double *b;
    const double *x_in;
    double *x_out;
    int k;
    DevState *state;
    double *partials;
    double *hist;  // nullable device array: hist[m-1] = rel_res(x^(m-1)) (sync modes)
    double *dist_out = nullptr;  // multi-GPU: receives this rank's [sum r^2, sum b^2]
    const uint8_t *frozen = nullptr;  // N1: rows that do not update in this launch (nullable)
    double tau = 1.0;                 // N3: relaxation weight, B = I - tau D^-1 A
    long long m0 = 0;                 // single-launch async: global iteration of the first sweep
    int64_t l_begin = 0, l_end = 0;   // sweep only subdomains [l_begin, l_end) (l_end = 0: all);
                                      // cudaErrorNotSupported where the chosen kernel cannot
    const int *stop = nullptr;        // stop flag polled by the kernels (nullptr: state->stop)
    double *ring = nullptr;           // single-launch resident kernel, lazy publication:
    double *bsum_arr = nullptr;       //   Workspace::ring / bsum_arr (nullptr: the blocking path)
};
int64_t num_blocks_for(const Layout &L, bar_mode mode);
int64_t rowwise_grid(const Layout &L);
cudaError_t launch_sweep(const SweepArgs &a, bar_mode mode, cudaStream_t st);
// Fully asynchronous persistent solve: claims [work, w_end) = global iterations up to w_end / q
// in ONE launch; cudaErrorNotSupported when the layout/vectors do not fit the staged kernel.
cudaError_t launch_async_multi(const SweepArgs &a, long long w_end, cudaStream_t st);
// init_check: the last block also applies k_init_check's rule (one launch fewer on the
// single-launch async path)
cudaError_t launch_residual(const Layout &L, const double *b, const double *x, DevState *state,
                            double *partials, cudaStream_t st, double *dist_out = nullptr, bool init_check = false);
// Multi-GPU helpers (sweep.cu): gather the values peers need; apply the stopping rule to the
// rank-ordered sum of every rank's [sum r^2, sum b^2] (identical decision on every rank).
cudaError_t launch_pack(const double *x_own, const int32_t *idx, int64_t cnt, double *out, cudaStream_t st);
cudaError_t launch_dist_decide(DevState *state, const double *gathered, int nranks, bool residual_only,
                               cudaStream_t st);
// exact residual of x^(0) = 0 without the SpMV: b - A 0 = b, so ||r||_2 = ||b||_2 and rel_res = 1
// (0 for b = 0) — a read of b instead of the matrix (x0 == NULL in bar_solve)
cudaError_t launch_zero_start_residual(const Layout &L, const double *b, DevState *state, double *partials,
                                       cudaStream_t st, bool init_check = false);
cudaError_t launch_check_finite(const double *v, int64_t n, int *flag, cudaStream_t st);
cudaError_t launch_init_state(DevState *state, double tol, cudaStream_t st);
// after the exact residual of x^(0): init_rel = exact_rel; if x^(0) already meets tol (or b = 0,
// or it is not finite) raise stop and close the work queue, so a following single-launch async
// kernel returns at once — the x^(0) check without a host round trip
cudaError_t launch_init_check(DevState *state, cudaStream_t st);
// reopen a closed async queue; clear_slots: also zero the per-iteration residual slots
// (k_block_resident restarts every block at the last completed iteration)
cudaError_t launch_resume_queue(DevState *state, cudaStream_t st, bool clear_slots = false);
// after an aborted single-launch solve (DevState::aborted): iter = iters_done, stop / aborted cleared
cudaError_t launch_continue_per_launch(DevState *state, cudaStream_t st);

}  // namespace bar
