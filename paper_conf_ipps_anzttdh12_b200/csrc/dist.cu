// dist.cu — multi-GPU row-partitioned solve (include/bar.h "multi-GPU").
//
// Paper: §3.4 splits the system into row blocks per device, then per thread block,
// with an asynchronous iteration between devices; its data paths (AMC through host memory,
// DC/DK through a master GPU) were PCIe workarounds. Here every rank keeps its own rows and
// reads the x values it does not own ("ghosts") in one of two ways:
//
//   * collective (sync-block, Jacobi; async with p2p off): once per global iteration an NCCL
//     grouped send/recv (or one ncclAllGather) refreshes the ghost slots, the per-rank residual
//     sums are all-gathered and summed in rank order, so every rank applies the same stopping
//     rule to the same bits;
//   * peer memory (async, the default when every rank can map every other rank's memory): each
//     rank PULLS its ghosts from the owners' live iterates with relaxed system-scope loads
//     before every local sweep and pushes its residual partial into every rank's "board" (a
//     small array in each rank's device memory, mapped by all ranks through CUDA IPC). There is
//     no collective and no barrier while iterating (the paper's DK idea, without a master
//     GPU): stop requests travel as tagged words through the boards, and the ranks meet only to
//     confirm the stop with an exact residual (a board barrier, below).
//
// Local vector ("extended x"): [pad | ghosts below | owned rows | ghosts above]; the owned
// block starts 16-byte aligned and every kernel indexes it with columns relative to the owned
// block (ghosts below negative), which keeps each row's entries in their global order: the
// per-row arithmetic, and so every sync-block / Jacobi iterate, is bitwise the one-GPU result.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstring>
#include <vector>

#include "bar_internal.cuh"

#ifdef BAR_WITH_NCCL
#include <nccl.h>
#endif

// Board of rank r (device memory of r, mapped by every rank), in 8-byte words, P ranks:
//   [0, 2P)    part:    latest [sum r^2, sum b^2] estimate partial of each rank (async iteration)
//   [2P, 3P)   stopreq: u64 tag of the latest stop request of each rank (>= the phase tag: stop)
//   [3P, 4P)   arrive:  u64 latest board-barrier epoch each rank has reached
//   [4P, 8P)   exact:   [sum r^2, sum b^2, global iterations, launches issued] of each rank, published
//                       with an arrival
constexpr int kBoardWordsPerRank = 8;

struct bar_dist_s {
    bar_matrix A = nullptr;  // local layout: n_local rows, columns [-n_glo, n_local + n_ghi)
    int rank = 0, nranks = 1, device = 0;
    int64_t n_global = 0, row_begin = 0, row_end = 0, n_local = 0, n_glo = 0, n_ghi = 0;
    int64_t glo_pad = 0, ext = 0;  // owned block offset in the extended vector; its length
    double *xa = nullptr, *xb = nullptr;  // extended iterate buffers
    double *bbuf = nullptr;               // owned b (device)
    int32_t *send_idx = nullptr;          // device, local row indices
    double *send_buf = nullptr;           // device
    int64_t n_send = 0;
    std::vector<int64_t> send_cnt, send_off, recv_cnt, recv_pos;  // recv_pos: owned-relative index
    double *part = nullptr;      // device [2]: this rank's [sum r^2, sum b^2]
    // halo exchange by ncclAllGather (bar_tuning.halo = 1): every rank packs its send buffer into
    // its slot of ag_buf (ag_max doubles per rank) and the gather runs in place; each receiver
    // copies its segment of every sender p out of slot p (peer_off[p] = where p's segment for this
    // rank starts). Planned on the first exchange.
    bool ag_ready = false;
    int64_t ag_max = 0;
    double *ag_buf = nullptr;  // device [nranks * ag_max]
    std::vector<int64_t> peer_off;
    double *gathered = nullptr;  // device [2 * nranks]
    // peer memory (bar_dist_enable_p2p)
    bool p2p = false;
    int32_t *g_rank = nullptr, *g_idx = nullptr;  // device, per ghost: owner rank, owner-local row
    double **d_peer_own = nullptr;                // device [nranks]: owned block of each rank's x
    double **d_peer_board = nullptr;              // device [nranks]: each rank's board
    double *board = nullptr;                      // device [kBoardWordsPerRank * nranks]
    double *h_exact = nullptr;                    // pinned host copy of the board's exact section
    uint64_t epoch = 0;                           // board barriers passed (the same on every rank)
    std::vector<void *> opened;                   // IPC mappings to close
    bool loopback = false;                        // ranks of one process, linked (bar_dist_link_loopback)
    bool has_nccl = false;
    bool owner_handle = false;                    // A was returned by bar_create_csr_dist (A->dist == this)
    // interior / boundary overlap of the collective path: subdomains [ib, ie) read no ghost, so
    // they are swept on a second stream while the halo exchange runs; the boundary ones follow it
    int64_t ib = 0, ie = 0;                       // interior subdomains (ib >= ie: none)
    cudaStream_t s2 = nullptr;                    // interior stream
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    bar::DevState *state2 = nullptr;              // the interior launches' reduction state
    double *partials2 = nullptr;                  // and per-block partials
    double *parts3 = nullptr;                     // device [6]: [lo | interior | hi] partial sums
    std::vector<bar_dist> peers;                  // loopback group (peers[r] is rank r)
#ifdef BAR_WITH_NCCL
    ncclComm_t comm = nullptr;
#endif
};

namespace bar {
namespace {

constexpr unsigned long long kBarrierTimeoutNs = 20ull * 1000 * 1000 * 1000;  // 20 s: a peer is gone

bar_status nccl_fail(int code, const char *what) {
#ifdef BAR_WITH_NCCL
    set_error(std::string(what) + ": " + ncclGetErrorString((ncclResult_t)code));
#else
    (void)code;
    set_error(std::string(what) + ": libbar was built without NCCL");
#endif
    return BAR_ERR_NCCL;
}

#ifdef BAR_WITH_NCCL
#define BAR_NCCL(call)                                                  \
    do {                                                                \
        ncclResult_t _r = (call);                                       \
        if (_r != ncclSuccess) return ::bar::nccl_fail((int)_r, #call); \
    } while (0)
#endif

template <class T>
bar_status to_device(const T *src, int64_t count, T **dst) {
    BAR_CUDA(cudaMalloc((void **)dst, sizeof(T) * (size_t)(count > 0 ? count : 1)));
    if (count > 0) BAR_CUDA(cudaMemcpy(*dst, src, sizeof(T) * (size_t)count, cudaMemcpyDefault));
    return BAR_OK;
}

template <class T>
std::vector<T> to_host(const T *src, int64_t count, bar_status &st) {
    std::vector<T> h((size_t)(count > 0 ? count : 0));
    if (count > 0 && cudaMemcpy(h.data(), src, sizeof(T) * (size_t)count, cudaMemcpyDefault) != cudaSuccess)
        st = cuda_fail(cudaGetLastError(), "copy to host");
    return h;
}

double *own(const bar_dist D, double *ext) { return ext + D->glo_pad; }

// ---- system-scope accesses to boards (own and peers') ----------------------------------------
__device__ __forceinline__ double ld_relaxed_sys(const double *p) {
    double v;
    asm volatile("ld.relaxed.sys.global.f64 %0, [%1];" : "=d"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed_sys(double *p, double v) {
    asm volatile("st.relaxed.sys.global.f64 [%0], %1;" ::"l"(p), "d"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_relaxed_sys_u64(const void *p) {
    unsigned long long v;
    asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long ld_acquire_sys_u64(const void *p) {
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed_sys_u64(void *p, unsigned long long v) {
    asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_release_sys_u64(void *p, unsigned long long v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long now_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

// Pull every ghost value from its owner's live iterate: x "as it stands" (eq. 3), read over
// NVLink with relaxed system-scope loads, no synchronisation with the owner.
__global__ void k_pull_ghosts(double *__restrict__ x_own, int64_t n_glo, int64_t n_local, int64_t n_ghost,
                              const int32_t *__restrict__ g_rank, const int32_t *__restrict__ g_idx,
                              double *const *__restrict__ peer_own) {
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n_ghost;
         j += (int64_t)gridDim.x * blockDim.x) {
        const double *src = peer_own[g_rank[j]] + g_idx[j];
        const double v = ld_relaxed_sys(src);
        double *dst = j < n_glo ? x_own - n_glo + j : x_own + n_local + (j - n_glo);
        asm volatile("st.relaxed.gpu.global.f64 [%0], %1;" ::"l"(dst), "d"(v) : "memory");
    }
}

// After a local async sweep (single thread): push this rank's partial into slot `rank` of every
// board, estimate the global residual from this rank's board (rank-ordered sum; other ranks'
// entries may be a few sweeps old — the estimate of eq. 3's shifted iterate), apply the stopping
// rule, and exchange stop requests: a rank that stops tags every board's stopreq[rank] with the
// phase tag; a rank that finds a request carrying the current tag stops too. No waiting.
__global__ void k_p2p_publish_decide(DevState *S, const double *__restrict__ part, double *const *peer_board,
                                     const double *board, int rank, int P, unsigned long long tag) {
    if (*(volatile int *)&S->stop) return;  // launches queued after the stop swept nothing
    const double p0 = part[0], p1 = part[1];
    for (int p = 0; p < P; ++p) {
        st_relaxed_sys(peer_board[p] + 2 * rank, p0);
        st_relaxed_sys(peer_board[p] + 2 * rank + 1, p1);
    }
    double ss = 0.0, bsq = 0.0;
    for (int r = 0; r < P; ++r) {
        ss += ld_relaxed_sys(board + 2 * r);
        bsq += ld_relaxed_sys(board + 2 * r + 1);
    }
    // ++iter; stop when the estimate meets tol (or diverges: the exact residual decides)
    const long long m = ++S->iter;
    const double bn = sqrt(bsq);
    const double rel = bn != 0.0 ? sqrt(ss) / bn : 0.0;
    S->last_rel = rel;
    S->bnorm = bn;
    bool stop = bn == 0.0 || !isfinite(rel) || rel > 1e30 || rel <= S->tol;
    if (stop) {
        for (int p = 0; p < P; ++p) st_relaxed_sys_u64(peer_board[p] + 2 * P + rank, tag);
    } else {
        for (int r = 0; r < P && !stop; ++r) stop = ld_relaxed_sys_u64(board + 2 * P + r) >= tag;
    }
    if (stop) {
        S->stop = 1;
        S->conv_iter = m;
    }
}

// Board barrier (single thread). publish: write the payload [sum r^2, sum b^2, iters] (optional)
// into every board's exact section, then RELEASE this rank's arrival epoch into every board;
// wait: ACQUIRE every rank's arrival in this rank's board until all reached `epoch`. A wait longer
// than the timeout sets S->aborted = 2 (a peer is gone) instead of hanging the device.
__global__ void k_board_barrier(DevState *S, const double *board, double *const *peer_board, int rank, int P,
                                unsigned long long epoch, const double *payload, double issued, int publish, int wait) {
    if (publish) {
        if (payload) {
            const double a = payload[0], b = payload[1], it = (double)S->iter;
            for (int p = 0; p < P; ++p) {
                double *ex = peer_board[p] + 4 * P + 4 * rank;
                st_relaxed_sys(ex, a);
                st_relaxed_sys(ex + 1, b);
                st_relaxed_sys(ex + 2, it);
                st_relaxed_sys(ex + 3, issued);
            }
        }
        for (int p = 0; p < P; ++p) st_release_sys_u64(peer_board[p] + 3 * P + rank, epoch);
    }
    if (wait) {
        const unsigned long long t0 = now_ns();
        for (int r = 0; r < P; ++r) {
            while (ld_acquire_sys_u64(board + 3 * P + r) < epoch) {
                if (now_ns() - t0 > kBarrierTimeoutNs) {
                    S->aborted = 2;
                    return;
                }
                __nanosleep(256);
            }
        }
    }
}

// Start of a peer-memory solve: this rank's estimate slots read "unknown" (huge partials keep
// the estimate above tol until every rank has published once).
__global__ void k_board_reset(double *board, int P) {
    for (int i = threadIdx.x; i < 2 * P; i += blockDim.x) board[i] = 1e300;
}

// Overlap: this rank's [sum r^2, sum b^2] from the three launches, in a fixed order.
__global__ void k_sum_parts(const double *__restrict__ p3, const bar::DevState *S, double *__restrict__ part) {
    if (S->stop) return;  // queued iterations after the stop: nothing was swept
    part[0] = (p3[0] + p3[2]) + p3[4];
    part[1] = (p3[1] + p3[3]) + p3[5];
}

// ---- planning (host) -----------------------------------------------------------------------
// Sorted distinct ghost columns of a row block: those below row_begin, then those >= row_end.
void ghost_lists(int64_t row_begin, int64_t row_end, int64_t nnz_local, const int32_t *col, std::vector<int32_t> &lo,
                 std::vector<int32_t> &hi) {
    lo.clear();
    hi.clear();
    for (int64_t e = 0; e < nnz_local; ++e) {
        const int64_t c = col[e];
        if (c < row_begin) lo.push_back((int32_t)c);
        else if (c >= row_end) hi.push_back((int32_t)c);
    }
    std::sort(lo.begin(), lo.end());
    lo.erase(std::unique(lo.begin(), lo.end()), lo.end());
    std::sort(hi.begin(), hi.end());
    hi.erase(std::unique(hi.begin(), hi.end()), hi.end());
}

// The exchange plan of `rank` from every rank's row range and sorted ghost list (ghosts_all =
// the lists concatenated in rank order): recv_counts[p] = how many of this rank's ghosts p owns
// (consecutive in ghost order), send_counts[p] / send_idx = the owned rows p needs (local index,
// in p's ghost order), ghost_src[j] = owner-local row of this rank's ghost j.
bar_status plan(int P, int rank, const int64_t *ranges, const int64_t *gcount, const int32_t *ghosts_all,
                std::vector<int64_t> &recv_counts, std::vector<int64_t> &send_counts, std::vector<int32_t> &send_idx,
                std::vector<int32_t> &ghost_src) {
    std::vector<int64_t> goff(P + 1, 0);
    for (int p = 0; p < P; ++p) goff[p + 1] = goff[p] + gcount[p];
    auto owner = [&](int64_t c) -> int {
        for (int p = 0; p < P; ++p)
            if (c >= ranges[2 * p] && c < ranges[2 * p + 1]) return p;
        return -1;
    };
    recv_counts.assign(P, 0);
    send_counts.assign(P, 0);
    send_idx.clear();
    ghost_src.clear();
    int last = -1;
    for (int64_t j = goff[rank]; j < goff[rank + 1]; ++j) {
        const int64_t c = ghosts_all[j];
        const int o = owner(c);
        if (o < 0 || o == rank || o < last) {
            set_error("ghost column not owned by another rank (or ghost list not sorted by owner)");
            return BAR_ERR_INVALID_ARG;
        }
        last = o;
        ++recv_counts[o];
        ghost_src.push_back((int32_t)(c - ranges[2 * o]));
    }
    const int64_t b0 = ranges[2 * rank], b1 = ranges[2 * rank + 1];
    for (int p = 0; p < P; ++p) {
        if (p == rank) continue;
        for (int64_t j = goff[p]; j < goff[p + 1]; ++j) {
            const int64_t c = ghosts_all[j];
            if (c >= b0 && c < b1) {
                send_idx.push_back((int32_t)(c - b0));
                ++send_counts[p];
            }
        }
    }
    return BAR_OK;
}

bar_status localize(int64_t row_begin, int64_t row_end, int64_t nnz_local, const int32_t *col,
                    const std::vector<int32_t> &lo, const std::vector<int32_t> &hi, int32_t *col_local) {
    const int64_t nl = row_end - row_begin, nlo = (int64_t)lo.size();
    for (int64_t e = 0; e < nnz_local; ++e) {
        const int64_t c = col[e];
        if (c < row_begin) {
            auto it = std::lower_bound(lo.begin(), lo.end(), (int32_t)c);
            if (it == lo.end() || *it != c) {
                set_error("column missing from the ghost list");
                return BAR_ERR_INVALID_ARG;
            }
            col_local[e] = (int32_t)(-nlo + (it - lo.begin()));
        } else if (c >= row_end) {
            auto it = std::lower_bound(hi.begin(), hi.end(), (int32_t)c);
            if (it == hi.end() || *it != c) {
                set_error("column missing from the ghost list");
                return BAR_ERR_INVALID_ARG;
            }
            col_local[e] = (int32_t)(nl + (it - hi.begin()));
        } else {
            col_local[e] = (int32_t)(c - row_begin);
        }
    }
    return BAR_OK;
}

// ---- halo exchange and reductions of the collective path -------------------------------------

// All-gather halo plan: the largest send buffer of the group and, for this rank, the offset of
// its segment in every sender's buffer (NCCL: one all-gather of the send counts at first use;
// loopback: read from the linked peers).
bar_status plan_allgather(bar_dist *ranks, int nr, cudaStream_t st) {
    for (int i = 0; i < nr; ++i) {
        bar_dist D = ranks[i];
        if (D->ag_ready) continue;
        const int P = D->nranks;
        std::vector<int64_t> cnt((size_t)P * P, 0);  // cnt[p * P + d]: what p sends to d
        if (!D->has_nccl) {
            for (int p = 0; p < P; ++p)
                for (int d = 0; d < P; ++d) cnt[(size_t)p * P + d] = D->peers[p]->send_cnt[d];
        } else {
#ifdef BAR_WITH_NCCL
            int64_t *dev = nullptr;
            BAR_CUDA(cudaMalloc(&dev, sizeof(int64_t) * (size_t)P * (P + 1)));
            BAR_CUDA(cudaMemcpyAsync(dev, D->send_cnt.data(), sizeof(int64_t) * P, cudaMemcpyHostToDevice, st));
            BAR_NCCL(ncclAllGather(dev, dev + P, (size_t)P, ncclInt64, D->comm, st));
            BAR_CUDA(cudaMemcpyAsync(cnt.data(), dev + P, sizeof(int64_t) * (size_t)P * P, cudaMemcpyDeviceToHost, st));
            BAR_CUDA(cudaStreamSynchronize(st));
            cudaFree(dev);
#else
            return nccl_fail(0, "plan_allgather");
#endif
        }
        D->ag_max = 1;
        D->peer_off.assign(P, 0);
        for (int p = 0; p < P; ++p) {
            int64_t tot = 0, off = 0;
            for (int d = 0; d < P; ++d) {
                if (d == D->rank) off = tot;
                tot += cnt[(size_t)p * P + d];
            }
            D->peer_off[p] = off;
            if (tot > D->ag_max) D->ag_max = tot;
            if (cnt[(size_t)p * P + D->rank] != D->recv_cnt[p]) {
                set_error("all-gather plan mismatch: send/recv counts differ");
                return BAR_ERR_INVALID_ARG;
            }
        }
        if (D->n_send > D->ag_max) {  // cannot happen: ag_max is the largest send total
            set_error("all-gather plan: send count exceeds the slot size");
            return BAR_ERR_INVALID_ARG;
        }
        BAR_CUDA(cudaMalloc(&D->ag_buf, sizeof(double) * (size_t)P * D->ag_max));
        D->ag_ready = true;
    }
    return BAR_OK;
}

// Refresh the ghost slots of the extended vector `ext` of every rank in `ranks` (NCCL: the
// calling rank only; loopback: all ranks of the process, in order, on one stream).
bar_status exchange(bar_dist *ranks, int nr, double *const *ext, cudaStream_t st) {
    if (ranks[0]->A->L.tune.halo == 1) {  // one in-place ncclAllGather of every rank's packed slot
        bar_status r = plan_allgather(ranks, nr, st);
        if (r != BAR_OK) return r;
        const int P = ranks[0]->nranks;
        const int64_t M = ranks[0]->ag_max;
        for (int i = 0; i < nr; ++i) {
            bar_dist D = ranks[i];
            BAR_CUDA(launch_pack(own(D, ext[i]), D->send_idx, D->n_send, D->ag_buf + (size_t)D->rank * M, st));
        }
        if (ranks[0]->has_nccl) {
#ifdef BAR_WITH_NCCL
            bar_dist D = ranks[0];
            BAR_NCCL(ncclAllGather(D->ag_buf + (size_t)D->rank * M, D->ag_buf, (size_t)M, ncclDouble, D->comm, st));
#else
            return nccl_fail(0, "exchange");
#endif
        } else {  // loopback: assemble the same gathered buffer by copies into every rank's ag_buf
            for (int i = 0; i < nr; ++i)
                for (int p = 0; p < P; ++p)
                    if (p != i && ranks[p]->n_send)
                        BAR_CUDA(cudaMemcpyAsync(ranks[i]->ag_buf + (size_t)p * M, ranks[p]->ag_buf + (size_t)p * M,
                                                 sizeof(double) * (size_t)ranks[p]->n_send, cudaMemcpyDeviceToDevice,
                                                 st));
        }
        for (int i = 0; i < nr; ++i) {  // each receiver: its segment of every sender's slot
            bar_dist D = ranks[i];
            for (int p = 0; p < P; ++p) {
                if (p == D->rank || !D->recv_cnt[p]) continue;
                BAR_CUDA(cudaMemcpyAsync(own(D, ext[i]) + D->recv_pos[p], D->ag_buf + (size_t)p * M + D->peer_off[p],
                                         sizeof(double) * (size_t)D->recv_cnt[p], cudaMemcpyDeviceToDevice, st));
            }
        }
        return BAR_OK;
    }
    for (int i = 0; i < nr; ++i) {
        bar_dist D = ranks[i];
        BAR_CUDA(launch_pack(own(D, ext[i]), D->send_idx, D->n_send, D->send_buf, st));
    }
    if (ranks[0]->has_nccl) {
#ifdef BAR_WITH_NCCL
        bar_dist D = ranks[0];
        double *xo = own(D, ext[0]);
        BAR_NCCL(ncclGroupStart());
        for (int p = 0; p < D->nranks; ++p) {
            if (p == D->rank) continue;
            if (D->send_cnt[p])
                BAR_NCCL(ncclSend(D->send_buf + D->send_off[p], (size_t)D->send_cnt[p], ncclDouble, p, D->comm, st));
            if (D->recv_cnt[p])
                BAR_NCCL(ncclRecv(xo + D->recv_pos[p], (size_t)D->recv_cnt[p], ncclDouble, p, D->comm, st));
        }
        BAR_NCCL(ncclGroupEnd());
        return BAR_OK;
#else
        return nccl_fail(0, "exchange");
#endif
    }
    for (int i = 0; i < nr; ++i) {  // loopback: receiver i pulls from every sender p
        bar_dist D = ranks[i];
        for (int p = 0; p < nr; ++p) {
            if (p == i || !D->recv_cnt[p]) continue;
            bar_dist S = ranks[p];
            if (S->send_cnt[i] != D->recv_cnt[p]) {
                set_error("loopback plan mismatch: send/recv counts differ");
                return BAR_ERR_INVALID_ARG;
            }
            BAR_CUDA(cudaMemcpyAsync(own(D, ext[i]) + D->recv_pos[p], S->send_buf + S->send_off[i],
                                     sizeof(double) * (size_t)D->recv_cnt[p], cudaMemcpyDeviceToDevice, st));
        }
    }
    return BAR_OK;
}

// All-gather the per-rank partial sums and apply the stopping rule on every rank.
bar_status reduce_decide(bar_dist *ranks, int nr, bool residual_only, cudaStream_t st) {
    if (ranks[0]->has_nccl) {
#ifdef BAR_WITH_NCCL
        bar_dist D = ranks[0];
        BAR_NCCL(ncclAllGather(D->part, D->gathered, 2, ncclDouble, D->comm, st));
        BAR_CUDA(launch_dist_decide(D->A->W.state, D->gathered, D->nranks, residual_only, st));
        return BAR_OK;
#else
        return nccl_fail(0, "reduce");
#endif
    }
    bar_dist D0 = ranks[0];
    for (int i = 0; i < nr; ++i)
        BAR_CUDA(cudaMemcpyAsync(D0->gathered + 2 * i, ranks[i]->part, 2 * sizeof(double), cudaMemcpyDeviceToDevice,
                                 st));
    for (int i = 0; i < nr; ++i) {
        if (i) BAR_CUDA(cudaMemcpyAsync(ranks[i]->gathered, D0->gathered, 2 * sizeof(double) * nr,
                                        cudaMemcpyDeviceToDevice, st));
        BAR_CUDA(launch_dist_decide(ranks[i]->A->W.state, ranks[i]->gathered, nr, residual_only, st));
    }
    return BAR_OK;
}

// ---- peer memory ---------------------------------------------------------------------------

bar_status pull_ghosts(bar_dist D, cudaStream_t st) {
    const int64_t ng = D->n_glo + D->n_ghi;
    if (ng <= 0) return BAR_OK;
    int64_t blocks = (ng + 255) / 256;
    if (blocks > 1024) blocks = 1024;
    k_pull_ghosts<<<(unsigned)blocks, 256, 0, st>>>(own(D, D->xa), D->n_glo, D->n_local, ng, D->g_rank, D->g_idx,
                                                     D->d_peer_own);
    BAR_CUDA(cudaGetLastError());
    return BAR_OK;
}

// Every rank of `ranks` passes the next board-barrier epoch (optionally publishing its payload
// [sum r^2, sum b^2] from D->part, its iterations and `issued` launches). Separate processes: one
// publish+wait launch per rank; the loopback group (one stream): all publishes, then all waits.
bar_status board_barrier(bar_dist *ranks, int nr, bool payload, cudaStream_t st, int64_t issued = 0) {
    const bool split = ranks[0]->loopback;
    for (int i = 0; i < nr; ++i) {
        bar_dist D = ranks[i];
        ++D->epoch;
        k_board_barrier<<<1, 1, 0, st>>>(D->A->W.state, D->board, D->d_peer_board, D->rank, D->nranks, D->epoch,
                                          payload ? D->part : nullptr, (double)issued, 1, split ? 0 : 1);
        BAR_CUDA(cudaGetLastError());
    }
    if (split)
        for (int i = 0; i < nr; ++i) {
            bar_dist D = ranks[i];
            k_board_barrier<<<1, 1, 0, st>>>(D->A->W.state, D->board, D->d_peer_board, D->rank, D->nranks, D->epoch,
                                              nullptr, 0.0, 0, 1);
            BAR_CUDA(cudaGetLastError());
        }
    return BAR_OK;
}

// Confirming residual of the peer-memory path: all ranks stopped sweeping (barrier), pull the
// now-frozen ghosts, exact residual partials, publish them with the next barrier; every rank
// then sums the board's exact section in rank order on the host (the same bits everywhere).
bar_status p2p_exact(bar_dist *ranks, int nr, double *const *xv, cudaStream_t st, double &ss, double &bsq,
                     int64_t &it_min, int64_t &it_max, int64_t issued, int64_t &issued_min) {
    NvtxRange nv("peer memory: barrier, ghost pull, exact residual, barrier");
    bar_status r;
    if ((r = board_barrier(ranks, nr, false, st)) != BAR_OK) return r;
    for (int i = 0; i < nr; ++i) {
        bar_dist D = ranks[i];
        if ((r = pull_ghosts(D, st)) != BAR_OK) return r;
        BAR_CUDA(launch_residual(D->A->L, D->bbuf, own(D, xv[i]), D->A->W.state, D->A->W.partials, st, D->part));
    }
    if ((r = board_barrier(ranks, nr, true, st, issued)) != BAR_OK) return r;
    bar_dist D0 = ranks[0];
    const int P = D0->nranks;
    BAR_CUDA(cudaMemcpyAsync(D0->h_exact, D0->board + 4 * P, sizeof(double) * 4 * (size_t)P, cudaMemcpyDeviceToHost,
                             st));
    for (int i = 0; i < nr; ++i)
        if ((r = read_state(ranks[i]->A, st)) != BAR_OK) return r;
    for (int i = 0; i < nr; ++i)
        if (ranks[i]->A->W.h_state->aborted == 2) {
            set_error("peer-memory barrier timed out (a rank stopped participating)");
            return BAR_ERR_NCCL;
        }
    ss = bsq = 0.0;
    it_min = issued_min = INT64_MAX;
    it_max = 0;
    for (int p = 0; p < P; ++p) {
        ss += D0->h_exact[4 * p];
        bsq += D0->h_exact[4 * p + 1];
        const int64_t it = (int64_t)D0->h_exact[4 * p + 2];
        it_min = std::min(it_min, it);
        it_max = std::max(it_max, it);
        issued_min = std::min(issued_min, (int64_t)D0->h_exact[4 * p + 3]);
    }
    return BAR_OK;
}

void fill_info(bar_solve_info *info, bar_dist *ranks, int nr, int64_t iters, int64_t it_max, double rel,
               int converged, int64_t launches, const KernelTimer &T) {
    if (!info) return;
    info->iters = iters;
    info->rel_res = rel;
    info->converged = converged;
    info->cta_iters_min = iters;
    info->cta_iters_max = it_max > iters ? it_max : iters;
    double mb = 0.0;
    for (int i = 0; i < nr; ++i) mb += model_bytes(ranks[i]->A->L);
    info->model_bytes_per_iter = mb;
    info->kernel_launches = launches;
    info->sweep_kernel_ms = T.ms;
    info->sweep_kernel_iters = T.iters;
}

// Lazily created resources of the overlapped iteration (collective or peer-memory path).
bar_status ensure_overlap(bar_dist D) {
    if (D->s2) return BAR_OK;
    BAR_CUDA(cudaStreamCreateWithFlags(&D->s2, cudaStreamNonBlocking));
    BAR_CUDA(cudaEventCreateWithFlags(&D->ev_fork, cudaEventDisableTiming));
    BAR_CUDA(cudaEventCreateWithFlags(&D->ev_join, cudaEventDisableTiming));
    BAR_CUDA(cudaMalloc(&D->state2, sizeof(DevState)));
    BAR_CUDA(cudaMemset(D->state2, 0, sizeof(DevState)));
    BAR_CUDA(cudaMalloc(&D->partials2, sizeof(double) * 2 * (size_t)num_blocks_for(D->A->L, BAR_MODE_SYNC_BLOCK)));
    BAR_CUDA(cudaMalloc(&D->parts3, sizeof(double) * 6));
    return BAR_OK;
}

// One global iteration with the interior subdomains swept on the second stream while the halo
// arrives (every rank of `ranks`): fork -> interior sweeps on s2 || exchange (collective) or
// ghost pull (peer memory) + low and high boundary sweeps on st -> join -> partial sums.
// supported = false (nothing enqueued) where the sweep kernel cannot take subdomain ranges.
bar_status overlapped_iteration(bar_dist *ranks, int nr, double *const *vin, double *const *vout, int32_t k,
                                bar_mode mode, cudaStream_t st, bool &supported, bool p2p = false) {
    bar_status r;
    supported = true;
    for (int i = 0; i < nr; ++i) {
        bar_dist D = ranks[i];
        if ((r = ensure_overlap(D)) != BAR_OK) return r;
        BAR_CUDA(cudaEventRecord(D->ev_fork, st));
        BAR_CUDA(cudaStreamWaitEvent(D->s2, D->ev_fork, 0));
        SweepArgs a{&D->A->L, D->bbuf, own(D, vin[i]), own(D, vout[i]), k, D->state2, D->partials2, nullptr,
                    D->parts3 + 2};
        a.l_begin = D->ib;
        a.l_end = D->ie;
        a.stop = &D->A->W.state->stop;
        const cudaError_t e = launch_sweep(a, mode, D->s2);
        if (e == cudaErrorNotSupported) {
            cudaGetLastError();
            supported = false;
            return BAR_OK;
        }
        BAR_CUDA(e);
        BAR_CUDA(cudaEventRecord(D->ev_join, D->s2));
    }
    if (p2p) {  // peer memory: pull the ghosts as they stand while the interior sweeps run
        for (int i = 0; i < nr; ++i)
            if ((r = pull_ghosts(ranks[i], st)) != BAR_OK) return r;
    } else if ((r = exchange(ranks, nr, vin, st)) != BAR_OK) {
        return r;
    }
    for (int i = 0; i < nr; ++i) {
        bar_dist D = ranks[i];
        const int64_t q = D->A->L.q;
        for (int side = 0; side < 2; ++side) {
            SweepArgs a{&D->A->L, D->bbuf, own(D, vin[i]), own(D, vout[i]), k, D->A->W.state, D->A->W.partials,
                        nullptr, D->parts3 + (side ? 4 : 0)};
            a.l_begin = side ? D->ie : 0;
            a.l_end = side ? q : D->ib;
            if (a.l_end <= a.l_begin) {  // empty side: a zero partial
                BAR_CUDA(cudaMemsetAsync(D->parts3 + (side ? 4 : 0), 0, 2 * sizeof(double), st));
                continue;
            }
            BAR_CUDA(launch_sweep(a, mode, st));
        }
        BAR_CUDA(cudaStreamWaitEvent(st, D->ev_join, 0));
        k_sum_parts<<<1, 1, 0, st>>>(D->parts3, D->A->W.state, D->part);
        BAR_CUDA(cudaGetLastError());
    }
    return BAR_OK;
}

// async-(k) across ranks over peer memory: per global iteration and rank, pull ghosts, sweep,
// publish + decide — no collective, no barrier; then the confirming residual (board barriers).
bar_status p2p_solve(bar_dist *ranks, int nr, int32_t k, int64_t max_iters, double tol, cudaStream_t st,
                     bar_solve_info *info) {
    bar_status r;
    NvtxRange nv("dist async over peer memory");
    const int P = ranks[0]->nranks;
    for (int i = 0; i < nr; ++i) {
        k_board_reset<<<1, 32, 0, st>>>(ranks[i]->board, P);
        BAR_CUDA(cudaGetLastError());
    }
    if ((r = board_barrier(ranks, nr, false, st)) != BAR_OK) return r;  // boards reset, x set up
    for (int i = 0; i < nr; ++i) {  // a rank that never arrives: fail now, not after the iterations
        if ((r = read_state(ranks[i]->A, st)) != BAR_OK) return r;
        if (ranks[i]->A->W.h_state->aborted == 2) {
            set_error("peer-memory barrier timed out (a rank did not join the solve)");
            return BAR_ERR_NCCL;
        }
    }
    unsigned long long tag = ranks[0]->epoch;
    bar_dist D0 = ranks[0];
    DevState &H = *D0->A->W.h_state;
    KernelTimer &T = D0->A->W.timer;
    timer_reset(T);
    int64_t issued = 0, chunk = 8, launches = 2 * nr, iters = 0, it_max = 0;
    ChunkSizer sizer;
    double rel = 0.0;
    int converged = 0;
    bool diverged = false, bzero = false;
    std::vector<double *> xs(nr);
    for (int i = 0; i < nr; ++i) xs[i] = ranks[i]->xa;
    bool overlap = D0->A->L.tune.overlap >= 0 && P > 1;
    for (int i = 0; i < nr; ++i) overlap = overlap && ranks[i]->ib < ranks[i]->ie;
    for (;;) {
        bool stopped = false;
        while (issued < max_iters && !stopped) {
            const int64_t c = std::min(chunk, max_iters - issued);
            for (int64_t it = 0; it < c; ++it) {
                bool done = false;
                if (overlap) {  // interior sweeps on the second stream while the ghosts are pulled
                    if ((r = timer_begin(T, issued + it + 1, st)) != BAR_OK) return r;
                    bool supported = true;
                    if ((r = overlapped_iteration(ranks, nr, xs.data(), xs.data(), k, BAR_MODE_ASYNC, st, supported,
                                                  true)) != BAR_OK)
                        return r;
                    if ((r = timer_end(T, st)) != BAR_OK) return r;
                    done = supported;
                    if (!supported) {
                        overlap = false;
                        T.used = T.used > 0 ? T.used - 1 : 0;
                    }
                }
                for (int i = 0; i < nr; ++i) {
                    bar_dist D = ranks[i];
                    if (!done) {
                        if ((r = pull_ghosts(D, st)) != BAR_OK) return r;
                        SweepArgs a{&D->A->L, D->bbuf, own(D, D->xa), own(D, D->xa), k, D->A->W.state,
                                    D->A->W.partials, nullptr, D->part};
                        if (i == 0 && (r = timer_begin(T, issued + it + 1, st)) != BAR_OK) return r;
                        BAR_CUDA(launch_sweep(a, BAR_MODE_ASYNC, st));
                        if (i == 0 && (r = timer_end(T, st)) != BAR_OK) return r;
                    }
                    k_p2p_publish_decide<<<1, 1, 0, st>>>(D->A->W.state, D->part, D->d_peer_board, D->board, D->rank,
                                                          P, tag);
                    BAR_CUDA(cudaGetLastError());
                }
                launches += (done ? 6 : 3) * nr;  // overlapped: pull, three sweeps, sum, publish
            }
            issued += c;
            for (int i = nr - 1; i >= 0; --i) {  // loopback: the last rank's request reaches the others next time
                if ((r = read_state(ranks[i]->A, st)) != BAR_OK) return r;
                stopped = stopped || ranks[i]->A->W.h_state->stop != 0;
            }
            if ((r = timer_collect(T, (int64_t)H.iter, 1.0)) != BAR_OK) return r;
            chunk = sizer.next(chunk, (long long)H.iter, H.last_rel, tol);
        }
        double ss = 0.0, bsq = 0.0;
        int64_t it_min = 0, issued_min = 0;
        if ((r = p2p_exact(ranks, nr, xs.data(), st, ss, bsq, it_min, it_max, issued, issued_min)) != BAR_OK) return r;
        launches += 4 * nr;
        iters = it_min;
        const double bn = std::sqrt(bsq);
        rel = bn != 0.0 ? std::sqrt(ss) / bn : 0.0;
        if (bn == 0.0) bzero = true;
        else if (!std::isfinite(rel) || rel > 1e30) diverged = true;
        else converged = rel <= tol;
        // decided from the board's exact section only (the same bits on every rank; a rank's own
        // `stopped` / `issued` may differ from its peers'): done, or every rank has issued all
        // max_iters global iterations
        if (converged || diverged || bzero || issued_min >= max_iters) break;
        // an estimate met tol but the exact residual did not: every rank resumes
        for (int i = 0; i < nr; ++i) BAR_CUDA(cudaMemsetAsync(&ranks[i]->A->W.state->stop, 0, sizeof(int), st));
        tag = ranks[0]->epoch;  // older stop requests are stale now
        (void)stopped;
    }
    if (bzero) {
        for (int i = 0; i < nr; ++i)
            BAR_CUDA(cudaMemsetAsync(own(ranks[i], ranks[i]->xa), 0, sizeof(double) * (size_t)ranks[i]->n_local, st));
        iters = 0;
        rel = 0.0;
        converged = 1;
        diverged = false;
    }
    fill_info(info, ranks, nr, iters, it_max, rel, converged, launches, T);
    if (diverged) {
        set_error("relative residual became non-finite or exceeded 1e30");
        return BAR_ERR_DIVERGED;
    }
    return BAR_OK;
}

const char *overlap_name(bar_dist D, bar_mode mode) {
    if (mode == BAR_MODE_ASYNC) return "dist async, collective halo exchange";
    return D->ib < D->ie && D->A->L.tune.overlap >= 0 ? "dist sync, halo exchange overlapped with interior sweeps"
                                                       : "dist sync, halo exchange then sweep";
}

// The solve for the ranks this process drives (1 with NCCL / separate processes, all with
// loopback). b, x0, x are each rank's owned rows (device or host).
bar_status dist_solve(bar_dist *ranks, int nr, const double *const *b, const double *const *x0, double *const *x,
                      int32_t k, int64_t max_iters, double tol, bar_mode mode, cudaStream_t st,
                      bar_solve_info *info) {
    if ((mode != BAR_MODE_JACOBI && k < 1) || max_iters < 0 || !(tol >= 0.0) ||
        (mode != BAR_MODE_ASYNC && mode != BAR_MODE_SYNC_BLOCK && mode != BAR_MODE_JACOBI)) {
        set_error("need k >= 1, max_global_iters >= 0, tol >= 0, a valid mode");
        return BAR_ERR_INVALID_ARG;
    }
    if (mode == BAR_MODE_JACOBI) k = 1;
    bar_status r;
    bar_dist D0 = ranks[0];
    const bool p2p = mode == BAR_MODE_ASYNC && D0->p2p && D0->A->L.tune.peer >= 0;
    if (!p2p && !D0->loopback && !D0->has_nccl && D0->nranks > 1) {
        set_error("this rank has no NCCL communicator: only the peer-memory async mode is available");
        return BAR_ERR_INVALID_ARG;
    }
    DeviceGuard g(D0->device);
    std::vector<double *> xa(nr), xb(nr);
    for (int i = 0; i < nr; ++i) {
        bar_dist D = ranks[i];
        if ((r = ensure_workspace(D->A)) != BAR_OK) return r;
        const size_t nb = sizeof(double) * (size_t)D->n_local;
        BAR_CUDA(cudaMemcpyAsync(D->bbuf, b[i], nb, cudaMemcpyDefault, st));
        BAR_CUDA(cudaMemsetAsync(D->xa, 0, sizeof(double) * (size_t)D->ext, st));
        BAR_CUDA(cudaMemsetAsync(D->xb, 0, sizeof(double) * (size_t)D->ext, st));
        if (x0 && x0[i]) BAR_CUDA(cudaMemcpyAsync(own(D, D->xa), x0[i], nb, cudaMemcpyDefault, st));
        BAR_CUDA(launch_init_state(D->A->W.state, tol, st));
        xa[i] = D->xa;
        xb[i] = D->xb;
    }
    if (p2p) {
        if ((r = p2p_solve(ranks, nr, k, max_iters, tol, st, info)) != BAR_OK && r != BAR_ERR_DIVERGED) return r;
        for (int i = 0; i < nr; ++i)
            BAR_CUDA(cudaMemcpyAsync(x[i], own(ranks[i], ranks[i]->xa), sizeof(double) * (size_t)ranks[i]->n_local,
                                     cudaMemcpyDefault, st));
        BAR_CUDA(cudaStreamSynchronize(st));
        return r;
    }
    NvtxRange nv(overlap_name(D0, mode));
    int64_t launches = nr;
    DevState &H = *D0->A->W.h_state;
    // device time of the local sweeps of this process's first rank (bar_solve_info.sweep_kernel_*)
    KernelTimer &T = D0->A->W.timer;
    timer_reset(T);
    int64_t issued = 0, chunk = 8;
    ChunkSizer sizer;  // sized from the agreed state (identical on every rank)
    // interior / boundary overlap: every rank of this process has an interior, and the tuning
    // allows it (the kernel's support for subdomain ranges is found at the first iteration)
    bool overlap = D0->A->L.tune.overlap >= 0 && D0->nranks > 1;
    for (int i = 0; i < nr; ++i) overlap = overlap && ranks[i]->ib < ranks[i]->ie;
    int64_t iters = 0;
    double rel = 0.0;
    int converged = 0;
    bool diverged = false, bzero = false;
    std::vector<double *> res(nr);
    for (;;) {
        bool stopped = false;
        // global iteration m: x^(m-1) in (m odd ? xa : xb) (async: always xa, in place)
        while (issued < max_iters && !stopped) {
            const int64_t c = std::min(chunk, max_iters - issued);
            for (int64_t it = 0; it < c; ++it) {
                const int64_t m = issued + it + 1;
                const bool odd = (m & 1) || mode == BAR_MODE_ASYNC;
                const std::vector<double *> &vin = odd ? xa : xb;
                const std::vector<double *> &vout = mode == BAR_MODE_ASYNC ? xa : (odd ? xb : xa);
                bool done = false;
                if (overlap) {  // interior sweeps on the second stream while the exchange runs
                    if ((r = timer_begin(T, m, st)) != BAR_OK) return r;
                    bool supported = true;
                    if ((r = overlapped_iteration(ranks, nr, vin.data(), vout.data(), k, mode, st, supported)) != BAR_OK)
                        return r;
                    if ((r = timer_end(T, st)) != BAR_OK) return r;
                    done = supported;
                    if (!supported) {
                        overlap = false;
                        T.used = T.used > 0 ? T.used - 1 : 0;
                    }
                }
                if (!done) {
                    if ((r = exchange(ranks, nr, vin.data(), st)) != BAR_OK) return r;
                    for (int i = 0; i < nr; ++i) {
                        bar_dist D = ranks[i];
                        SweepArgs a{&D->A->L, D->bbuf, own(D, vin[i]), own(D, vout[i]), k, D->A->W.state,
                                    D->A->W.partials, nullptr, D->part};
                        if (i == 0 && (r = timer_begin(T, m, st)) != BAR_OK) return r;
                        BAR_CUDA(launch_sweep(a, mode, st));
                        if (i == 0 && (r = timer_end(T, st)) != BAR_OK) return r;
                    }
                }
                if ((r = reduce_decide(ranks, nr, false, st)) != BAR_OK) return r;
                launches += (done ? 5 : 2) * nr;  // overlapped: three sweeps and the partial sum
            }
            issued += c;
            if ((r = read_state(D0->A, st)) != BAR_OK) return r;
            stopped = H.stop != 0;
            if ((r = timer_collect(T, (int64_t)H.iter, 1.0)) != BAR_OK) return r;
            chunk = sizer.next(chunk, (long long)H.iter, H.last_rel, tol);
        }
        if (stopped && mode != BAR_MODE_ASYNC) {
            iters = H.conv_iter;
            rel = H.last_rel;
            if (H.diverged == 2) bzero = true;
            else if (H.diverged == 1) diverged = true;
            else converged = 1;
            for (int i = 0; i < nr; ++i) res[i] = (iters & 1) ? xb[i] : xa[i];
            break;
        }
        // async (its fused estimate mixed old and new values) or max_global_iters reached:
        // exact residual of the returned iterate, after a fresh exchange
        iters = stopped ? (int64_t)H.iter : max_iters;
        const bool est_diverged = stopped && H.diverged == 1;
        for (int i = 0; i < nr; ++i) res[i] = mode == BAR_MODE_ASYNC ? xa[i] : ((iters & 1) ? xb[i] : xa[i]);
        if ((r = exchange(ranks, nr, res.data(), st)) != BAR_OK) return r;
        for (int i = 0; i < nr; ++i) {
            bar_dist D = ranks[i];
            BAR_CUDA(launch_residual(D->A->L, D->bbuf, own(D, res[i]), D->A->W.state, D->A->W.partials, st, D->part));
        }
        if ((r = reduce_decide(ranks, nr, true, st)) != BAR_OK) return r;
        if ((r = read_state(D0->A, st)) != BAR_OK) return r;
        rel = H.exact_rel;
        if (H.bnorm == 0.0) bzero = true;
        else if (est_diverged || !std::isfinite(rel) || rel > 1e30) diverged = true;
        else converged = rel <= tol;
        if (converged || diverged || bzero || !stopped || issued >= max_iters) break;
        // the async estimate met tol but the exact residual did not: resume
        for (int i = 0; i < nr; ++i)
            BAR_CUDA(cudaMemsetAsync(&ranks[i]->A->W.state->stop, 0, sizeof(int), st));
    }
    for (int i = 0; i < nr; ++i) {
        bar_dist D = ranks[i];
        const size_t nb = sizeof(double) * (size_t)D->n_local;
        if (bzero) BAR_CUDA(cudaMemsetAsync(x[i], 0, nb, st));
        else BAR_CUDA(cudaMemcpyAsync(x[i], own(D, res[i]), nb, cudaMemcpyDefault, st));
    }
    BAR_CUDA(cudaStreamSynchronize(st));
    if (bzero) {
        iters = 0;
        rel = 0.0;
        converged = 1;
        diverged = false;
    }
    fill_info(info, ranks, nr, iters, iters, rel, converged, launches, T);
    if (diverged) {
        set_error("relative residual became non-finite or exceeded 1e30");
        return BAR_ERR_DIVERGED;
    }
    return BAR_OK;
}

// Collective exact residual ||b - A x||_2 of a row-partitioned x (every rank calls it).
bar_status dist_residual(bar_dist D, const double *b, const double *x, cudaStream_t st, double *res_norm2,
                         double *b_norm2) {
    if (D->loopback && D->nranks > 1) {
        set_error("loopback ranks: use bar_dist_solve_loopback");
        return BAR_ERR_INVALID_ARG;
    }
    bar_status r;
    DeviceGuard g(D->device);
    if ((r = ensure_workspace(D->A)) != BAR_OK) return r;
    const size_t nb = sizeof(double) * (size_t)D->n_local;
    BAR_CUDA(cudaMemcpyAsync(D->bbuf, b, nb, cudaMemcpyDefault, st));
    BAR_CUDA(cudaMemcpyAsync(own(D, D->xa), x, nb, cudaMemcpyDefault, st));
    BAR_CUDA(launch_init_state(D->A->W.state, 0.0, st));
    double ss = 0.0, bsq = 0.0;
    if (!D->has_nccl && D->nranks > 1) {  // separate processes without NCCL: peer memory
        if (!D->p2p) {
            set_error("this rank has neither an NCCL communicator nor peer-memory access");
            return BAR_ERR_INVALID_ARG;
        }
        double *xs[1] = {D->xa};
        int64_t a = 0, c = 0, e = 0;
        if ((r = p2p_exact(&D, 1, xs, st, ss, bsq, a, c, 0, e)) != BAR_OK) return r;
    } else {
        double *xs[1] = {D->xa};
        if ((r = exchange(&D, 1, xs, st)) != BAR_OK) return r;
        BAR_CUDA(launch_residual(D->A->L, D->bbuf, own(D, D->xa), D->A->W.state, D->A->W.partials, st, D->part));
        if ((r = reduce_decide(&D, 1, true, st)) != BAR_OK) return r;
        if ((r = read_state(D->A, st)) != BAR_OK) return r;
        ss = D->A->W.h_state->exact_ss;
        bsq = D->A->W.h_state->bnorm * D->A->W.h_state->bnorm;
    }
    *res_norm2 = std::sqrt(ss);
    if (b_norm2) *b_norm2 = std::sqrt(bsq);
    return BAR_OK;
}

// One rank's share from an explicit plan (bar_dist_create / bar_create_csr_dist).
bar_status create_share(int64_t n_global, int64_t row_begin, int64_t row_end, int64_t nnz_local, const int32_t *rowptr,
                        const int32_t *col_local, const double *val, int64_t n_ghost_lo, int64_t n_ghost_hi,
                        int nranks, int rank, const int64_t *recv_counts, const int64_t *send_counts,
                        const int32_t *send_idx, int32_t rows_per_block, int device, bar_dist *out) {
    *out = nullptr;
    const int64_t nl = row_end - row_begin;
    if (nranks < 1 || rank < 0 || rank >= nranks || nl < 1 || row_begin < 0 || row_end > n_global ||
        rows_per_block < 1 || rows_per_block > BAR_MAX_ROWS_PER_BLOCK || row_begin % rows_per_block != 0 ||
        n_ghost_lo < 0 || n_ghost_hi < 0 || !recv_counts || !send_counts || !rowptr || !val ||
        (nnz_local > 0 && !col_local)) {
        set_error("invalid partition (row_begin must be a multiple of rows_per_block) or argument");
        return BAR_ERR_INVALID_ARG;
    }
    int64_t nrecv = 0, nsend = 0;
    for (int p = 0; p < nranks; ++p) {
        if (recv_counts[p] < 0 || send_counts[p] < 0 || (p == rank && (recv_counts[p] || send_counts[p]))) {
            set_error("invalid send/recv counts");
            return BAR_ERR_INVALID_ARG;
        }
        nrecv += recv_counts[p];
        nsend += send_counts[p];
    }
    if (nrecv != n_ghost_lo + n_ghost_hi || (nsend > 0 && !send_idx)) {
        set_error("recv counts must add up to the ghost count");
        return BAR_ERR_INVALID_ARG;
    }
    DeviceGuard g(device);
    if (!g.ok) return cuda_fail(cudaGetLastError(), "cudaSetDevice");
    auto *D = new bar_dist_s();
    D->rank = rank;
    D->nranks = nranks;
    D->device = device;
    D->n_global = n_global;
    D->row_begin = row_begin;
    D->row_end = row_end;
    D->n_local = nl;
    D->n_glo = n_ghost_lo;
    D->n_ghi = n_ghost_hi;
    D->glo_pad = (n_ghost_lo + 1) & ~(int64_t)1;  // owned block 16-byte aligned
    D->ext = D->glo_pad + nl + n_ghost_hi + 2;
    D->send_cnt.assign(send_counts, send_counts + nranks);
    D->recv_cnt.assign(recv_counts, recv_counts + nranks);
    D->send_off.assign(nranks, 0);
    D->recv_pos.assign(nranks, 0);
    for (int p = 1; p < nranks; ++p) D->send_off[p] = D->send_off[p - 1] + D->send_cnt[p - 1];
    {
        int64_t pos = -n_ghost_lo;  // ghosts of ranks below, then (skipping the owned block) above
        for (int p = 0; p < nranks; ++p) {
            if (p == rank) pos = nl;
            D->recv_pos[p] = pos;
            pos += D->recv_cnt[p];
        }
    }
    D->n_send = nsend;
    bar_status st = BAR_OK;
    // local layout: rows [0, nl), columns [-n_glo, nl + n_ghi)
    {
        const int32_t *d_rp = rowptr, *d_col = col_local;
        const double *d_val = val;
        int32_t *t_rp = nullptr, *t_col = nullptr;
        double *t_val = nullptr;
        if (!is_device_ptr(rowptr)) st = to_device(rowptr, nl + 1, &t_rp), d_rp = t_rp;
        if (st == BAR_OK && !is_device_ptr(col_local)) st = to_device(col_local, nnz_local, &t_col), d_col = t_col;
        if (st == BAR_OK && !is_device_ptr(val)) st = to_device(val, nnz_local, &t_val), d_val = t_val;
        if (st == BAR_OK) {
            D->A = new bar_matrix_s();
            D->A->device = device;
            st = build_layout(D->A->L, nl, nnz_local, d_rp, d_col, d_val, rows_per_block, nullptr, -n_ghost_lo,
                              nl + n_ghost_hi);
            if (st != BAR_OK) {
                delete D->A;
                D->A = nullptr;
            }
        }
        cudaFree(t_rp);
        cudaFree(t_col);
        cudaFree(t_val);
    }
    if (st == BAR_OK) {  // interior subdomains: [ib, ie) with no ghost column in any row
        std::vector<int32_t> hrp = to_host(rowptr, nl + 1, st);
        std::vector<int32_t> hcol = to_host(col_local, nnz_local, st);
        const int64_t R = rows_per_block, q = (nl + R - 1) / R;
        std::vector<uint8_t> glo(q, 0), ghi(q, 0);
        for (int64_t i = 0; st == BAR_OK && i < nl; ++i)
            for (int32_t e = hrp[i]; e < hrp[i + 1]; ++e) {
                if (hcol[e] < 0) glo[i / R] = 1;
                else if (hcol[e] >= nl) ghi[i / R] = 1;
            }
        int64_t ib = 0, ie = q;
        for (int64_t l = 0; l < q; ++l)
            if (glo[l]) ib = l + 1;
        for (int64_t l = q - 1; l >= 0; --l)
            if (ghi[l]) ie = l;
        bool clean = ib < ie;
        for (int64_t l = ib; clean && l < ie; ++l) clean = !glo[l] && !ghi[l];
        D->ib = clean ? ib : 0;
        D->ie = clean ? ie : 0;
    }
    if (st == BAR_OK) {
        std::vector<int32_t> hidx = to_host(send_idx, nsend, st);
        for (int64_t i = 0; st == BAR_OK && i < nsend; ++i)
            if (hidx[i] < 0 || hidx[i] >= nl) {
                set_error("send_idx out of the owned rows");
                st = BAR_ERR_INVALID_ARG;
            }
        if (st == BAR_OK) st = to_device(hidx.data(), nsend, &D->send_idx);
    }
    auto dalloc = [&](double **p, int64_t n) {
        if (st == BAR_OK && cudaMalloc((void **)p, sizeof(double) * (size_t)(n > 0 ? n : 1)) != cudaSuccess)
            st = cuda_fail(cudaGetLastError(), "cudaMalloc");
    };
    dalloc(&D->xa, D->ext);
    dalloc(&D->xb, D->ext);
    dalloc(&D->bbuf, nl);
    dalloc(&D->send_buf, nsend);
    dalloc(&D->part, 2);
    dalloc(&D->gathered, 2 * (int64_t)nranks);
    dalloc(&D->board, kBoardWordsPerRank * (int64_t)nranks);
    if (st == BAR_OK && cudaMemset(D->board, 0, sizeof(double) * kBoardWordsPerRank * (size_t)nranks) != cudaSuccess)
        st = cuda_fail(cudaGetLastError(), "cudaMemset");
    if (st == BAR_OK &&
        cudaMallocHost((void **)&D->h_exact, sizeof(double) * 4 * (size_t)nranks) != cudaSuccess)
        st = cuda_fail(cudaGetLastError(), "cudaMallocHost");
    if (st != BAR_OK) {
        bar_dist_destroy(D);
        return st;
    }
    D->peers.assign(1, D);
    *out = D;
    return BAR_OK;
}

// Map every rank's iterate and board (IPC handles, or the linked loopback peers) and switch the
// async mode to the peer-memory path.
bar_status enable_p2p(bar_dist D, const int32_t *ghost_src_idx, const void *handles, const int64_t *own_offsets) {
    const int64_t ng = D->n_glo + D->n_ghi;
    DeviceGuard g(D->device);
    std::vector<int32_t> grank(ng), gidx(ng);
    {
        int64_t j = 0;
        for (int p = 0; p < D->nranks; ++p)
            for (int64_t c = 0; c < D->recv_cnt[p]; ++c, ++j) grank[j] = p;
    }
    for (int64_t j = 0; j < ng; ++j) {
        gidx[j] = ghost_src_idx[j];
        if (gidx[j] < 0) {
            set_error("ghost source index < 0");
            return BAR_ERR_INVALID_ARG;
        }
    }
    std::vector<double *> pown(D->nranks), pboard(D->nranks);
    for (int p = 0; p < D->nranks; ++p) {
        if (handles == nullptr) {  // loopback: the peers live in this process
            bar_dist P = D->peers[p];
            pown[p] = own(P, P->xa);
            pboard[p] = P->board;
        } else if (p == D->rank) {
            pown[p] = own(D, D->xa);
            pboard[p] = D->board;
        } else {
            cudaIpcMemHandle_t hx, hb;
            std::memcpy(&hx, (const char *)handles + 128 * (size_t)p, 64);
            std::memcpy(&hb, (const char *)handles + 128 * (size_t)p + 64, 64);
            void *px = nullptr, *pb = nullptr;
            BAR_CUDA(cudaIpcOpenMemHandle(&px, hx, cudaIpcMemLazyEnablePeerAccess));
            D->opened.push_back(px);
            BAR_CUDA(cudaIpcOpenMemHandle(&pb, hb, cudaIpcMemLazyEnablePeerAccess));
            D->opened.push_back(pb);
            pown[p] = (double *)px + own_offsets[p];
            pboard[p] = (double *)pb;
        }
    }
    cudaFree(D->g_rank);
    cudaFree(D->g_idx);
    cudaFree(D->d_peer_own);
    cudaFree(D->d_peer_board);
    D->g_rank = D->g_idx = nullptr;
    D->d_peer_own = D->d_peer_board = nullptr;
    bar_status r;
    if ((r = to_device(grank.data(), ng, &D->g_rank)) != BAR_OK) return r;
    if ((r = to_device(gidx.data(), ng, &D->g_idx)) != BAR_OK) return r;
    if ((r = to_device(pown.data(), D->nranks, &D->d_peer_own)) != BAR_OK) return r;
    if ((r = to_device(pboard.data(), D->nranks, &D->d_peer_board)) != BAR_OK) return r;
    D->p2p = true;
    return BAR_OK;
}

}  // namespace

// bar_solve / bar_residual / bar_sweep / bar_destroy on a handle from bar_create_csr_dist (api.cu)
bar_status dist_solve_handle(bar_matrix A, const double *b, const double *x0, double *x, int32_t k,
                             int64_t max_global_iters, double tol, bar_mode mode, cudaStream_t st,
                             bar_solve_info *info) {
    bar_dist D = A->dist;
    const double *bb[1] = {b};
    const double *xx0[1] = {x0};
    double *xx[1] = {x};
    return dist_solve(&D, 1, bb, xx0, xx, k, max_global_iters, tol, mode, st, info);
}

bar_status dist_residual_handle(bar_matrix A, const double *b, const double *x, cudaStream_t st, double *res_norm2,
                                double *b_norm2) {
    return dist_residual(A->dist, b, x, st, res_norm2, b_norm2);
}

void dist_destroy_handle(bar_matrix A) { bar_dist_destroy(A->dist); }

// bar_sweep on a rank's share: b, x are the rank's rows (device); nsweeps local launches on x
// with the ghost slots as the last exchange left them (kernel timing, no exchange, no sync).
bar_status dist_sweep_handle(bar_matrix A, const double *b, double *x, int32_t k, int64_t nsweeps, bar_mode mode,
                             cudaStream_t st) {
    bar_dist D = A->dist;
    const size_t nb = sizeof(double) * (size_t)D->n_local;
    BAR_CUDA(cudaMemcpyAsync(D->bbuf, b, nb, cudaMemcpyDeviceToDevice, st));
    BAR_CUDA(cudaMemcpyAsync(own(D, D->xa), x, nb, cudaMemcpyDeviceToDevice, st));
    bar_status r = bar_dist_sweep(D, k, nsweeps, mode, st);
    if (r != BAR_OK) return r;
    const bool in_b = mode != BAR_MODE_ASYNC && (nsweeps & 1);
    BAR_CUDA(cudaMemcpyAsync(x, own(D, in_b ? D->xb : D->xa), nb, cudaMemcpyDeviceToDevice, st));
    return BAR_OK;
}

}  // namespace bar

using namespace bar;

extern "C" {

bar_status bar_dist_ghosts(int64_t row_begin, int64_t row_end, int64_t nnz_local, const int32_t *rowptr,
                           const int32_t *col, int64_t *n_ghost_lo, int64_t *n_ghost_hi, int32_t *ghosts) {
    if (!rowptr || (!col && nnz_local > 0) || !n_ghost_lo || !n_ghost_hi || row_end < row_begin || row_begin < 0) {
        set_error("invalid argument");
        return BAR_ERR_INVALID_ARG;
    }
    const int64_t nl = row_end - row_begin;
    if (rowptr[0] != 0 || rowptr[nl] != nnz_local) {
        set_error("rowptr[0] != 0 or rowptr[n_local] != nnz_local");
        return BAR_ERR_BAD_CSR;
    }
    std::vector<int32_t> lo, hi;
    ghost_lists(row_begin, row_end, nnz_local, col, lo, hi);
    *n_ghost_lo = (int64_t)lo.size();
    *n_ghost_hi = (int64_t)hi.size();
    if (ghosts) {
        std::copy(lo.begin(), lo.end(), ghosts);
        std::copy(hi.begin(), hi.end(), ghosts + lo.size());
    }
    return BAR_OK;
}

bar_status bar_dist_localize(int64_t row_begin, int64_t row_end, int64_t nnz_local, const int32_t *rowptr,
                             const int32_t *col, int64_t n_ghost_lo, int64_t n_ghost_hi, const int32_t *ghosts,
                             int32_t *col_local) {
    if (!rowptr || !col_local || (nnz_local > 0 && !col) || ((n_ghost_lo + n_ghost_hi) > 0 && !ghosts)) {
        set_error("invalid argument");
        return BAR_ERR_INVALID_ARG;
    }
    std::vector<int32_t> lo(ghosts, ghosts + n_ghost_lo), hi(ghosts + n_ghost_lo, ghosts + n_ghost_lo + n_ghost_hi);
    return localize(row_begin, row_end, nnz_local, col, lo, hi, col_local);
}

bar_status bar_dist_plan(int nranks, int rank, const int64_t *row_ranges, const int64_t *ghost_counts,
                         const int32_t *ghosts_all, int64_t *recv_counts, int64_t *send_counts, int32_t *send_idx,
                         int32_t *ghost_src_idx) {
    if (nranks < 1 || rank < 0 || rank >= nranks || !row_ranges || !ghost_counts || !recv_counts || !send_counts) {
        set_error("invalid argument");
        return BAR_ERR_INVALID_ARG;
    }
    int64_t tot = 0;
    for (int p = 0; p < nranks; ++p) {
        if (ghost_counts[p] < 0 || row_ranges[2 * p] > row_ranges[2 * p + 1] ||
            (p > 0 && row_ranges[2 * p] != row_ranges[2 * p - 1])) {
            set_error("row ranges must be contiguous and ascending; ghost counts >= 0");
            return BAR_ERR_INVALID_ARG;
        }
        tot += ghost_counts[p];
    }
    if (tot > 0 && !ghosts_all) {
        set_error("ghosts_all is NULL");
        return BAR_ERR_INVALID_ARG;
    }
    std::vector<int64_t> rc, sc;
    std::vector<int32_t> si, gs;
    bar_status r = plan(nranks, rank, row_ranges, ghost_counts, ghosts_all, rc, sc, si, gs);
    if (r != BAR_OK) return r;
    std::copy(rc.begin(), rc.end(), recv_counts);
    std::copy(sc.begin(), sc.end(), send_counts);
    if (send_idx) std::copy(si.begin(), si.end(), send_idx);
    if (ghost_src_idx) std::copy(gs.begin(), gs.end(), ghost_src_idx);
    return BAR_OK;
}

bar_status bar_nccl_unique_id(void *id128) {
    if (!id128) {
        set_error("NULL argument");
        return BAR_ERR_INVALID_ARG;
    }
#ifdef BAR_WITH_NCCL
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
    ncclUniqueId id;
    ncclResult_t rc = ncclGetUniqueId(&id);
    if (rc != ncclSuccess) return nccl_fail((int)rc, "ncclGetUniqueId");
    std::memcpy(id128, &id, sizeof(id));
    return BAR_OK;
#else
    return nccl_fail(0, "ncclGetUniqueId");
#endif
}

bar_status bar_dist_create(int64_t n_global, int64_t row_begin, int64_t row_end, int64_t nnz_local,
                           const int32_t *rowptr, const int32_t *col_local, const double *val, int64_t n_ghost_lo,
                           int64_t n_ghost_hi, int nranks, int rank, const int64_t *recv_counts,
                           const int64_t *send_counts, const int32_t *send_idx, int32_t rows_per_block, int device,
                           const void *nccl_id, bar_dist *out) {
    if (!out) {
        set_error("out is NULL");
        return BAR_ERR_INVALID_ARG;
    }
    bar_status st = create_share(n_global, row_begin, row_end, nnz_local, rowptr, col_local, val, n_ghost_lo,
                                 n_ghost_hi, nranks, rank, recv_counts, send_counts, send_idx, rows_per_block, device,
                                 out);
    if (st != BAR_OK || !nccl_id) return st;
#ifdef BAR_WITH_NCCL
    bar_dist D = *out;
    DeviceGuard g(device);
    ncclUniqueId id;
    std::memcpy(&id, nccl_id, sizeof(id));
    ncclResult_t rc = ncclCommInitRank(&D->comm, nranks, id, rank);
    if (rc != ncclSuccess) st = nccl_fail((int)rc, "ncclCommInitRank");
    D->has_nccl = st == BAR_OK;
#else
    st = nccl_fail(0, "ncclCommInitRank");
#endif
    if (st != BAR_OK) {
        bar_dist_destroy(*out);
        *out = nullptr;
    }
    return st;
}

bar_status bar_create_csr_dist(int64_t n_global, int64_t row_begin, int64_t row_end, int64_t nnz_local,
                               const int32_t *rowptr, const int32_t *col, const double *val, int32_t rows_per_block,
                               int device, const void *nccl_unique_id, int rank, int nranks, bar_matrix *out) {
    if (!out) {
        set_error("out is NULL");
        return BAR_ERR_INVALID_ARG;
    }
    *out = nullptr;
    const int64_t nl = row_end - row_begin;
    if (!nccl_unique_id || nranks < 1 || rank < 0 || rank >= nranks || nl < 1 || row_begin < 0 ||
        row_end > n_global || !rowptr || !val || (nnz_local > 0 && !col) || rows_per_block < 1 ||
        rows_per_block > BAR_MAX_ROWS_PER_BLOCK || row_begin % rows_per_block != 0 || nnz_local >= INT32_MAX) {
        set_error("invalid argument (nccl_unique_id required; row_begin a multiple of rows_per_block)");
        return BAR_ERR_INVALID_ARG;
    }
#ifndef BAR_WITH_NCCL
    (void)device;
    return nccl_fail(0, "bar_create_csr_dist");
#else
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) {
        cudaGetLastError();
        set_error("invalid CUDA device");
        return BAR_ERR_INVALID_ARG;
    }
    DeviceGuard g(device);
    bar_status st = BAR_OK;
    // host copies of the row block's structure (the arrays may be device memory)
    std::vector<int32_t> h_rp = to_host(rowptr, nl + 1, st);
    std::vector<int32_t> h_col = to_host(col, nnz_local, st);
    if (st != BAR_OK) return st;
    if (h_rp[0] != 0 || h_rp[nl] != nnz_local) {
        set_error("rowptr[0] != 0 or rowptr[n_local] != nnz_local");
        return BAR_ERR_BAD_CSR;
    }
    for (int64_t e = 0; e < nnz_local; ++e)
        if (h_col[e] < 0 || h_col[e] >= n_global) {
            set_error("column out of [0, n_global)");
            return BAR_ERR_BAD_CSR;
        }
    std::vector<int32_t> lo, hi;
    ghost_lists(row_begin, row_end, nnz_local, h_col.data(), lo, hi);
    // the communicator, then every rank's (row range, ghost count, device) and ghost list
    NvtxRange nv("bar_create_csr_dist: NCCL planning, layout, IPC mapping");
    ncclComm_t comm = nullptr;
    {
        ncclUniqueId id;
        std::memcpy(&id, nccl_unique_id, sizeof(id));
        BAR_NCCL(ncclCommInitRank(&comm, nranks, id, rank));
    }
    struct CommGuard {
        ncclComm_t c;
        ~CommGuard() {
            if (c) ncclCommDestroy(c);
        }
    } cg{comm};
    cudaStream_t s = nullptr;
    const int P = nranks;
    int64_t *dbuf = nullptr;
    std::vector<int64_t> meta((size_t)4 * P);
    {
        int64_t mine[4] = {row_begin, row_end, (int64_t)(lo.size() + hi.size()), (int64_t)device};
        BAR_CUDA(cudaMalloc(&dbuf, sizeof(int64_t) * 4 * (P + 1)));
        BAR_CUDA(cudaMemcpy(dbuf, mine, sizeof(mine), cudaMemcpyHostToDevice));
        BAR_NCCL(ncclAllGather(dbuf, dbuf + 4, 4, ncclInt64, comm, s));
        BAR_CUDA(cudaMemcpy(meta.data(), dbuf + 4, sizeof(int64_t) * 4 * P, cudaMemcpyDeviceToHost));
        cudaFree(dbuf);
    }
    std::vector<int64_t> ranges(2 * P), gcount(P);
    int64_t gmax = 1, gtot = 0;
    for (int p = 0; p < P; ++p) {
        ranges[2 * p] = meta[4 * p];
        ranges[2 * p + 1] = meta[4 * p + 1];
        gcount[p] = meta[4 * p + 2];
        gmax = std::max(gmax, gcount[p]);
        gtot += gcount[p];
    }
    std::vector<int32_t> gall((size_t)gtot);
    {
        std::vector<int32_t> mine((size_t)gmax, 0);
        std::copy(lo.begin(), lo.end(), mine.begin());
        std::copy(hi.begin(), hi.end(), mine.begin() + lo.size());
        int32_t *dg = nullptr;
        BAR_CUDA(cudaMalloc(&dg, sizeof(int32_t) * (size_t)gmax * (P + 1)));
        BAR_CUDA(cudaMemcpy(dg, mine.data(), sizeof(int32_t) * (size_t)gmax, cudaMemcpyHostToDevice));
        BAR_NCCL(ncclAllGather(dg, dg + gmax, (size_t)gmax, ncclInt32, comm, s));
        std::vector<int32_t> all((size_t)gmax * P);
        BAR_CUDA(cudaMemcpy(all.data(), dg + gmax, sizeof(int32_t) * (size_t)gmax * P, cudaMemcpyDeviceToHost));
        cudaFree(dg);
        int64_t o = 0;
        for (int p = 0; p < P; ++p)
            for (int64_t j = 0; j < gcount[p]; ++j) gall[(size_t)o++] = all[(size_t)p * gmax + j];
    }
    std::vector<int64_t> rc, sc;
    std::vector<int32_t> si, gsrc;
    if ((st = plan(P, rank, ranges.data(), gcount.data(), gall.data(), rc, sc, si, gsrc)) != BAR_OK) return st;
    std::vector<int32_t> col_local((size_t)nnz_local);
    if ((st = localize(row_begin, row_end, nnz_local, h_col.data(), lo, hi, col_local.data())) != BAR_OK) return st;
    bar_dist D = nullptr;
    st = create_share(n_global, row_begin, row_end, nnz_local, h_rp.data(), col_local.data(), val, (int64_t)lo.size(),
                      (int64_t)hi.size(), P, rank, rc.data(), sc.data(), si.data(), rows_per_block, device, &D);
    if (st != BAR_OK) return st;
    D->comm = comm;
    D->has_nccl = true;
    cg.c = nullptr;  // owned by D now
    // peer memory for the async mode: every rank must reach every other rank's memory (same
    // process group on one node: NVLink / NVSwitch peer access); agreed with a min all-reduce
    {
        int ok = 1;
        for (int p = 0; p < P && ok; ++p) {
            const int dev = (int)meta[4 * p + 3];
            if (p == rank || dev == device) continue;
            int can = 0;
            if (dev < 0 || dev >= ndev || cudaDeviceCanAccessPeer(&can, device, dev) != cudaSuccess || !can) ok = 0;
            cudaGetLastError();
        }
        int *dok = nullptr;
        st = BAR_OK;
        if (cudaMalloc(&dok, sizeof(int)) != cudaSuccess) st = cuda_fail(cudaGetLastError(), "cudaMalloc");
        if (st == BAR_OK) {
            cudaMemcpy(dok, &ok, sizeof(int), cudaMemcpyHostToDevice);
            ncclResult_t rr = ncclAllReduce(dok, dok, 1, ncclInt32, ncclMin, comm, s);
            if (rr != ncclSuccess) st = nccl_fail((int)rr, "ncclAllReduce");
            else if (cudaMemcpy(&ok, dok, sizeof(int), cudaMemcpyDeviceToHost) != cudaSuccess)
                st = cuda_fail(cudaGetLastError(), "cudaMemcpy");
        }
        cudaFree(dok);
        if (st == BAR_OK && ok) {
            // IPC handles of every rank's iterate and board, and owned-block offsets
            std::vector<unsigned char> mine(136, 0);
            int64_t off = 0;
            // (an export failure only disables peer memory: every rank still joins the gather)
            const bool exported = bar_dist_p2p_handles(D, mine.data(), &off) == BAR_OK;
            cudaGetLastError();
            std::memcpy(mine.data() + 128, &off, 8);
            unsigned char *dh = nullptr;
            if (st == BAR_OK && cudaMalloc(&dh, 136 * (size_t)(P + 1)) != cudaSuccess)
                st = cuda_fail(cudaGetLastError(), "cudaMalloc");
            std::vector<unsigned char> all(136 * (size_t)P);
            if (st == BAR_OK) {
                cudaMemcpy(dh, mine.data(), 136, cudaMemcpyHostToDevice);
                ncclResult_t rr = ncclAllGather(dh, dh + 136, 136, ncclUint8, comm, s);
                if (rr != ncclSuccess) st = nccl_fail((int)rr, "ncclAllGather");
                else if (cudaMemcpy(all.data(), dh + 136, all.size(), cudaMemcpyDeviceToHost) != cudaSuccess)
                    st = cuda_fail(cudaGetLastError(), "cudaMemcpy");
            }
            cudaFree(dh);
            if (st == BAR_OK) {
                std::vector<unsigned char> handles(128 * (size_t)P);
                std::vector<int64_t> offs(P);
                for (int p = 0; p < P; ++p) {
                    std::memcpy(handles.data() + 128 * (size_t)p, all.data() + 136 * (size_t)p, 128);
                    std::memcpy(&offs[p], all.data() + 136 * (size_t)p + 128, 8);
                }
                // a rank that cannot map its peers (IPC refused) is not an error of the solve: all
                // ranks agree (min all-reduce) and, if any failed, unmap and keep the collective
                // NCCL path for async as well
                int mapped = exported && enable_p2p(D, gsrc.data(), handles.data(), offs.data()) == BAR_OK ? 1 : 0;
                cudaGetLastError();
                int *dm = nullptr;
                if (cudaMalloc(&dm, sizeof(int)) != cudaSuccess) st = cuda_fail(cudaGetLastError(), "cudaMalloc");
                if (st == BAR_OK) {
                    cudaMemcpy(dm, &mapped, sizeof(int), cudaMemcpyHostToDevice);
                    ncclResult_t rr = ncclAllReduce(dm, dm, 1, ncclInt32, ncclMin, comm, s);
                    if (rr != ncclSuccess) st = nccl_fail((int)rr, "ncclAllReduce");
                    else if (cudaMemcpy(&mapped, dm, sizeof(int), cudaMemcpyDeviceToHost) != cudaSuccess)
                        st = cuda_fail(cudaGetLastError(), "cudaMemcpy");
                }
                cudaFree(dm);
                if (st == BAR_OK && !mapped) {
                    for (void *q : D->opened) cudaIpcCloseMemHandle(q);
                    D->opened.clear();
                    D->p2p = false;
                    cudaGetLastError();
                }
            }
        }
    }
    if (st != BAR_OK) {
        bar_dist_destroy(D);
        return st;
    }
    D->owner_handle = true;
    D->A->dist = D;
    *out = D->A;
    return BAR_OK;
#endif
}

bar_status bar_dist_link_loopback(bar_dist *ranks, int nranks) {
    if (!ranks || nranks < 1) {
        set_error("invalid argument");
        return BAR_ERR_INVALID_ARG;
    }
    for (int i = 0; i < nranks; ++i) {
        if (!ranks[i] || ranks[i]->has_nccl || ranks[i]->rank != i || ranks[i]->nranks != nranks ||
            ranks[i]->device != ranks[0]->device) {
            set_error("loopback ranks must be 0..nranks-1 of one group on one device, created with nccl_id = NULL");
            return BAR_ERR_INVALID_ARG;
        }
    }
    for (int i = 0; i < nranks; ++i) {
        ranks[i]->peers.assign(ranks, ranks + nranks);
        ranks[i]->loopback = true;
    }
    return BAR_OK;
}

bar_status bar_dist_solve(bar_dist D, const double *b, const double *x0, double *x, int32_t k,
                          int64_t max_global_iters, double tol, bar_mode mode, void *cuda_stream,
                          bar_solve_info *info) {
    if (!D || !b || !x) {
        set_error("NULL argument");
        return BAR_ERR_INVALID_ARG;
    }
    if (D->loopback && D->nranks > 1) {
        set_error("loopback ranks are driven together by bar_dist_solve_loopback");
        return BAR_ERR_INVALID_ARG;
    }
    const double *bb[1] = {b};
    const double *xx0[1] = {x0};
    double *xx[1] = {x};
    return dist_solve(&D, 1, bb, xx0, xx, k, max_global_iters, tol, mode, (cudaStream_t)cuda_stream, info);
}

bar_status bar_dist_solve_loopback(bar_dist *ranks, int nranks, const double *const *b, const double *const *x0,
                                   double *const *x, int32_t k, int64_t max_global_iters, double tol,
                                   bar_mode mode, void *cuda_stream, bar_solve_info *info) {
    if (!ranks || nranks < 1 || !b || !x) {
        set_error("NULL argument");
        return BAR_ERR_INVALID_ARG;
    }
    for (int i = 0; i < nranks; ++i)
        if (!ranks[i] || (nranks > 1 && !ranks[i]->loopback) || (int)ranks[i]->peers.size() != nranks ||
            ranks[i]->peers[0] != ranks[0]) {
            set_error("ranks are not a linked loopback group");
            return BAR_ERR_INVALID_ARG;
        }
    return dist_solve(ranks, nranks, b, x0, x, k, max_global_iters, tol, mode, (cudaStream_t)cuda_stream, info);
}

bar_status bar_dist_p2p_handles(bar_dist D, void *handles128, int64_t *own_offset) {
    if (!D || !handles128 || !own_offset) {
        set_error("NULL argument");
        return BAR_ERR_INVALID_ARG;
    }
    DeviceGuard g(D->device);
    cudaIpcMemHandle_t hx, hb;
    BAR_CUDA(cudaIpcGetMemHandle(&hx, D->xa));
    BAR_CUDA(cudaIpcGetMemHandle(&hb, D->board));
    static_assert(sizeof(cudaIpcMemHandle_t) == 64, "IPC handle size");
    std::memcpy(handles128, &hx, 64);
    std::memcpy((char *)handles128 + 64, &hb, 64);
    *own_offset = D->glo_pad;
    return BAR_OK;
}

bar_status bar_dist_enable_p2p(bar_dist D, const int32_t *ghost_src_idx, const void *handles,
                               const int64_t *own_offsets) {
    const int64_t ng = D ? D->n_glo + D->n_ghi : 0;
    if (!D || (ng > 0 && !ghost_src_idx) || ((handles == nullptr) != (own_offsets == nullptr)) ||
        (handles == nullptr && D->nranks > 1 && !D->loopback) ||
        (D->loopback && (int)D->peers.size() != D->nranks)) {
        set_error("invalid argument (loopback ranks must be linked first; separate processes need handles)");
        return BAR_ERR_INVALID_ARG;
    }
    return enable_p2p(D, ghost_src_idx, handles, own_offsets);
}

bar_status bar_dist_sweep(bar_dist D, int32_t k, int64_t nsweeps, bar_mode mode, void *cuda_stream) {
    if (!D || nsweeps < 0 || (mode != BAR_MODE_JACOBI && k < 1)) {
        set_error("invalid argument");
        return BAR_ERR_INVALID_ARG;
    }
    DeviceGuard g(D->device);
    bar_status r = ensure_workspace(D->A);
    if (r != BAR_OK) return r;
    cudaStream_t st = (cudaStream_t)cuda_stream;
    BAR_CUDA(launch_init_state(D->A->W.state, -1.0, st));
    for (int64_t m = 1; m <= nsweeps; ++m) {
        double *xi = (mode == BAR_MODE_ASYNC || (m & 1)) ? D->xa : D->xb;
        double *xo = mode == BAR_MODE_ASYNC ? D->xa : ((m & 1) ? D->xb : D->xa);
        SweepArgs a{&D->A->L, D->bbuf, own(D, xi), own(D, xo), mode == BAR_MODE_JACOBI ? 1 : k, D->A->W.state,
                    D->A->W.partials, nullptr, D->part};
        BAR_CUDA(launch_sweep(a, mode, st));
    }
    return BAR_OK;
}

bar_status bar_dist_set_tuning(bar_dist D, const bar_tuning *tuning) {
    if (!D) {
        set_error("NULL handle");
        return BAR_ERR_INVALID_ARG;
    }
    return bar_set_tuning(D->A, tuning);
}

void bar_dist_destroy(bar_dist D) {
    if (!D) return;
    DeviceGuard g(D->device);
#ifdef BAR_WITH_NCCL
    if (D->comm) ncclCommDestroy(D->comm);
#endif
    for (void *p : D->opened) cudaIpcCloseMemHandle(p);
    cudaFree(D->g_rank);
    cudaFree(D->g_idx);
    cudaFree(D->d_peer_own);
    cudaFree(D->d_peer_board);
    cudaFree(D->board);
    cudaFreeHost(D->h_exact);
    if (D->s2) cudaStreamDestroy(D->s2);
    if (D->ev_fork) cudaEventDestroy(D->ev_fork);
    if (D->ev_join) cudaEventDestroy(D->ev_join);
    cudaFree(D->state2);
    cudaFree(D->partials2);
    cudaFree(D->parts3);
    if (D->A) {
        D->A->dist = nullptr;
        bar_destroy(D->A);
    }
    cudaFree(D->xa);
    cudaFree(D->xb);
    cudaFree(D->bbuf);
    cudaFree(D->send_idx);
    cudaFree(D->send_buf);
    cudaFree(D->ag_buf);
    cudaFree(D->part);
    cudaFree(D->gathered);
    delete D;
}

}  // extern "C"
