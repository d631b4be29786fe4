// dist.cu — multi-GPU row-partitioned solve (include/bar.h "multi-GPU").
//
// Paper: §3.4 splits the system into row blocks per device, then per thread block,
// with an asynchronous iteration between devices; its data paths (AMC through host memory,
// DC/DK through a master GPU) were PCIe workarounds. Here every rank keeps its own rows and
// refreshes the x values it reads but does not own (ghosts) once per global iteration with an
// NCCL grouped send/recv over NVLink; the per-rank residual sums are all-gathered and summed
// in rank order, so every rank applies the same stopping rule to the same bits.
//
// Local vector ("extended x"): [pad | ghosts below | owned rows | ghosts above]; the owned
// block starts 16-byte aligned and every kernel indexes it with columns relative to the owned
// block (ghosts below negative), which keeps each row's entries in their global order: the
// per-row arithmetic, and so every sync-block / Jacobi iterate, is bitwise the one-GPU result.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>
#include <vector>

#include "bar_internal.cuh"

#ifdef BAR_WITH_NCCL
#include <nccl.h>
#endif

struct bar_dist_s {
    bar_matrix A = nullptr;  // local layout: n_local rows, columns [-n_glo, n_local + n_ghi)
    int rank = 0, nranks = 1, device = 0;
    int64_t n_global = 0, row_begin = 0, row_end = 0, n_local = 0, n_glo = 0, n_ghi = 0;
    int64_t glo_pad = 0, ext = 0;  // owned block offset in the extended vector; its length
    double *xa = nullptr, *xb = nullptr;  // extended iterate buffers
    double *bbuf = nullptr;               // owned b (device)
    double *xio = nullptr;                // owned x0 / x staging for host pointers
    int32_t *send_idx = nullptr;          // device, local row indices
    double *send_buf = nullptr;           // device
    int64_t n_send = 0;
    std::vector<int64_t> send_cnt, send_off, recv_cnt, recv_pos;  // recv_pos: owned-relative index
    double *part = nullptr;      // device [2]: this rank's [sum r^2, sum b^2]
    // halo exchange by ncclAllGather (SURVEY §8(e)'s primary design; BAR_HALO=allgather): every
    // rank contributes its whole send buffer padded to ag_max doubles, and each receiver copies
    // its segment of every sender p out of slot p of the gathered buffer (peer_off[p] = where p's
    // segment for this rank starts in p's send buffer). Planned on the first exchange.
    bool halo_allgather = false, ag_ready = false;
    int64_t ag_max = 0;
    double *ag_buf = nullptr;            // device [nranks * ag_max]
    std::vector<int64_t> peer_off;
    double *gathered = nullptr;  // device [2 * nranks]
    // async over peer memory (bar_dist_enable_p2p)
    bool p2p = false;
    int32_t *g_rank = nullptr, *g_idx = nullptr;     // device, per ghost: owner rank, owner-local row
    double **d_peer_own = nullptr;                  // device [nranks]: owned block of each rank's x
    double **d_peer_board = nullptr;                // device [nranks]: each rank's board
    double *board = nullptr;                        // device [2 * nranks]: latest partials of every rank
    int *d_flag = nullptr;                          // device: stop-request all-reduce
    std::vector<void *> opened;                     // IPC mappings to close
    bool loopback = true;
    std::vector<bar_dist> peers;  // loopback group (peers[r] is rank r)
#ifdef BAR_WITH_NCCL
    ncclComm_t comm = nullptr;
#endif
};

namespace bar {
namespace {

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
#define BAR_NCCL(call)                                                \
    do {                                                              \
        ncclResult_t _r = (call);                                     \
        if (_r != ncclSuccess) return ::bar::nccl_fail((int)_r, #call); \
    } while (0)
#endif

template <class T>
bar_status to_device(const T *src, int64_t count, T **dst) {
    BAR_CUDA(cudaMalloc((void **)dst, sizeof(T) * (size_t)(count > 0 ? count : 1)));
    if (count > 0) BAR_CUDA(cudaMemcpy(*dst, src, sizeof(T) * (size_t)count, cudaMemcpyDefault));
    return BAR_OK;
}

double *own(const bar_dist D, double *ext) { return ext + D->glo_pad; }

// All-gather halo plan: the largest send buffer of the group and, for this rank, the offset of
// its segment in every sender's buffer (NCCL: one all-gather of the send counts at first use;
// loopback: read from the linked peers).
bar_status plan_allgather(bar_dist *ranks, int nr, cudaStream_t st) {
    for (int i = 0; i < nr; ++i) {
        bar_dist D = ranks[i];
        if (D->ag_ready) continue;
        const int P = D->nranks;
        std::vector<int64_t> cnt((size_t)P * P, 0);  // cnt[p * P + d]: what p sends to d
        if (D->loopback) {
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
        BAR_CUDA(cudaMalloc(&D->ag_buf, sizeof(double) * (size_t)P * D->ag_max));
        D->ag_ready = true;
    }
    return BAR_OK;
}

// Refresh the ghost slots of the extended vector `ext` of every rank in `ranks` (NCCL: the
// calling rank only; loopback: all ranks of the process, in order, on one stream).
bar_status exchange(bar_dist *ranks, int nr, double *const *ext, cudaStream_t st) {
    for (int i = 0; i < nr; ++i) {
        bar_dist D = ranks[i];
        BAR_CUDA(launch_pack(own(D, ext[i]), D->send_idx, D->n_send, D->send_buf, st));
    }
    if (ranks[0]->halo_allgather) {
        bar_status r = plan_allgather(ranks, nr, st);
        if (r != BAR_OK) return r;
        const int P = ranks[0]->nranks;
        const int64_t M = ranks[0]->ag_max;
        if (!ranks[0]->loopback) {
#ifdef BAR_WITH_NCCL
            bar_dist D = ranks[0];
            BAR_NCCL(ncclAllGather(D->send_buf, D->ag_buf, (size_t)M, ncclDouble, D->comm, st));
#else
            return nccl_fail(0, "exchange");
#endif
        } else {  // loopback: the same gathered buffer, assembled by copies into every rank's ag_buf
            for (int i = 0; i < nr; ++i)
                for (int p = 0; p < P; ++p)
                    if (ranks[p]->n_send)
                        BAR_CUDA(cudaMemcpyAsync(ranks[i]->ag_buf + (size_t)p * M, ranks[p]->send_buf,
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
    if (!ranks[0]->loopback) {
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
    if (!ranks[0]->loopback) {
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

// ---- async over peer memory ----------------------------------------------------------------
// Pull every ghost value from its owner's live iterate: x "as it stands" (eq. 3), read over
// NVLink with relaxed system-scope loads, no synchronisation with the owner.
__global__ void k_pull_ghosts(double *__restrict__ x_own, int64_t n_glo, int64_t n_local, int64_t n_ghost,
                              const int32_t *__restrict__ g_rank, const int32_t *__restrict__ g_idx,
                              double *const *__restrict__ peer_own) {
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n_ghost;
         j += (int64_t)gridDim.x * blockDim.x) {
        const double *src = peer_own[g_rank[j]] + g_idx[j];
        double v;
        asm volatile("ld.relaxed.sys.global.f64 %0, [%1];" : "=d"(v) : "l"(src));
        double *dst = j < n_glo ? x_own - n_glo + j : x_own + n_local + (j - n_glo);
        asm volatile("st.relaxed.gpu.global.f64 [%0], %1;" ::"l"(dst), "d"(v) : "memory");
    }
}

// Push this rank's latest [sum r^2, sum b^2] into slot `rank` of every rank's board.
__global__ void k_publish(const double *__restrict__ part, double *const *__restrict__ peer_board, int rank,
                          int nranks) {
    const int p = threadIdx.x;
    if (p >= nranks) return;
    double *dst = peer_board[p] + 2 * rank;
    asm volatile("st.relaxed.sys.global.f64 [%0], %1;" ::"l"(dst), "d"(part[0]) : "memory");
    asm volatile("st.relaxed.sys.global.f64 [%0], %1;" ::"l"(dst + 1), "d"(part[1]) : "memory");
}

bar_status p2p_iteration(bar_dist D, const SweepArgs &a, bar_mode mode, cudaStream_t st, KernelTimer *T, int64_t m) {
    const int64_t ng = D->n_glo + D->n_ghi;
    if (ng > 0) {
        int64_t blocks = (ng + 255) / 256;
        if (blocks > 1024) blocks = 1024;
        k_pull_ghosts<<<(unsigned)blocks, 256, 0, st>>>(own(D, D->xa), D->n_glo, D->n_local, ng, D->g_rank, D->g_idx,
                                                         D->d_peer_own);
        BAR_CUDA(cudaGetLastError());
    }
    bar_status r;
    if (T && (r = timer_begin(*T, m, st)) != BAR_OK) return r;
    BAR_CUDA(launch_sweep(a, mode, st));
    if (T && (r = timer_end(*T, st)) != BAR_OK) return r;
    k_publish<<<1, 32 * ((D->nranks + 31) / 32), 0, st>>>(D->part, D->d_peer_board, D->rank, D->nranks);
    BAR_CUDA(cudaGetLastError());
    // the board holds every rank's latest partial (others' possibly a few launches old)
    BAR_CUDA(launch_dist_decide(D->A->W.state, D->board, D->nranks, false, st));
    return BAR_OK;
}

// Chunk-boundary agreement on the stop requests of all ranks (the only synchronisation of the
// asynchronous multi-GPU mode besides the exact confirming residual), and on the size of the next
// chunk: every rank sizes it from its own estimate (ChunkSizer) and all take the largest, so every
// rank reaches this all-reduce equally often.
bar_status agree_stop(bar_dist *ranks, int nr, cudaStream_t st, bool &any, ChunkSizer *sizers, int64_t chunk,
                      double tol, int64_t &next) {
    any = false;
    next = 1;
    for (int i = 0; i < nr; ++i) {
        bar_status r = read_state(ranks[i]->A, st);
        if (r != BAR_OK) return r;
        const DevState &h = *ranks[i]->A->W.h_state;
        any = any || h.stop != 0;
        next = std::max<int64_t>(next, sizers[i].next(chunk, (long long)h.iter, h.last_rel, tol));
    }
    if (!ranks[0]->loopback) {
#ifdef BAR_WITH_NCCL
        bar_dist D = ranks[0];
        int v[2] = {any ? 1 : 0, (int)next}, out[2] = {0, 0};
        BAR_CUDA(cudaMemcpyAsync(D->d_flag, v, sizeof(v), cudaMemcpyHostToDevice, st));
        BAR_NCCL(ncclAllReduce(D->d_flag, D->d_flag, 2, ncclInt32, ncclMax, D->comm, st));
        BAR_CUDA(cudaMemcpyAsync(out, D->d_flag, sizeof(out), cudaMemcpyDeviceToHost, st));
        BAR_CUDA(cudaStreamSynchronize(st));
        any = out[0] != 0;
        next = out[1];
#endif
    }
    return BAR_OK;
}

// The collective solve for the ranks this process drives (1 with NCCL, all with loopback).
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
    DeviceGuard g(ranks[0]->device);
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
    int64_t launches = nr;
    bar_dist D0 = ranks[0];
    DevState &H = *D0->A->W.h_state;
    const bool p2p = mode == BAR_MODE_ASYNC && D0->p2p;
    if (p2p) {  // boards start "unknown": huge partials keep the estimate above tol until published
        std::vector<double> init(2 * (size_t)D0->nranks, 1e300);
        for (int i = 0; i < nr; ++i)
            BAR_CUDA(cudaMemcpy(ranks[i]->board, init.data(), sizeof(double) * init.size(), cudaMemcpyHostToDevice));
        if (!D0->loopback) {
#ifdef BAR_WITH_NCCL
            BAR_CUDA(cudaStreamSynchronize(st));  // every rank's board reset before any peer publishes
            BAR_NCCL(ncclAllReduce(D0->d_flag, D0->d_flag, 1, ncclInt32, ncclMax, D0->comm, st));
            BAR_CUDA(cudaStreamSynchronize(st));
#endif
        }
    }
    // device time of the local sweeps of this process's first rank (bar_solve_info.sweep_kernel_*)
    KernelTimer &T = D0->A->W.timer;
    timer_reset(T);
    int64_t issued = 0, chunk = 8;
    ChunkSizer sizer;  // collective path: sized from the agreed state (identical on every rank)
    std::vector<ChunkSizer> p2p_sizers(nr);  // p2p: one per rank, agreed in agree_stop
    int64_t p2p_next = 8;
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
                if (p2p) {  // no collective: pull ghosts, sweep, publish, estimate — per rank
                    for (int i = 0; i < nr; ++i) {
                        bar_dist D = ranks[i];
                        SweepArgs a{&D->A->L, D->bbuf, own(D, D->xa), own(D, D->xa), k, D->A->W.state,
                                    D->A->W.partials, nullptr, D->part};
                        if ((r = p2p_iteration(D, a, mode, st, i == 0 ? &T : nullptr, m)) != BAR_OK) return r;
                    }
                    launches += 4 * nr;
                    continue;
                }
                if ((r = exchange(ranks, nr, vin.data(), st)) != BAR_OK) return r;
                for (int i = 0; i < nr; ++i) {
                    bar_dist D = ranks[i];
                    SweepArgs a{&D->A->L, D->bbuf, own(D, vin[i]), own(D, vout[i]), k, D->A->W.state,
                                D->A->W.partials, nullptr, D->part};
                    if (i == 0 && (r = timer_begin(T, m, st)) != BAR_OK) return r;
                    BAR_CUDA(launch_sweep(a, mode, st));
                    if (i == 0 && (r = timer_end(T, st)) != BAR_OK) return r;
                }
                if ((r = reduce_decide(ranks, nr, false, st)) != BAR_OK) return r;
                launches += 2 * nr;
            }
            issued += c;
            if (p2p) {
                if ((r = agree_stop(ranks, nr, st, stopped, p2p_sizers.data(), chunk, tol, p2p_next)) != BAR_OK)
                    return r;
            } else {
                if ((r = read_state(D0->A, st)) != BAR_OK) return r;
                stopped = H.stop != 0;
            }
            if ((r = timer_collect(T, (int64_t)H.iter, 1.0)) != BAR_OK) return r;
            // p2p: each rank's estimate comes from its own board; the ranks agree on the largest
            // of their chunk sizes in agree_stop
            chunk = p2p ? p2p_next : sizer.next(chunk, (long long)H.iter, H.last_rel, tol);
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
    if (info) {
        info->iters = iters;
        info->rel_res = rel;
        info->converged = converged;
        info->cta_iters_min = iters;
        info->cta_iters_max = iters;
        double mb = 0.0;
        for (int i = 0; i < nr; ++i) mb += model_bytes(ranks[i]->A->L);
        info->model_bytes_per_iter = mb;
        info->kernel_launches = launches;
        info->sweep_kernel_ms = T.ms;
        info->sweep_kernel_iters = T.iters;
    }
    if (diverged) {
        set_error("relative residual became non-finite or exceeded 1e30");
        return BAR_ERR_DIVERGED;
    }
    return BAR_OK;
}

}  // namespace
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
    for (int64_t e = 0; e < nnz_local; ++e) {
        const int64_t c = col[e];
        if (c < row_begin) lo.push_back((int32_t)c);
        else if (c >= row_end) hi.push_back((int32_t)c);
    }
    std::sort(lo.begin(), lo.end());
    lo.erase(std::unique(lo.begin(), lo.end()), lo.end());
    std::sort(hi.begin(), hi.end());
    hi.erase(std::unique(hi.begin(), hi.end()), hi.end());
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
    const int64_t nl = row_end - row_begin;
    const int32_t *lo = ghosts, *hi = ghosts + n_ghost_lo;
    for (int64_t e = 0; e < nnz_local; ++e) {
        const int64_t c = col[e];
        if (c < row_begin) {
            const int32_t *it = std::lower_bound(lo, lo + n_ghost_lo, (int32_t)c);
            if (it == lo + n_ghost_lo || *it != c) {
                set_error("column missing from the ghost list");
                return BAR_ERR_INVALID_ARG;
            }
            col_local[e] = (int32_t)(-n_ghost_lo + (it - lo));
        } else if (c >= row_end) {
            const int32_t *it = std::lower_bound(hi, hi + n_ghost_hi, (int32_t)c);
            if (it == hi + n_ghost_hi || *it != c) {
                set_error("column missing from the ghost list");
                return BAR_ERR_INVALID_ARG;
            }
            col_local[e] = (int32_t)(nl + (it - hi));
        } else {
            col_local[e] = (int32_t)(c - row_begin);
        }
    }
    (void)rowptr;
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
    *out = nullptr;
    const int64_t nl = row_end - row_begin;
    if (nranks < 1 || rank < 0 || rank >= nranks || nl < 1 || row_begin < 0 || row_end > n_global ||
        rows_per_block < 1 || rows_per_block > BAR_MAX_ROWS_PER_BLOCK || row_begin % rows_per_block != 0 ||
        n_ghost_lo < 0 || n_ghost_hi < 0 || !recv_counts || !send_counts) {
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
    {
        const char *he = getenv("BAR_HALO");
        D->halo_allgather = he && std::strcmp(he, "allgather") == 0;
    }
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
    if (st == BAR_OK) {
        std::vector<int32_t> hidx(nsend);
        if (nsend) {
            if (is_device_ptr(send_idx)) {
                if (cudaMemcpy(hidx.data(), send_idx, sizeof(int32_t) * nsend, cudaMemcpyDeviceToHost) != cudaSuccess)
                    st = cuda_fail(cudaGetLastError(), "send_idx");
            } else {
                std::memcpy(hidx.data(), send_idx, sizeof(int32_t) * nsend);
            }
        }
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
    D->loopback = nccl_id == nullptr;
    if (st == BAR_OK && !D->loopback) {
#ifdef BAR_WITH_NCCL
        ncclUniqueId id;
        std::memcpy(&id, nccl_id, sizeof(id));
        ncclResult_t rc = ncclCommInitRank(&D->comm, nranks, id, rank);
        if (rc != ncclSuccess) st = nccl_fail((int)rc, "ncclCommInitRank");
#else
        st = nccl_fail(0, "ncclCommInitRank");
#endif
    }
    if (st != BAR_OK) {
        bar_dist_destroy(D);
        return st;
    }
    if (D->loopback) D->peers.assign(1, D);
    *out = D;
    return BAR_OK;
}

bar_status bar_dist_link_loopback(bar_dist *ranks, int nranks) {
    if (!ranks || nranks < 1) {
        set_error("invalid argument");
        return BAR_ERR_INVALID_ARG;
    }
    for (int i = 0; i < nranks; ++i) {
        if (!ranks[i] || !ranks[i]->loopback || ranks[i]->rank != i || ranks[i]->nranks != nranks ||
            ranks[i]->device != ranks[0]->device) {
            set_error("loopback ranks must be 0..nranks-1 of one group on one device, created with nccl_id = NULL");
            return BAR_ERR_INVALID_ARG;
        }
    }
    for (int i = 0; i < nranks; ++i) ranks[i]->peers.assign(ranks, ranks + nranks);
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
        if (!ranks[i] || !ranks[i]->loopback || (int)ranks[i]->peers.size() != nranks || ranks[i]->peers[0] != ranks[0]) {
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
    if (!D->board) BAR_CUDA(cudaMalloc(&D->board, sizeof(double) * 2 * (size_t)D->nranks));
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
        (handles == nullptr && !D->loopback) || (D->loopback && (int)D->peers.size() != D->nranks)) {
        set_error("invalid argument (loopback ranks must be linked first; NCCL ranks need handles)");
        return BAR_ERR_INVALID_ARG;
    }
    DeviceGuard g(D->device);
    if (!D->board) BAR_CUDA(cudaMalloc(&D->board, sizeof(double) * 2 * (size_t)D->nranks));
    if (!D->d_flag) BAR_CUDA(cudaMalloc(&D->d_flag, 2 * sizeof(int)));  // [stop request, next chunk]
    BAR_CUDA(cudaMemset(D->d_flag, 0, 2 * sizeof(int)));
    // ghost j's owner: ghosts are ordered by owner (recv_counts), owners' ranges are contiguous
    std::vector<int32_t> grank(ng), gidx(ng);
    {
        int64_t j = 0;
        for (int p = 0; p < D->nranks; ++p)
            for (int64_t c = 0; c < D->recv_cnt[p]; ++c, ++j) grank[j] = p;
    }
    for (int64_t j = 0; j < ng; ++j) gidx[j] = ghost_src_idx[j];
    std::vector<double *> pown(D->nranks), pboard(D->nranks);
    for (int p = 0; p < D->nranks; ++p) {
        if (handles == nullptr) {  // loopback: the peers live in this process
            bar_dist P = D->peers[p];
            if (!P->board) BAR_CUDA(cudaMalloc(&P->board, sizeof(double) * 2 * (size_t)P->nranks));
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
    cudaFree(D->d_flag);
    bar_destroy(D->A);
    cudaFree(D->xa);
    cudaFree(D->xb);
    cudaFree(D->bbuf);
    cudaFree(D->xio);
    cudaFree(D->send_idx);
    cudaFree(D->send_buf);
    cudaFree(D->ag_buf);
    cudaFree(D->part);
    cudaFree(D->gathered);
    delete D;
}

}  // extern "C"
