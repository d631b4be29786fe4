// api.cu — the C ABI of include/bar.h and the global-iteration driver.
//
// Driver. Sync modes (Jacobi, sync-block): launch m reads x^(m-1) from one buffer, writes x^(m)
// to the other and fuses rel_res(x^(m-1)); its last block sets a device stop flag when
// rel_res(x^(m-1)) <= tol, after which queued launches return immediately. The host enqueues
// launches in growing chunks and reads the 64-byte device state once per chunk (the only
// device->host traffic inside the loop). Async mode iterates in place; its fused residual mixes
// old and new values (eq. 3's shift), so a stop request is confirmed by an exact residual.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstring>
#include <string>

#include "bar_internal.cuh"

namespace bar {

static thread_local std::string g_err;

void set_error(const std::string &msg) { g_err = msg; }

bar_status cuda_fail(cudaError_t e, const char *what) {
    g_err = std::string(what) + ": " + cudaGetErrorString(e);
    cudaGetLastError();
    return e == cudaErrorMemoryAllocation ? BAR_ERR_OOM : BAR_ERR_CUDA;
}

// Helpers shared with dist.cu (declared in bar_internal.cuh).

bool is_device_ptr(const void *p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

bar_status ensure_workspace(bar_matrix A) {
    Workspace &W = A->W;
    const Layout &L = A->L;
    if (!W.state) {
        BAR_CUDA(cudaMalloc(&W.state, sizeof(DevState)));
        BAR_CUDA(cudaMallocHost(&W.h_state, sizeof(DevState)));
        BAR_CUDA(cudaMemset(W.state, 0, sizeof(DevState)));
    }
    if (!W.ring && L.q <= 8192 && use_async_multi(L)) {  // the single-launch kernel's residual ring
        BAR_CUDA(cudaMalloc(&W.ring, sizeof(double) * (kSlots + 1) * (size_t)L.q));  // + the fused residual's row
        BAR_CUDA(cudaMemset(W.ring, 0xFF, sizeof(double) * (kSlots + 1) * (size_t)L.q));  // no tag matches
        BAR_CUDA(cudaMalloc(&W.bsum_arr, sizeof(double) * (size_t)L.q));
    }
    int64_t need = std::max(num_blocks_for(L, BAR_MODE_SYNC_BLOCK), num_blocks_for(L, BAR_MODE_JACOBI));
    if (W.npartials < need) {
        cudaFree(W.partials);
        W.partials = nullptr;
        BAR_CUDA(cudaMalloc(&W.partials, sizeof(double) * 2 * (size_t)need));
        W.npartials = need;
    }
    return BAR_OK;
}

bar_status ensure_buf(double **p, int64_t n) {
    if (!*p) BAR_CUDA(cudaMalloc(p, sizeof(double) * (size_t)n));
    return BAR_OK;
}

double model_bytes(const Layout &L) { return (double)L.nnz * (8 + 4) + (double)L.n * (8 + 8 + 8 + 4); }

// Async driver choice. The fully asynchronous single-launch kernel removes per-iteration
// launches and host round trips, which dominate when one global iteration moves little data;
// for large systems the per-launch kernel streams faster (fewer registers on the hot path).
// bar_tuning.single_launch = 1 / -1 forces either.
bool use_async_multi(const Layout &L) {
    if (L.tune.single_launch) return L.tune.single_launch > 0;
    return model_bytes(L) < 256e6;
}

// single-launch kernels with static ownership (k_block_resident): they count their sweeps in
// res_sweeps and restart at the last completed iteration after a resume
static bool static_multi(const char *k) { return std::strstr(k, "resident") != nullptr; }

bar_status read_state(bar_matrix A, cudaStream_t st) {
    BAR_CUDA(cudaMemcpyAsync(A->W.h_state, A->W.state, sizeof(DevState), cudaMemcpyDeviceToHost, st));
    BAR_CUDA(cudaStreamSynchronize(st));
    return BAR_OK;
}

void timer_reset(KernelTimer &T) {
    T.used = 0;
    T.ms = 0.0;
    T.iters = 0.0;
}

bar_status timer_begin(KernelTimer &T, int64_t m, cudaStream_t st) {
    if (T.used >= KernelTimer::kMax) return BAR_OK;  // not recorded (never reached: chunks <= kMax)
    cudaEvent_t &e0 = T.ev[2 * T.used], &e1 = T.ev[2 * T.used + 1];
    if (!e0) BAR_CUDA(cudaEventCreate(&e0));
    if (!e1) BAR_CUDA(cudaEventCreate(&e1));
    T.m[T.used] = m;
    BAR_CUDA(cudaEventRecord(e0, st));
    return BAR_OK;
}

bar_status timer_end(KernelTimer &T, cudaStream_t st) {
    if (T.used >= KernelTimer::kMax) return BAR_OK;
    BAR_CUDA(cudaEventRecord(T.ev[2 * T.used + 1], st));
    ++T.used;
    return BAR_OK;
}

bar_status timer_collect(KernelTimer &T, int64_t bound, double iters_each) {
    for (int i = 0; i < T.used; ++i) {
        if (T.m[i] > bound) continue;
        float ms = 0.f;
        BAR_CUDA(cudaEventElapsedTime(&ms, T.ev[2 * i], T.ev[2 * i + 1]));
        T.ms += ms;
        T.iters += iters_each;
    }
    T.used = 0;
    return BAR_OK;
}

void timer_free(KernelTimer &T) {
    for (auto &e : T.ev)
        if (e) cudaEventDestroy(e), e = nullptr;
    T.used = 0;
}

}  // namespace bar

using namespace bar;

extern "C" {

const char *bar_last_error(void) { return g_err.c_str(); }

#ifndef BAR_SOURCE_ID
#define BAR_SOURCE_ID "unknown"
#endif
const char *bar_build_id(void) { return "src:" BAR_SOURCE_ID " sm_100a"; }

bar_status bar_create_csr(int64_t n, int64_t nnz, const int32_t *rowptr, const int32_t *col, const double *val,
                          int32_t rows_per_block, int device, bar_matrix *out) {
    g_err.clear();
    if (!out) {
        set_error("out is NULL");
        return BAR_ERR_INVALID_ARG;
    }
    *out = nullptr;
    if (n < 1 || nnz < n || nnz >= (int64_t)INT32_MAX || n >= (int64_t)INT32_MAX || !rowptr || !col || !val) {
        set_error("invalid n/nnz or NULL array (need n >= 1, n <= nnz < 2^31, diagonal in every row)");
        return nnz < n && n >= 1 && rowptr && col && val ? BAR_ERR_BAD_CSR : BAR_ERR_INVALID_ARG;
    }
    if (rows_per_block < 1 || rows_per_block > BAR_MAX_ROWS_PER_BLOCK) {
        set_error("rows_per_block out of [1, BAR_MAX_ROWS_PER_BLOCK]");
        return BAR_ERR_INVALID_ARG;
    }
    NvtxRange nv("bar_create_csr (a1: validate, layout, codes)");
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) {
        cudaGetLastError();
        set_error("invalid CUDA device");
        return BAR_ERR_INVALID_ARG;
    }
    DeviceGuard g(device);
    if (!g.ok) return cuda_fail(cudaGetLastError(), "cudaSetDevice");

    // Inputs: stage host arrays through device copies; device arrays are used in place.
    const int32_t *d_rowptr = rowptr, *d_col = col;
    const double *d_val = val;
    int32_t *t_rowptr = nullptr, *t_col = nullptr;
    double *t_val = nullptr;
    bar_status st_ = BAR_OK;
    int32_t ends[2] = {0, 0};
    cudaStream_t s = nullptr;
    auto *A = new bar_matrix_s();
    A->device = device;
    auto stage = [&](const void *src, void **dst, size_t bytes) -> bar_status {
        if (is_device_ptr(src)) return BAR_OK;
        BAR_CUDA(cudaMalloc(dst, bytes ? bytes : 1));
        BAR_CUDA(cudaMemcpy(*dst, src, bytes, cudaMemcpyHostToDevice));
        return BAR_OK;
    };
    if ((st_ = stage(rowptr, (void **)&t_rowptr, sizeof(int32_t) * (size_t)(n + 1))) != BAR_OK) goto fail;
    if ((st_ = stage(col, (void **)&t_col, sizeof(int32_t) * (size_t)nnz)) != BAR_OK) goto fail;
    if ((st_ = stage(val, (void **)&t_val, sizeof(double) * (size_t)nnz)) != BAR_OK) goto fail;
    if (t_rowptr) d_rowptr = t_rowptr;
    if (t_col) d_col = t_col;
    if (t_val) d_val = t_val;
    if (cudaMemcpy(&ends[0], d_rowptr, sizeof(int32_t), cudaMemcpyDeviceToHost) != cudaSuccess ||
        cudaMemcpy(&ends[1], d_rowptr + n, sizeof(int32_t), cudaMemcpyDeviceToHost) != cudaSuccess) {
        st_ = cuda_fail(cudaGetLastError(), "read rowptr");
        goto fail;
    }
    if (ends[0] != 0 || ends[1] != nnz) {
        set_error("rowptr[0] != 0 or rowptr[n] != nnz");
        st_ = BAR_ERR_BAD_CSR;
        goto fail;
    }
    st_ = build_layout(A->L, n, nnz, d_rowptr, d_col, d_val, rows_per_block, s);
    if (st_ != BAR_OK) goto fail;
    cudaFree(t_rowptr);
    cudaFree(t_col);
    cudaFree(t_val);
    *out = A;
    return BAR_OK;
fail:
    cudaFree(t_rowptr);
    cudaFree(t_col);
    cudaFree(t_val);
    delete A;
    return st_;
}

void bar_destroy(bar_matrix A) {
    if (!A) return;
    if (A->dist) {  // a rank's share (bar_create_csr_dist): its communicator, mappings, buffers
        dist_destroy_handle(A);
        return;
    }
    DeviceGuard g(A->device);
    free_layout(A->L);
    Workspace &W = A->W;
    timer_free(W.timer);
    if (W.graph.exec) cudaGraphExecDestroy(W.graph.exec);
    if (W.graph.cap) cudaStreamDestroy(W.graph.cap);
    cudaFree(W.xbuf);
    cudaFree(W.stage_b);
    cudaFree(W.stage_x);
    cudaFree(W.partials);
    cudaFree(W.frozen);
    cudaFree(W.ring);
    cudaFree(W.bsum_arr);
    cudaFree(W.state);
    cudaFreeHost(W.h_state);
    delete A;
}

bar_status bar_set_tuning(bar_matrix A, const bar_tuning *tuning) {
    g_err.clear();
    if (!A) {
        set_error("NULL handle");
        return BAR_ERR_INVALID_ARG;
    }
    bar_tuning t{};
    if (tuning) t = *tuning;
    if (t.kernel < 0 || t.kernel > 4 || t.async_order < 0 || t.async_order > 3 || t.fronts < 0 || t.async_queue < 0 ||
        t.async_queue > 1 || t.lead < 0 || t.lead > 48 || t.grid_cap < 0 || t.warps < 0 || t.warps > 32 ||
        t.halo < 0 || t.halo > 1 || t.peer > 0 || t.coded > 2 || t.overlap > 0 || t.unroll_off > 0 ||
        t.fuse_residual > 0 || t.lazy_publish > 2 || t.gather_ahead > 0) {
        set_error("bar_tuning field out of range");
        return BAR_ERR_INVALID_ARG;
    }
    A->L.tune = t;
    A->W.graph.b = nullptr;  // a captured solve may have used other kernels: capture again
    A->W.graph.x = nullptr;
    return BAR_OK;
}

bar_status bar_matrix_get_info(bar_matrix A, bar_matrix_info *info) {
    if (!A || !info) {
        set_error("NULL argument");
        return BAR_ERR_INVALID_ARG;
    }
    const Layout &L = A->L;
    info->n = L.n;
    info->nnz = L.nnz;
    info->rows_per_block = L.R;
    info->num_subdomains = L.q;
    info->layout_entries = L.entries;
    info->local_entries = L.local_entries;
    info->model_bytes_per_iter = model_bytes(L);
    info->device = A->device;
    info->last_sweep_kernel = L.last_kernel;
    info->coded = L.codes != nullptr;
    info->layout_bytes_per_iter = (double)L.entries * (8 + (L.codes ? 1 : 4)) + (double)L.n * 24 +
                                  (double)L.nslices * 12 + (L.codes ? (double)L.dict_entries * 4 + (double)L.q * 4 : 0.0) +
                                  (L.xs_len > 0 ? (double)L.q * kMaxIv * 16 : 0.0);
    return BAR_OK;
}

bar_status bar_residual(bar_matrix A, const double *b, const double *x, void *cuda_stream, double *res_norm2,
                        double *b_norm2) {
    g_err.clear();
    if (!A || !b || !x || !res_norm2) {
        set_error("NULL argument");
        return BAR_ERR_INVALID_ARG;
    }
    if (A->dist) return dist_residual_handle(A, b, x, (cudaStream_t)cuda_stream, res_norm2, b_norm2);
    DeviceGuard g(A->device);
    cudaStream_t st = (cudaStream_t)cuda_stream;
    bar_status r = ensure_workspace(A);
    if (r != BAR_OK) return r;
    const int64_t n = A->L.n;
    const double *db = b, *dx = x;
    if (!is_device_ptr(b)) {
        if ((r = ensure_buf(&A->W.stage_b, n)) != BAR_OK) return r;
        BAR_CUDA(cudaMemcpyAsync(A->W.stage_b, b, sizeof(double) * n, cudaMemcpyHostToDevice, st));
        db = A->W.stage_b;
    }
    if (!is_device_ptr(x)) {
        if ((r = ensure_buf(&A->W.stage_x, n)) != BAR_OK) return r;
        BAR_CUDA(cudaMemcpyAsync(A->W.stage_x, x, sizeof(double) * n, cudaMemcpyHostToDevice, st));
        dx = A->W.stage_x;
    }
    BAR_CUDA(launch_init_state(A->W.state, 0.0, st));
    BAR_CUDA(launch_residual(A->L, db, dx, A->W.state, A->W.partials, st));
    if ((r = read_state(A, st)) != BAR_OK) return r;
    *res_norm2 = std::sqrt(A->W.h_state->exact_ss);
    if (b_norm2) *b_norm2 = A->W.h_state->bnorm;
    return BAR_OK;
}

bar_status bar_sweep(bar_matrix A, const double *b, double *x, int32_t k, int64_t nsweeps, bar_mode mode,
                     void *cuda_stream) {
    g_err.clear();
    if (!A || !b || !x || nsweeps < 0 || (mode != BAR_MODE_JACOBI && k < 1) ||
        (mode != BAR_MODE_ASYNC && mode != BAR_MODE_SYNC_BLOCK && mode != BAR_MODE_JACOBI)) {
        set_error("invalid argument");
        return BAR_ERR_INVALID_ARG;
    }
    if (mode == BAR_MODE_JACOBI) k = 1;
    DeviceGuard g(A->device);
    if (!is_device_ptr(b) || !is_device_ptr(x)) {
        set_error("bar_sweep takes device pointers only");
        return BAR_ERR_INVALID_ARG;
    }
    if (A->dist) return dist_sweep_handle(A, b, x, k, nsweeps, mode, (cudaStream_t)cuda_stream);
    cudaStream_t st = (cudaStream_t)cuda_stream;
    bar_status r = ensure_workspace(A);
    if (r != BAR_OK) return r;
    double *buf1 = x;
    if (mode != BAR_MODE_ASYNC) {
        if ((r = ensure_buf(&A->W.xbuf, A->L.n)) != BAR_OK) return r;
        buf1 = A->W.xbuf;
    }
    BAR_CUDA(launch_init_state(A->W.state, -1.0, st));
    if (mode == BAR_MODE_ASYNC && nsweeps > 0) {  // the fully asynchronous kernel when it applies
        SweepArgs a{&A->L, b, x, x, k, A->W.state, A->W.partials, nullptr};
        a.ring = A->W.ring;
        a.bsum_arr = A->W.bsum_arr;
        if (use_async_multi(A->L)) {
            // ||b|| for the single launch's residual estimates (the tagged publication reads the
            // one the x^(0) residual stores; bar_sweep has none otherwise)
            BAR_CUDA(launch_zero_start_residual(A->L, b, A->W.state, A->W.partials, st));
            cudaError_t e = launch_async_multi(a, (long long)nsweeps * A->L.q, st);
            if (e == cudaSuccess) return BAR_OK;
            if (e != cudaErrorNotSupported) return cuda_fail(e, "launch_async_multi");
            cudaGetLastError();
        }
    }
    for (int64_t m = 1; m <= nsweeps; ++m) {
        const double *xi = (m & 1) ? x : buf1;
        double *xo = (mode == BAR_MODE_ASYNC) ? x : ((m & 1) ? buf1 : x);
        SweepArgs a{&A->L, b, xi, xo, k, A->W.state, A->W.partials, nullptr};
        BAR_CUDA(launch_sweep(a, mode, st));
    }
    if (mode != BAR_MODE_ASYNC && (nsweeps & 1))
        BAR_CUDA(cudaMemcpyAsync(x, buf1, sizeof(double) * (size_t)A->L.n, cudaMemcpyDeviceToDevice, st));
    return BAR_OK;
}

bar_status bar_solve_ex(bar_matrix A, const double *b, const double *x0, double *x, int32_t k,
                        int64_t max_global_iters, double tol, bar_mode mode, void *cuda_stream, bar_solve_info *info,
                        const bar_solve_opts *opts) {
    g_err.clear();
    if (!A || !b || !x) {
        set_error("NULL argument");
        return BAR_ERR_INVALID_ARG;
    }
    if (mode != BAR_MODE_ASYNC && mode != BAR_MODE_SYNC_BLOCK && mode != BAR_MODE_JACOBI) {
        set_error("invalid mode");
        return BAR_ERR_INVALID_ARG;
    }
    if ((mode != BAR_MODE_JACOBI && k < 1) || max_global_iters < 0 || !(tol >= 0.0)) {
        set_error("need k >= 1, max_global_iters >= 0, tol >= 0");
        return BAR_ERR_INVALID_ARG;
    }
    if (mode == BAR_MODE_JACOBI) k = 1;
    NvtxRange nv(mode == BAR_MODE_ASYNC ? "bar_solve async" : mode == BAR_MODE_SYNC_BLOCK ? "bar_solve sync-block"
                                                                                          : "bar_solve jacobi");
    if (A->dist) {  // one rank of a row-partitioned solve (collective over its group)
        if (opts && (opts->tau != 1.0 || opts->fail_mask || opts->res_history)) {
            set_error("bar_solve_ex options are not supported on multi-GPU handles");
            return BAR_ERR_INVALID_ARG;
        }
        return dist_solve_handle(A, b, x0, x, k, max_global_iters, tol, mode, (cudaStream_t)cuda_stream, info);
    }
    const double tau = opts ? opts->tau : 1.0;
    if (!(tau > 0.0) || !std::isfinite(tau)) {
        set_error("tau must be a positive finite number");
        return BAR_ERR_INVALID_ARG;
    }
    DeviceGuard g(A->device);
    if (!g.ok) return cuda_fail(cudaGetLastError(), "cudaSetDevice");
    cudaStream_t st = (cudaStream_t)cuda_stream;
    const Layout &L = A->L;
    Workspace &W = A->W;
    const int64_t n = L.n;
    const size_t bytes = sizeof(double) * (size_t)n;
    bar_status r = ensure_workspace(A);
    if (r != BAR_OK) return r;
    KernelTimer &T = W.timer;
    timer_reset(T);
    int64_t launches = 0;
    // N1 failure mask (device copy) and the per-launch window; residual history buffer
    const uint8_t *d_mask = nullptr;
    const int64_t f0 = opts ? opts->fail_start : 0, f1 = opts ? opts->fail_stop : -1;
    if (opts && opts->fail_mask) {
        if (!W.frozen) BAR_CUDA(cudaMalloc(&W.frozen, (size_t)n));
        BAR_CUDA(cudaMemcpyAsync(W.frozen, opts->fail_mask, (size_t)n, cudaMemcpyDefault, st));
        d_mask = W.frozen;
    }
    auto mask_at = [&](int64_t m) -> const uint8_t * {
        return (d_mask && m >= f0 && (f1 < 0 || m < f1)) ? d_mask : nullptr;
    };
    double *d_hist = nullptr;
    struct HistFree {
        double *&p;
        ~HistFree() { cudaFree(p); }
    } hist_free{d_hist};
    if (opts && opts->res_history) BAR_CUDA(cudaMalloc(&d_hist, sizeof(double) * (size_t)(max_global_iters + 2)));
    const bool ext_opts = tau != 1.0 || d_mask || d_hist;

    // End-to-end path: host vectors are staged through device buffers inside the call.
    const double *db = b;
    const bool x_dev = is_device_ptr(x);
    if (!is_device_ptr(b)) {
        if ((r = ensure_buf(&W.stage_b, n)) != BAR_OK) return r;
        BAR_CUDA(cudaMemcpyAsync(W.stage_b, b, bytes, cudaMemcpyHostToDevice, st));
        db = W.stage_b;
    }
    double *buf0 = x;  // iterate buffer 0 (in place for async)
    if (!x_dev) {
        if ((r = ensure_buf(&W.stage_x, n)) != BAR_OK) return r;
        buf0 = W.stage_x;
    }
    // the single-launch async path enqueues the zero start and the state reset with its first
    // pass (inside the replayed graph: two API launches fewer per solve)
    bool async_multi = mode == BAR_MODE_ASYNC && use_async_multi(L);
    if (opts && opts->async_single_launch >= 0) async_multi = mode == BAR_MODE_ASYNC && opts->async_single_launch == 1;
    async_multi = async_multi && !ext_opts && max_global_iters > 0;
    if (x0 == nullptr) {
        if (!async_multi) BAR_CUDA(cudaMemsetAsync(buf0, 0, bytes, st));
    } else if (x0 != x || !x_dev) {
        BAR_CUDA(cudaMemcpyAsync(buf0, x0, bytes, cudaMemcpyDefault, st));
    }
    double *buf1 = nullptr;
    if (mode != BAR_MODE_ASYNC) {
        if ((r = ensure_buf(&W.xbuf, n)) != BAR_OK) return r;
        buf1 = W.xbuf;
    }
    if (!async_multi) BAR_CUDA(launch_init_state(W.state, tol, st));
    ++launches;

    DevState &H = *W.h_state;
    int64_t iters = 0, cta_max = -1;
    double rel = 0.0;
    int converged = 0;
    bool diverged = false, nonfinite = false, bzero = false;
    double *result = buf0;
    int64_t chunk = 8;
    ChunkSizer sizer;  // per-launch sweeps are queued in chunks (bar_internal.cuh)
    auto next_chunk = [&](int64_t c) -> int64_t { return sizer.next(c, (long long)H.iter, H.last_rel, tol); };

    if (mode != BAR_MODE_ASYNC) {
        NvtxRange nvs("global iterations (per-launch sweeps, fused residual)");
        int64_t issued = 0;  // launches m = 1..issued
        bool stopped = false;
        while (issued < max_global_iters && !stopped) {
            const int64_t c = std::min(chunk, max_global_iters - issued);
            for (int64_t i = 0; i < c; ++i) {
                const int64_t m = issued + i + 1;
                SweepArgs a{&L, db, (m & 1) ? buf0 : buf1, (m & 1) ? buf1 : buf0, k, W.state, W.partials, d_hist};
                a.frozen = mask_at(m);
                a.tau = tau;
                if ((r = timer_begin(T, m, st)) != BAR_OK) return r;
                BAR_CUDA(launch_sweep(a, mode, st));
                if ((r = timer_end(T, st)) != BAR_OK) return r;
            }
            launches += c;
            issued += c;
            if ((r = read_state(A, st)) != BAR_OK) return r;
            stopped = H.stop != 0;
            // H.iter counts the launches that ran (those queued after the stop returned at once)
            if ((r = timer_collect(T, (int64_t)H.iter, 1.0)) != BAR_OK) return r;
            chunk = next_chunk(chunk);
        }
        if (stopped) {
            iters = H.conv_iter;
            rel = H.last_rel;
            if (H.diverged == 2) bzero = true;
            else if (H.diverged == 1) diverged = true;
            else converged = 1;
            result = (iters & 1) ? buf1 : buf0;
        } else {
            iters = max_global_iters;
            result = (iters & 1) ? buf1 : buf0;
            BAR_CUDA(launch_residual(L, db, result, W.state, W.partials, st));
            ++launches;
            if ((r = read_state(A, st)) != BAR_OK) return r;
            if (H.bnorm == 0.0) {
                bzero = true;
            } else {
                rel = H.exact_rel;
                if (!std::isfinite(rel) || rel > 1e30) diverged = true;
                converged = rel <= tol;
            }
        }
    } else {
        // async-(k): in place on buf0. Check x^(0) first (exact), then iterate.
        bool multi = async_multi;
        // the single-launch path decides the x^(0) check on the device (k_init_check), so the
        // x^(0) residual, the solve and the confirming residual need ONE host round trip
        auto apply_init = [&](double r0) {
            rel = r0;
            if (H.bnorm == 0.0) bzero = true;
            else if (!std::isfinite(r0)) diverged = true;
            else if (r0 <= tol) converged = 1;
        };
        bool used_multi = false;
        bool fallback = false;  // the single-launch kernel aborted (blocks not co-resident)
        const long long w_end = (long long)max_global_iters * (long long)L.q;
        unsigned long long claimed_before = 0;
        long long m0 = 0;  // static-ownership single-launch kernels: restart iteration after a resume
        double graph_ms = -1.0;  // >= 0: device time of a graph-replayed launch (kernel timestamps)
        // after a single launch (and its confirming residual) completed: iteration accounting and
        // the decision; returns true when the solve must be resumed
        auto after_launch = [&](bool &resume) -> bar_status {
            resume = false;
            used_multi = true;
            const bool resident = static_multi(L.last_kernel);
            {  // this launch swept (claimed now - claimed before) subdomains = that / q global iterations
                const unsigned long long claimed_now = resident ? H.res_sweeps : (H.stop ? H.work_resume : H.work);
                const double its = (double)(claimed_now - claimed_before) / (double)L.q;
                claimed_before = claimed_now;
                if (graph_ms >= 0.0) {  // graph replay: the kernel's own timestamps
                    if (graph_ms > 0.0) {
                        T.ms += graph_ms;
                        T.iters += its;
                    }
                    T.used = 0;
                } else {
                    bar_status rs = timer_collect(T, 1, its);
                    if (rs != BAR_OK) return rs;
                }
            }
            if (H.diverged == 1) {
                diverged = true;
                return BAR_OK;
            }
            rel = H.exact_rel;
            if (!std::isfinite(rel) || rel > 1e30) diverged = true;
            else if (rel <= tol) converged = 1;
            else if (H.aborted) fallback = true;  // continue below with per-launch kernels
            else if (!H.stop || (!resident && (long long)H.work_resume >= w_end)) return BAR_OK;  // max iters
            else {
                m0 = H.iters_done;
                BAR_CUDA(launch_resume_queue(W.state, st, resident));
                resume = true;
            }
            return BAR_OK;
        };
        if (!multi) {
            if (x0 == nullptr) BAR_CUDA(launch_zero_start_residual(L, db, W.state, W.partials, st));
            else BAR_CUDA(launch_residual(L, db, buf0, W.state, W.partials, st));
            ++launches;
            if ((r = read_state(A, st)) != BAR_OK) return r;
            apply_init(H.exact_rel);
        } else {
            // first pass: x^(0) residual, device-side x^(0) check (k_init_check: the kernel then
            // returns at once), the single-launch solve between the timer events, the confirming
            // residual and the state read-back — ONE host round trip
            if ((r = timer_begin(T, 1, st)) != BAR_OK) return r;  // creates the events
            T.used = 0;
            cudaEvent_t ev0 = T.ev[0], ev1 = T.ev[1];
            // k_block_resident with the lazy publication computes the confirming residual itself
            // (sweep.cu, KP::fuse_residual): no residual kernel in the first pass
            auto fused_now = [&]() {
                return static_multi(L.last_kernel) && W.ring && L.tune.lazy_publish >= 0 && L.tune.fuse_residual >= 0;
            };
            auto enqueue_first = [&](cudaStream_t s) -> cudaError_t {
                cudaError_t e = cudaSuccess;
                if (x0 == nullptr && (e = cudaMemsetAsync(buf0, 0, bytes, s)) != cudaSuccess) return e;
                if ((e = launch_init_state(W.state, tol, s)) != cudaSuccess) return e;
                // the residual kernel's last block applies the x^(0) check (k_init_check's rule)
                e = x0 == nullptr ? launch_zero_start_residual(L, db, W.state, W.partials, s, true)
                                  : launch_residual(L, db, buf0, W.state, W.partials, s, nullptr, true);
                if (e != cudaSuccess) return e;
                if ((e = cudaEventRecord(ev0, s)) != cudaSuccess) return e;
                SweepArgs a{&L, db, buf0, buf0, k, W.state, W.partials, nullptr};
                a.ring = W.ring;
                a.bsum_arr = W.bsum_arr;
                if ((e = launch_async_multi(a, w_end, s)) != cudaSuccess) return e;
                if ((e = cudaEventRecord(ev1, s)) != cudaSuccess) return e;
                if (!fused_now() && (e = launch_residual(L, db, buf0, W.state, W.partials, s)) != cudaSuccess) return e;
                return cudaMemcpyAsync(W.h_state, W.state, sizeof(DevState), cudaMemcpyDeviceToHost, s);
            };
            SolveGraph &Gr = W.graph;
            const bool same = Gr.b == db && Gr.x0 == x0 && Gr.x == buf0 && Gr.k == k &&
                              Gr.max_iters == max_global_iters && Gr.tol == tol;
            bool use_graph = L.tune.graph >= 0 && !(same && Gr.unsupported);
            if (use_graph && !(same && Gr.exec)) {  // (re)capture for this call
                if (Gr.exec) cudaGraphExecDestroy(Gr.exec);
                Gr.exec = nullptr;
                Gr.b = db, Gr.x0 = x0, Gr.x = buf0, Gr.k = k, Gr.max_iters = max_global_iters, Gr.tol = tol;
                Gr.unsupported = false;
                if (!Gr.cap) BAR_CUDA(cudaStreamCreateWithFlags(&Gr.cap, cudaStreamNonBlocking));
                cudaGraph_t graph = nullptr;
                BAR_CUDA(cudaStreamBeginCapture(Gr.cap, cudaStreamCaptureModeRelaxed));
                const cudaError_t ec = enqueue_first(Gr.cap);
                const cudaError_t ee = cudaStreamEndCapture(Gr.cap, &graph);
                cudaGetLastError();
                if (ec == cudaSuccess && ee == cudaSuccess && graph &&
                    cudaGraphInstantiate(&Gr.exec, graph, 0) != cudaSuccess)
                    Gr.exec = nullptr;
                if (ec == cudaErrorNotSupported) Gr.unsupported = true;
                if (graph) cudaGraphDestroy(graph);
                cudaGetLastError();
                use_graph = Gr.exec != nullptr;
                Gr.kernel = L.last_kernel;
            }
            if (use_graph) L.last_kernel = Gr.kernel;  // what the replayed graph launches
            cudaError_t e = use_graph ? cudaGraphLaunch(Gr.exec, st) : enqueue_first(st);
            launches += 3;
            if (e == cudaErrorNotSupported) {  // no single-launch kernel: per-launch kernels below
                cudaGetLastError();
                multi = false;
                launches -= 2;
                if ((r = read_state(A, st)) != BAR_OK) return r;
                apply_init(H.init_rel);
            } else {
                BAR_CUDA(e);
                BAR_CUDA(cudaStreamSynchronize(st));
                if (fused_now()) {
                    --launches;
                    if (!H.exact_fused) {  // the fused pass gave up (blocks not co-resident): the kernel
                        BAR_CUDA(launch_residual(L, db, buf0, W.state, W.partials, st));
                        ++launches;
                        if ((r = read_state(A, st)) != BAR_OK) return r;
                    }
                }
                // kernel time from the events, or (graph replay) from the kernel's own timestamps
                T.m[0] = 1;
                T.used = use_graph ? 0 : 1;
                graph_ms = !use_graph ? -1.0 : H.t_last > H.t_first ? (H.t_last - H.t_first) * 1e-6 : 0.0;
                apply_init(H.init_rel);
                if (converged || bzero || diverged) {  // x^(0) met tol: the kernel returned at once
                    T.used = 0;
                } else {
                    bool resume = false;
                    if ((r = after_launch(resume)) != BAR_OK) return r;
                    graph_ms = -1.0;  // resumes launch directly and time with events
                    while (resume && !converged && !diverged) {  // rare: estimate met tol, exact did not
                        SweepArgs a{&L, db, buf0, buf0, k, W.state, W.partials, nullptr};
                        a.m0 = m0;
                        a.ring = W.ring;
                        a.bsum_arr = W.bsum_arr;
                        if ((r = timer_begin(T, 1, st)) != BAR_OK) return r;
                        BAR_CUDA(launch_async_multi(a, w_end, st));
                        if ((r = timer_end(T, st)) != BAR_OK) return r;
                        BAR_CUDA(launch_residual(L, db, buf0, W.state, W.partials, st));
                        launches += 2;
                        if ((r = read_state(A, st)) != BAR_OK) return r;
                        if ((r = after_launch(resume)) != BAR_OK) return r;
                    }
                }
            }
        }
        if (fallback) {
            // the single-launch kernel's blocks were not all resident (other work on the device):
            // continue from the current iterate, counting from the completed global iterations
            BAR_CUDA(launch_continue_per_launch(W.state, st));
            ++launches;
            if ((r = read_state(A, st)) != BAR_OK) return r;
            used_multi = false;
            multi = false;
        }
        if (used_multi) {
            // global iterations needed: the iteration whose fused estimate met tol (the returned
            // x has that many complete global iterations plus the sweeps still in flight when
            // the queue closed, counted in cta_iters_max)
            iters = (converged && H.stop_iter > 0) ? H.stop_iter : H.iters_done;
            // a resident launch that ran to max_global_iters without a stop: every block swept the
            // same number of times (its last iterations may not have been evaluated yet with the
            // lazy residual publication)
            if (!H.stop && static_multi(L.last_kernel)) iters = std::max<int64_t>(iters, (int64_t)(H.res_sweeps / L.q));
            const unsigned long long claimed = static_multi(L.last_kernel) ? H.res_sweeps
                                                                           : (H.stop ? H.work_resume : H.work);
            cta_max = (int64_t)((claimed + L.q - 1) / L.q);
        }
        NvtxRange nvs(multi ? "async: single-launch solve done; per-launch continuation"
                            : "async: global iterations (per-launch sweeps)");
        while (!multi && !converged && !bzero && !diverged && H.iter < max_global_iters) {
            const int64_t c = std::min<int64_t>(chunk, max_global_iters - (int64_t)H.iter);
            for (int64_t i = 0; i < c; ++i) {
                // global iteration index of this launch (launches after a stop request no-op)
                const int64_t m = (int64_t)H.iter + i + 1;
                SweepArgs a{&L, db, buf0, buf0, k, W.state, W.partials, d_hist};
                a.frozen = mask_at(m);
                a.tau = tau;
                if ((r = timer_begin(T, m, st)) != BAR_OK) return r;
                BAR_CUDA(launch_sweep(a, mode, st));
                if ((r = timer_end(T, st)) != BAR_OK) return r;
            }
            launches += c;
            if ((r = read_state(A, st)) != BAR_OK) return r;
            if ((r = timer_collect(T, (int64_t)H.iter, 1.0)) != BAR_OK) return r;  // H.iter: launches that ran
            chunk = next_chunk(chunk);
            if (H.diverged == 1) {
                diverged = true;
                break;
            }
            if (H.stop || H.iter >= max_global_iters) {
                BAR_CUDA(launch_residual(L, db, buf0, W.state, W.partials, st));
                ++launches;
                if ((r = read_state(A, st)) != BAR_OK) return r;
                rel = H.exact_rel;
                if (!std::isfinite(rel) || rel > 1e30) diverged = true;
                else if (rel <= tol) converged = 1;
                else if (H.stop) BAR_CUDA(cudaMemsetAsync(&W.state->stop, 0, sizeof(int), st));
            }
        }
        if (!used_multi) iters = H.iter;
        result = buf0;
    }
    if (bzero) {
        BAR_CUDA(cudaMemsetAsync(buf0, 0, bytes, st));
        result = buf0;
        iters = 0;
        rel = 0.0;
        converged = 1;
        diverged = false;
    }
    if (diverged && iters == 0 && !std::isfinite(rel)) nonfinite = true;
    if (result != x) BAR_CUDA(cudaMemcpyAsync(x, result, bytes, x_dev ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, st));
    BAR_CUDA(cudaStreamSynchronize(st));
    if (d_hist && iters > 0) {  // the device wrote entry m-1 during global iteration m
        const int64_t have = std::min<int64_t>(iters, max_global_iters);
        BAR_CUDA(cudaMemcpy(opts->res_history, d_hist, sizeof(double) * (size_t)have, cudaMemcpyDeviceToHost));
    }
    if (d_hist) opts->res_history[iters] = rel;  // the returned iterate, exactly
    if (info) {
        info->iters = iters;
        info->rel_res = rel;
        info->converged = converged;
        info->cta_iters_min = iters;
        info->cta_iters_max = cta_max >= iters ? cta_max : iters;
        info->model_bytes_per_iter = model_bytes(L);
        info->kernel_launches = launches;
        info->sweep_kernel_ms = T.ms;
        info->sweep_kernel_iters = T.iters;
    }
    if (nonfinite) {
        set_error("non-finite b or x0");
        return BAR_ERR_NONFINITE;
    }
    if (diverged) {
        set_error("relative residual became non-finite or exceeded 1e30 (rho(B) > 1?)");
        return BAR_ERR_DIVERGED;
    }
    return BAR_OK;
}

}  // extern "C"

extern "C" bar_status bar_solve(bar_matrix A, const double *b, const double *x0, double *x, int32_t k,
                                int64_t max_global_iters, double tol, bar_mode mode, void *cuda_stream,
                                bar_solve_info *info) {
    return bar_solve_ex(A, b, x0, x, k, max_global_iters, tol, mode, cuda_stream, info, nullptr);
}
