// sweep.cu — the hot path: block-asynchronous relaxation sweeps on sm_100a.
//
//   k_block<MAXR, ASYNC>  one thread block per subdomain J_l (Alg. 1):
//       a2/a3  read x "as it stands" (ASYNC: relaxed gpu-scope loads of the live in-place x,
//              eq. 3's shift function; SYNC: x^(m) through the read-only path) and form the
//              off-block part s_i = b_i - sum_{j notin J_l} a_ij x_j once (Alg. 1 line 3)
//       a4     k local Jacobi sweeps on shared-memory copies y of x_J (Alg. 1 lines 4-8,
//              double-buffered, CTA barrier between sweeps), in the residual-correction form
//              of eq. 4: y_i <- y_i + (s_i - sum_{j in J_l} a_ij y_j) / a_ii
//       a5     the first sweep's correction numerator IS r_i = (b - A x)_i, so the l2 residual
//               is fused: per-block sum of squares -> fixed-order last-block reduction
//       a6     write y^k back (x_next for sync-block; in place with relaxed stores for async)
//   k_jacobi  eq. 2 in the same correction form, warp per 32-row slice, residual fused.
//   k_residual  standalone ||b - A x||_2 and ||b||_2 (bar_residual, async confirmation).
//
// Every kernel is HBM-bound (about 0.17 flop/byte): no tensor cores. Matrix entries are read
// with coalesced warp-wide loads from the sliced layout (bar_internal.cuh).
#include "bar_internal.cuh"

namespace bar {
namespace {

struct KP {
    const double *__restrict__ val;
    const int32_t *__restrict__ col;
    const int64_t *__restrict__ sptr;
    const int32_t *__restrict__ sw;
    int64_t n;
    int32_t R;
    int32_t spb;
    int64_t nslices;
    const double *b;
    const double *x_in;
    double *x_out;
    int k;
    DevState *state;
    double *partials;  // 2 doubles per block: sum r_i^2, sum b_i^2
    double *hist;
};

enum Kind { kSync = 0, kAsync = 1, kResidual = 2 };

template <bool ASYNC>
__device__ __forceinline__ double ldx(const double *p) {
    if constexpr (ASYNC) {
        double v;
        asm volatile("ld.relaxed.gpu.global.f64 %0, [%1];" : "=d"(v) : "l"(p));
        return v;
    } else {
        return __ldg(p);
    }
}

template <bool ASYNC>
__device__ __forceinline__ void stx(double *p, double v) {
    if constexpr (ASYNC) {
        asm volatile("st.relaxed.gpu.global.f64 [%0], %1;" ::"l"(p), "d"(v) : "memory");
    } else {
        *p = v;
    }
}

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// Deterministic two-level reduction of (rr, bb) over the grid: fixed shuffle tree per warp,
// warps summed in order by thread 0, per-block partials summed in a fixed order by the last
// block to arrive. The last block then updates the device state (stopping rule).
template <int KIND>
__device__ __forceinline__ void reduce_finalize(double rr, double bb, const KP &p) {
    __shared__ double red[2][32];
    __shared__ bool is_last;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, W = blockDim.x >> 5;
    rr = warp_sum(rr);
    bb = warp_sum(bb);
    if (lane == 0) {
        red[0][warp] = rr;
        red[1][warp] = bb;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        double t0 = 0.0, t1 = 0.0;
        for (int w = 0; w < W; ++w) {
            t0 += red[0][w];
            t1 += red[1][w];
        }
        p.partials[2 * blockIdx.x] = t0;
        p.partials[2 * blockIdx.x + 1] = t1;
        __threadfence();
        unsigned int tk = atomicAdd(&p.state->counter, 1u);
        is_last = (tk == gridDim.x - 1);
    }
    __syncthreads();
    if (!is_last) return;
    __threadfence();
    double s0 = 0.0, s1 = 0.0;
    for (unsigned int i = threadIdx.x; i < gridDim.x; i += blockDim.x) {
        s0 += __ldcg(p.partials + 2 * i);
        s1 += __ldcg(p.partials + 2 * i + 1);
    }
    s0 = warp_sum(s0);
    s1 = warp_sum(s1);
    __syncthreads();
    if (lane == 0) {
        red[0][warp] = s0;
        red[1][warp] = s1;
    }
    __syncthreads();
    if (threadIdx.x != 0) return;
    double ss = 0.0, bsq = 0.0;
    for (int w = 0; w < W; ++w) {
        ss += red[0][w];
        bsq += red[1][w];
    }
    DevState *S = p.state;
    S->counter = 0;
    double bn = sqrt(bsq);
    S->bnorm = bn;
    if (KIND == kResidual) {
        S->exact_ss = ss;
        S->exact_rel = bn != 0.0 ? sqrt(ss) / bn : 0.0;
        return;
    }
    long long m = ++S->iter;  // this launch produced x^(m) from x^(m-1)
    double rel = bn != 0.0 ? sqrt(ss) / bn : 0.0;
    S->last_rel = rel;
    if (p.hist) p.hist[m - 1] = rel;
    if (bn == 0.0) {  // b = 0: x = 0 is the answer (reading R2)
        S->stop = 1;
        S->conv_iter = 0;
        S->diverged = 2;
    } else if (!isfinite(rel) || rel > 1e30) {
        S->stop = 1;
        S->diverged = 1;
        S->conv_iter = m - 1;
    } else if (rel <= S->tol) {
        S->stop = 1;
        S->conv_iter = m - 1;  // sync: x^(m-1) (still in the input buffer) is the answer
    }
}

template <int MAXR, bool ASYNC>
__global__ void __launch_bounds__(1024, 1) k_block(KP p) {
    if (*(volatile int *)&p.state->stop) return;
    extern __shared__ double sm[];
    const int R = p.R;
    double *y0 = sm;
    double *y1 = sm + R;
    const int64_t l = blockIdx.x;
    const int64_t TS = l * (int64_t)R;
    const int nrows = (int)min((int64_t)R, p.n - TS);
    const int nsl = (nrows + kSlice - 1) / kSlice;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, W = blockDim.x >> 5;

    // y^0 = x_J (Alg. 1: "read x from global memory")
    for (int i = threadIdx.x; i < nrows; i += blockDim.x) y0[i] = ldx<ASYNC>(p.x_in + TS + i);
    __syncthreads();

    double s[MAXR], dinv[MAXR];
    double rr = 0.0, bb = 0.0;
#pragma unroll
    for (int r = 0; r < MAXR; ++r) {
        const int j = warp + r * W;
        const int loc = j * kSlice + lane;
        s[r] = 0.0;
        dinv[r] = 0.0;
        if (j < nsl && loc < nrows) {
            const int64_t sl = l * p.spb + j;
            const int64_t base = p.sptr[sl] + lane;
            const int w = p.sw[sl];
            const int wl = w & 0xffff, wo = w >> 16;
            const double bi = p.b[TS + loc];
            bb += bi * bi;
            // off-block part, x as it stands (a3)
            double acc = bi;
            const double *vo = p.val + base + (int64_t)wl * kSlice;
            const int32_t *co = p.col + base + (int64_t)wl * kSlice;
            for (int e = 0; e < wo; ++e) acc -= __ldg(vo + e * kSlice) * ldx<ASYNC>(p.x_in + __ldg(co + e * kSlice));
            s[r] = acc;
            const double *vl = p.val + base;
            const int32_t *cl = p.col + base;
            dinv[r] = 1.0 / __ldg(vl);  // local entry 0 is a_ii
            // first local sweep; its correction numerator is the residual r_i (a5)
            for (int e = 0; e < wl; ++e) acc -= __ldg(vl + e * kSlice) * y0[__ldg(cl + e * kSlice)];
            rr += acc * acc;
            y1[loc] = y0[loc] + dinv[r] * acc;
        }
    }
    __syncthreads();
    // sweeps 2..k with the off-block part frozen
    for (int t = 1; t < p.k; ++t) {
        const double *yi = (t & 1) ? y1 : y0;
        double *yo = (t & 1) ? y0 : y1;
#pragma unroll
        for (int r = 0; r < MAXR; ++r) {
            const int j = warp + r * W;
            const int loc = j * kSlice + lane;
            if (j < nsl && loc < nrows) {
                const int64_t sl = l * p.spb + j;
                const int64_t base = p.sptr[sl] + lane;
                const int wl = p.sw[sl] & 0xffff;
                const double *vl = p.val + base;
                const int32_t *cl = p.col + base;
                double acc = s[r];
                for (int e = 0; e < wl; ++e) acc -= __ldg(vl + e * kSlice) * yi[__ldg(cl + e * kSlice)];
                yo[loc] = yi[loc] + dinv[r] * acc;
            }
        }
        __syncthreads();
    }
    const double *yk = (p.k & 1) ? y1 : y0;
    for (int i = threadIdx.x; i < nrows; i += blockDim.x) stx<ASYNC>(p.x_out + TS + i, yk[i]);
    reduce_finalize<ASYNC ? kAsync : kSync>(rr, bb, p);
}

// Jacobi (eq. 2) and the standalone residual: one warp per 32-row slice, 8 slices per block.
template <bool RESIDUAL_ONLY>
__global__ void __launch_bounds__(256) k_rowwise(KP p) {
    if (!RESIDUAL_ONLY && *(volatile int *)&p.state->stop) return;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t sl = (int64_t)blockIdx.x * 8 + warp;
    double rr = 0.0, bb = 0.0;
    if (sl < p.nslices) {
        const int64_t l = sl / p.spb;
        const int64_t TS = l * (int64_t)p.R;
        const int64_t loc = (sl - l * p.spb) * kSlice + lane;
        const int64_t row = TS + loc;
        if (loc < p.R && row < p.n) {
            const int64_t base = p.sptr[sl] + lane;
            const int w = p.sw[sl];
            const int wl = w & 0xffff, wo = w >> 16;
            const double bi = p.b[row];
            bb = bi * bi;
            double acc = bi;
            const double *vo = p.val + base + (int64_t)wl * kSlice;
            const int32_t *co = p.col + base + (int64_t)wl * kSlice;
            for (int e = 0; e < wo; ++e) acc -= __ldg(vo + e * kSlice) * __ldg(p.x_in + __ldg(co + e * kSlice));
            const double *vl = p.val + base;
            const int32_t *cl = p.col + base;
            const double *xJ = p.x_in + TS;
            for (int e = 0; e < wl; ++e) acc -= __ldg(vl + e * kSlice) * __ldg(xJ + __ldg(cl + e * kSlice));
            rr = acc * acc;
            if (!RESIDUAL_ONLY) p.x_out[row] = __ldg(p.x_in + row) + (1.0 / __ldg(vl)) * acc;
        }
    }
    reduce_finalize<RESIDUAL_ONLY ? kResidual : kSync>(rr, bb, p);
}

__global__ void k_init_state(DevState *S, double tol) {
    S->counter = 0;
    S->stop = 0;
    S->diverged = 0;
    S->iter = 0;
    S->conv_iter = -1;
    S->tol = tol;
    S->last_rel = -1.0;
    S->exact_rel = -1.0;
}

KP make_kp(const Layout &L) {
    KP p{};
    p.val = L.val;
    p.col = L.col;
    p.sptr = L.sptr;
    p.sw = L.sw;
    p.n = L.n;
    p.R = L.R;
    p.spb = L.spb;
    p.nslices = L.nslices;
    return p;
}

template <int MAXR, bool ASYNC>
cudaError_t launch_block_t(const KP &p, int threads, size_t smem, unsigned grid, cudaStream_t st) {
    static bool attr_set = false;
    if (!attr_set) {
        cudaError_t e = cudaFuncSetAttribute(k_block<MAXR, ASYNC>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             2 * BAR_MAX_ROWS_PER_BLOCK * (int)sizeof(double));
        if (e != cudaSuccess) return e;
        attr_set = true;
    }
    k_block<MAXR, ASYNC><<<grid, threads, smem, st>>>(p);
    return cudaGetLastError();
}

template <bool ASYNC>
cudaError_t launch_block(const KP &p, const Layout &L, cudaStream_t st) {
    const int W = L.spb < 32 ? L.spb : 32;
    const int need = (L.spb + W - 1) / W;
    const size_t smem = 2 * (size_t)L.R * sizeof(double);
    const unsigned grid = (unsigned)L.q;
    if (need <= 1) return launch_block_t<1, ASYNC>(p, W * 32, smem, grid, st);
    if (need <= 2) return launch_block_t<2, ASYNC>(p, W * 32, smem, grid, st);
    if (need <= 4) return launch_block_t<4, ASYNC>(p, W * 32, smem, grid, st);
    return launch_block_t<8, ASYNC>(p, W * 32, smem, grid, st);
}

}  // namespace

int64_t num_blocks_for(const Layout &L, bar_mode mode) {
    int64_t rowwise = (L.nslices + 7) / 8;
    if (mode == BAR_MODE_JACOBI) return rowwise;
    return L.q > rowwise ? L.q : rowwise;
}

cudaError_t launch_sweep(const SweepArgs &a, bar_mode mode, cudaStream_t st) {
    KP p = make_kp(*a.L);
    p.b = a.b;
    p.x_in = a.x_in;
    p.x_out = a.x_out;
    p.k = a.k;
    p.state = a.state;
    p.partials = a.partials;
    p.hist = a.hist;
    if (mode == BAR_MODE_JACOBI) {
        k_rowwise<false><<<(unsigned)((a.L->nslices + 7) / 8), 256, 0, st>>>(p);
        return cudaGetLastError();
    }
    if (mode == BAR_MODE_ASYNC) return launch_block<true>(p, *a.L, st);
    return launch_block<false>(p, *a.L, st);
}

cudaError_t launch_residual(const Layout &L, const double *b, const double *x, DevState *state, double *partials,
                            cudaStream_t st) {
    KP p = make_kp(L);
    p.b = b;
    p.x_in = x;
    p.state = state;
    p.partials = partials;
    k_rowwise<true><<<(unsigned)((L.nslices + 7) / 8), 256, 0, st>>>(p);
    return cudaGetLastError();
}

cudaError_t launch_init_state(DevState *state, double tol, cudaStream_t st) {
    k_init_state<<<1, 1, 0, st>>>(state, tol);
    return cudaGetLastError();
}

}  // namespace bar
