// sweep.cu — the hot path: block-asynchronous relaxation sweeps on sm_100a.
//
//   k_block<ASYNC, STAGE>  one thread block per subdomain J_l (Alg. 1):
//       a2/a3  read x "as it stands" (ASYNC: relaxed gpu-scope loads of the live in-place x,
//              eq. 3's shift function; SYNC: x^(m) through the read-only path) and form the
//              off-block part s_i = b_i - sum_{j notin J_l} a_ij x_j once (Alg. 1 line 3)
//       a4     k local Jacobi sweeps on shared-memory copies y of x_J (Alg. 1 lines 4-8,
//              double-buffered, CTA barrier between sweeps). The first sweep uses the
//              residual-correction form of eq. 4, y_i <- y_i + (s_i - sum_{j in J_l}
//              a_ij y_j) / a_ii; sweeps 2..k the direct form of Alg. 1 line 6 with the block's
//              local entries staged in shared memory (1/a_ii in the diagonal's slot)
//       a5     the first sweep's correction numerator IS r_i = (b - A x)_i, so the l2 residual
//               is fused: per-block sum of squares -> fixed-order last-block reduction
//       a6     write y^k back (x_next for sync-block; in place with relaxed stores for async)
//   k_rowwise<false>  eq. 2 in the same correction form, warp per 32-row slice, residual fused.
//   k_rowwise<true>  standalone ||b - A x||_2 and ||b||_2 (bar_residual, async confirmation).
//
// Every kernel is HBM-bound (about 0.17 flop/byte): no tensor cores. Matrix entries are read
// with coalesced warp-wide loads from the sliced layout (bar_internal.cuh).
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <map>
#include <mutex>
#include <utility>

#include "bar_internal.cuh"
#include "tma.cuh"

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
    int wlmax;
    int wmax;  // widest slice (local + off-block entries)
    long long w_end;  // async persistent: claims [0, w_end) = global iterations [0, w_end / q)
    long long m0;     // k_block_resident: global iteration index of this launch's first sweep
    int lead;         // k_block_resident: max sweeps a block may run ahead of the last completed iteration
    int fresh_xj;     // async persistent with q < 4 * grid: read x_J when a subdomain starts
    double *dist_out; // multi-GPU: [sum r^2, sum b^2] of this rank (no stopping decision here)
    const uint8_t *frozen;  // N1 failure injection: rows that keep their value (nullable)
    double tau;             // N3: every update scaled, x + tau (v - x)
    int static_claims;      // async: round-robin subdomain order instead of the work queue
    const int32_t *gr;      // ghost-range table (Layout::gr): L2 prefetch targets of the a3 gathers
    int64_t grid_cap;       // > 0: at most this many persistent blocks (k_block_pipe / k_block_duo)
    int claim_chunk;        // static claims: contiguous chunks of subdomains instead of round robin
    int fronts;             // > 0: F fronts (claims_of), async_order = 3
    int64_t l_begin, l_end; // subdomains this launch sweeps (l_end = 0: all; k_block_duo / _pipe only)
    const int *stop;        // the stop flag the kernels poll at start (default &state->stop)
    int slab_ahead;         // k_block_duo: L2 bulk prefetch of the slab two subdomains ahead
    int fuse_residual;      // k_block_resident<LAZY>: exact residual of the final x at the end of the launch
    int gather_ahead;       // k_block_resident (256-thread variants): next iteration's gathers issued after the write-back
    double *ring;           // k_block_resident<LAZY>: [kSlots][q] per-block residual partials
    double *bsum_arr;       //   and [q] per-block sums of b_i^2
    const uint8_t *codes;   // coded layout (Layout::codes): per entry, index into its subdomain's
    const int32_t *dict;    //   dictionary dict[dptr[l] ..) of column offsets d = col - row
    const int32_t *dptr;
    const int32_t *sdict;   // staged gathers (Layout::sdict / iv / xs_len): shared-memory index
    const int32_t *iv;      //   offsets per code, the subdomain's x intervals, their buffer length
    int32_t xs_len;
    int init_check;         // residual kernels: the last block also applies the x^(0) check
};

// Static subdomain claims of persistent block c of G (k_block_pipe / k_block_duo), R15: round
// robin l_j = c + j G (every block advances through the matrix in one front of G subdomains), or
// one contiguous chunk per block, l_j = floor(c q / G) + j < floor((c + 1) q / G) (each block
// sweeps its chunk in order, so a subdomain sees this iteration's values of its predecessors in
// the chunk: eq. 4's shift s(k+1, j) > 0, the block Gauss-Seidel flavour of P:209, on every
// coupling shorter than the chunk). Either way each subdomain is swept exactly once per launch (R7).
struct Claims {
    long long l0, step, lend;
};

// A third order, F "fronts" (tuning.async_order = 3): the subdomains are cut into F contiguous
// ranges and the G / F blocks of front f sweep range f round robin, so each front advances as one
// narrow window of G / F subdomains (F = 1 is round robin over the whole matrix, F = G the chunks).
// A subdomain's far couplings (the plane below on a 3D grid) then lie many rounds back in its
// front, and the x written meanwhile is F windows of about one plane — small enough for L2.
// Claims cover the subdomains [l_begin, l_end) (the whole matrix unless a multi-GPU rank sweeps
// its interior and boundary subdomains in separate launches, dist.cu).
__device__ __forceinline__ Claims claims_of(const KP &p, int64_t q) {
    const long long G = gridDim.x, c = blockIdx.x;
    const long long b0 = p.l_begin, Q = (p.l_end > 0 ? p.l_end : (long long)q) - b0;
    if (p.fronts > 0) {
        const long long F = p.fronts, Gf = G / F, f = c / Gf;
        if (f >= F) return {0, 1, 0};  // G not a multiple of F: the remainder blocks idle
        return {b0 + f * Q / F + c % Gf, Gf, b0 + (f + 1) * Q / F};
    }
    if (p.claim_chunk) return {b0 + c * Q / G, 1, b0 + (c + 1) * Q / G};
    return {b0 + c, G, b0 + Q};
}



// Thread 0: start copying subdomain l's ghost-range entry (kGhostRanges pairs, 32 B) into
// shared memory with cp.async (completion: cp.async.wait_all before reading it).
__device__ __forceinline__ void fetch_ghost_entry(const KP &p, long long l, int64_t q, int32_t *dst) {
    static_assert(kGhostRanges * 2 * sizeof(int32_t) == 32, "two 16-byte cp.async");
    if (l >= q || !p.gr) return;
    const int32_t *src = p.gr + 2 * (int64_t)l * kGhostRanges;
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst + 4)), "l"(src + 4) : "memory");
    asm volatile("cp.async.commit_group;" ::: "memory");
}

// N1/N3 update rule (R17/R18): x_old -> v unless the row is frozen; tau-scaled.
__device__ __forceinline__ double ext_update(double xold, double v, bool frozen, double tau) {
    if (frozen) return xold;
    return tau == 1.0 ? v : xold + tau * (v - xold);
}

// Bounds checks of a checking build only (-DBAR_CHECK_BOUNDS -> libbar_check.so, tools/build.py
// --check-bounds): shared-memory reads against the launch's dynamic allocation and the ring /
// tag indices of the single-launch kernel; a failed check prints the site and traps. (The pool's
// compute-sanitizer was closed during round 2; this build stands in for its memcheck on the
// kernel paths added since the last sanitizer run.)
#ifdef BAR_CHECK_BOUNDS
__device__ __forceinline__ uint32_t dyn_smem_bytes() {
    uint32_t v;
    asm volatile("mov.u32 %0, %%dynamic_smem_size;" : "=r"(v));
    return v;
}
#define BAR_CHECK(cond, what)                                                                          \
    do {                                                                                               \
        if (!(cond)) {                                                                                 \
            printf("BAR_CHECK failed: %s (block %d thread %d, line %d)\n", what, (int)blockIdx.x,     \
                   (int)threadIdx.x, __LINE__);                                                        \
            __trap();                                                                                  \
        }                                                                                              \
    } while (0)
#else
#define BAR_CHECK(cond, what) \
    do {                      \
    } while (0)
#endif

enum Kind { kSync = 0, kAsync = 1, kResidual = 2 };

// Guards the per-kernel static caches of the launchers (dynamic-smem attribute, occupancy):
// different matrices may be used from different host threads at once.
std::recursive_mutex g_launch_mu;

constexpr size_t kSmemBudget = 200 * 1024;  // dynamic smem per block; leaves room for static scratch
constexpr size_t kSmemMax = 227 * 1024 - 1024;  // hardware limit per block minus static scratch

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

// After the exact residual of x^(0) (a7, O5: m = 0 is checked first): init_rel = exact_rel; if
// x^(0) already meets tol (or b = 0, or it is not finite) the solve stops before the first sweep.
__device__ __forceinline__ void init_check_rule(DevState *S) {
    S->init_rel = S->exact_rel;
    if (S->bnorm == 0.0 || !isfinite(S->exact_rel) || S->exact_rel <= S->tol) {
        S->stop = 1;
        S->work = 0x3fffffffffffffffull;  // closed: every claim is past any w_end
    }
}

// The stopping rule (R2/R6/R14) on the global sums of r_i^2 and b_i^2.
// A sweep launch that produced x^(m) reports rel_res(x^(m-1)).
__device__ __forceinline__ void apply_stop_rule(DevState *S, double ss, double bsq, bool residual_only,
                                                double *hist) {
    const double bn = sqrt(bsq);
    S->bnorm = bn;
    if (residual_only) {
        S->exact_ss = ss;
        S->exact_rel = bn != 0.0 ? sqrt(ss) / bn : 0.0;
        return;
    }
    const long long m = ++S->iter;  // this launch produced x^(m) from x^(m-1)
    const double rel = bn != 0.0 ? sqrt(ss) / bn : 0.0;
    S->last_rel = rel;
    if (hist) hist[m - 1] = rel;
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
    if (KIND != kResidual) S->work = 0;  // per-launch async queue (not the persistent one)
    if (p.dist_out) {  // multi-GPU: this rank's sums; the stopping rule runs after the exchange
        p.dist_out[0] = ss;
        p.dist_out[1] = bsq;
        return;
    }
    apply_stop_rule(S, ss, bsq, KIND == kResidual, p.hist);
    if (KIND == kResidual && p.init_check) init_check_rule(S);
}

constexpr int U = 4;  // stored entries of a row loaded together (loads in flight per thread)

// One ascending pass over a row's stored entries — the off-block entries first, then the local
// ones with the diagonal first (layout.cu) — with U loads in flight per chunk:
//   s    = b_i - sum_{j notin J} a_ij x_j          (Alg. 1 line 3, x "as it stands")
//   r    = s - sum_{j in J} a_ij y_j               (= (b - A x)_i when y = x_J: the residual, a5)
//   dinv = 1 / a_ii
// LOCAL_SMEM: local columns index y (shared memory); otherwise y points at x + TS (global).
// STAGE: copy the local entries into shared memory for sweeps 2..k (a4).
template <bool ASYNC, bool LOCAL_SMEM, bool STAGE>
__device__ __forceinline__ void row_pass(const double *__restrict__ v, const int32_t *__restrict__ c, int wo, int w,
                                         const double *x, const double *y, double bi, double &s, double &r,
                                         double &dinv, double *sv, int32_t *sc, int sstride) {
    double acc = bi;
    s = bi;
    dinv = 0.0;
    for (int e0 = 0; e0 < w; e0 += U) {
        double a[U], xv[U];
        int ci[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            if (e0 + u < w) {
                a[u] = __ldg(v + (e0 + u) * kSlice);
                ci[u] = __ldg(c + (e0 + u) * kSlice);
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int e = e0 + u;
            if (e < w) {
                if (e < wo) xv[u] = ldx<ASYNC>(x + ci[u]);
                else if (LOCAL_SMEM) xv[u] = y[ci[u]];
                else xv[u] = ldx<ASYNC>(y + ci[u]);
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int e = e0 + u;
            if (e < w) {
                if (e == wo) {
                    s = acc;
                    dinv = 1.0 / a[u];
                }
                acc -= a[u] * xv[u];
                if (STAGE && e >= wo) {  // slot 0 (the diagonal) keeps 1/a_ii for the direct form
                    sv[(e - wo) * sstride] = e == wo ? dinv : a[u];
                    sc[(e - wo) * sstride] = ci[u];
                }
            }
        }
    }
    r = acc;
}

template <bool ASYNC, bool STAGE>
__global__ void __launch_bounds__(1024, 1) k_block(KP p) {
    if (*(volatile int *)&p.state->stop) return;
    extern __shared__ __align__(128) unsigned char smraw[];
    const int R = p.R;
    const int sstride = p.spb * kSlice;
    double *y0 = reinterpret_cast<double *>(smraw);  // y^t, double-buffered
    double *y1 = y0 + R;
    double *ss = y1 + R;                              // s_i (off-block part, frozen)
    double *sv = ss + R;                              // [wlmax][spb*32] staged local values
    int32_t *sc = reinterpret_cast<int32_t *>(sv + (STAGE ? (size_t)p.wlmax * sstride : 0));  // local cols
    const int64_t l = blockIdx.x;
    const int64_t TS = l * (int64_t)R;
    const int nrows = (int)min((int64_t)R, p.n - TS);
    const int nsl = (nrows + kSlice - 1) / kSlice;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, W = blockDim.x >> 5;
    const int64_t sl0 = l * p.spb;

    // y^0 = x_J (Alg. 1: "read x from global memory")
    for (int i = threadIdx.x; i < nrows; i += blockDim.x) y0[i] = ldx<ASYNC>(p.x_in + TS + i);
    __syncthreads();

    double rr = 0.0, bb = 0.0;
    for (int j = warp; j < nsl; j += W) {
        const int loc = j * kSlice + lane;
        if (loc < nrows) {
            const int64_t base = p.sptr[sl0 + j] + lane;
            const int w = p.sw[sl0 + j];
            const int wl = w & 0xffff, wo = w >> 16;
            const double bi = p.b[TS + loc];
            bb += bi * bi;
            double s, res, dinv;
            // a3 + first local sweep (its correction numerator is the residual, a5)
            row_pass<ASYNC, true, STAGE>(p.val + base, p.col + base, wo, wo + wl, p.x_in, y0, bi, s, res, dinv,
                                         sv + loc, sc + loc, sstride);
            rr += res * res;
            ss[loc] = s;
            y1[loc] = ext_update(y0[loc], y0[loc] + dinv * res, p.frozen && p.frozen[TS + loc], p.tau);
        }
    }
    __syncthreads();
    // a4: sweeps 2..k on the subdomain with the off-block part frozen, in the direct
    // form of Alg. 1 line 6: y_i <- (s_i - sum_{j in J, j != i} a_ij y_j) / a_ii
    for (int t = 1; t < p.k; ++t) {
        const double *yi = (t & 1) ? y1 : y0;
        double *yo = (t & 1) ? y0 : y1;
        for (int j = warp; j < nsl; j += W) {
            const int loc = j * kSlice + lane;
            if (loc < nrows) {
                const int w = p.sw[sl0 + j];
                const int wl = w & 0xffff;
                double acc = ss[loc];
                if (STAGE) {
                    const double *lv = sv + loc;
                    const int32_t *lc = sc + loc;
#pragma unroll 4
                    for (int e = 1; e < wl; ++e) acc -= lv[e * sstride] * yi[lc[e * sstride]];
                    yo[loc] = ext_update(yi[loc], lv[0] * acc, p.frozen && p.frozen[TS + loc], p.tau);
                } else {
                    const int64_t base = p.sptr[sl0 + j] + lane + (int64_t)(w >> 16) * kSlice;
                    const double *vl = p.val + base;
                    const int32_t *cl = p.col + base;
#pragma unroll 4
                    for (int e = 1; e < wl; ++e) acc -= __ldg(vl + e * kSlice) * yi[__ldg(cl + e * kSlice)];
                    yo[loc] = ext_update(yi[loc], acc / __ldg(vl), p.frozen && p.frozen[TS + loc], p.tau);
                }
            }
        }
        __syncthreads();
    }
    // a6: write back
    const double *yk = (p.k & 1) ? y1 : y0;
    for (int i = threadIdx.x; i < nrows; i += blockDim.x) stx<ASYNC>(p.x_out + TS + i, yk[i]);
    reduce_finalize<ASYNC ? kAsync : kSync>(rr, bb, p);
}

// Register-resident variant of k_block for subdomains of at most 32*32*RPT rows whose rows have
// at most WLR local entries: each thread keeps its RPT rows' local entries (values and local
// columns) in registers, so sweeps 2..k read only y from shared memory, and the shared-memory
// footprint (y^t double buffer, 16 B/row) lets two or more blocks share an SM — one block's HBM
// phase overlaps another's local sweeps.
template <bool ASYNC, int WLR, int RPT>
__global__ void __launch_bounds__(1024, 1) k_reg(KP p) {
    if (*(volatile int *)&p.state->stop) return;
    extern __shared__ __align__(128) unsigned char smraw[];
    const int R = p.R;
    double *y0 = reinterpret_cast<double *>(smraw);
    double *y1 = y0 + R;
    const int64_t l = blockIdx.x;
    const int64_t TS = l * (int64_t)R;
    const int nrows = (int)min((int64_t)R, p.n - TS);
    const int nsl = (nrows + kSlice - 1) / kSlice;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, W = blockDim.x >> 5;
    const int64_t sl0 = l * p.spb;
    constexpr int NP = WLR / 2;  // local columns packed two per register (R <= 65536)

    for (int i = threadIdx.x; i < nrows; i += blockDim.x) y0[i] = ldx<ASYNC>(p.x_in + TS + i);
    __syncthreads();

    double lv[RPT][WLR];   // lv[r][0] = 1/a_ii, lv[r][e>0] = local off-diagonal a_ij
    uint32_t lc[RPT][NP];  // local column e in 16-bit half (e & 1) of lc[r][e >> 1]
    double s[RPT];
    bool ok[RPT];
    double rr = 0.0, bb = 0.0;
#pragma unroll
    for (int r = 0; r < RPT; ++r) {
        const int j = warp + r * W;
        const int loc = j * kSlice + lane;
        ok[r] = j < nsl && loc < nrows;
        s[r] = 0.0;
#pragma unroll
        for (int e = 0; e < WLR; ++e) lv[r][e] = 0.0;
#pragma unroll
        for (int e = 0; e < NP; ++e) lc[r][e] = 0;
        if (ok[r]) {
            const int64_t base = p.sptr[sl0 + j] + lane;
            const int w = p.sw[sl0 + j];
            const int wl = w & 0xffff, wo = w >> 16;
            const double *vl = p.val + base + (int64_t)wo * kSlice;
            const int32_t *cl = p.col + base + (int64_t)wo * kSlice;
#pragma unroll
            for (int e = 0; e < WLR; ++e) {
                if (e < wl) {
                    lv[r][e] = __ldg(vl + e * kSlice);
                    lc[r][e >> 1] |= (uint32_t)__ldg(cl + e * kSlice) << (16 * (e & 1));
                }
            }
            const double bi = p.b[TS + loc];
            bb += bi * bi;
            double acc, sdum, ddum;
            // a3: off-block part, x as it stands
            row_pass<ASYNC, false, false>(p.val + base, p.col + base, wo, wo, p.x_in, nullptr, bi, sdum, acc, ddum,
                                          nullptr, nullptr, 0);
            s[r] = acc;
            // first local sweep = residual (a5)
#pragma unroll
            for (int e = 0; e < WLR; ++e) acc -= lv[r][e] * y0[(lc[r][e >> 1] >> (16 * (e & 1))) & 0xffff];
            lv[r][0] = 1.0 / lv[r][0];
            rr += acc * acc;
            y1[loc] = y0[loc] + lv[r][0] * acc;
        }
    }
    __syncthreads();
    // a4: sweeps 2..k, direct form, off-block part frozen
    for (int t = 1; t < p.k; ++t) {
        const double *yi = (t & 1) ? y1 : y0;
        double *yo = (t & 1) ? y0 : y1;
#pragma unroll
        for (int r = 0; r < RPT; ++r) {
            if (ok[r]) {
                const int loc = (warp + r * W) * kSlice + lane;
                double acc = s[r];
#pragma unroll
                for (int e = 1; e < WLR; ++e) acc -= lv[r][e] * yi[(lc[r][e >> 1] >> (16 * (e & 1))) & 0xffff];
                yo[loc] = lv[r][0] * acc;
            }
        }
        __syncthreads();
    }
    const double *yk = (p.k & 1) ? y1 : y0;
    for (int i = threadIdx.x; i < nrows; i += blockDim.x) stx<ASYNC>(p.x_out + TS + i, yk[i]);
    reduce_finalize<ASYNC ? kAsync : kSync>(rr, bb, p);
}

// Bytes of one warp's slice buffer (values + columns) for slices of width <= wmax entries.
__host__ __device__ __forceinline__ uint32_t slice_buf_bytes(int wmax) {
    return (uint32_t)wmax * kSlice * (sizeof(double) + sizeof(int32_t));
}

// Lane 0 of a warp: stream slice `sl` (width w) into buf with two bulk copies completing on bar.
__device__ __forceinline__ void issue_slice(const KP &p, int64_t sl, int w, unsigned char *buf, uint64_t *bar,
                                            int wmax) {
    const int64_t e0 = p.sptr[sl];
    const uint32_t vb = (uint32_t)w * kSlice * sizeof(double), cb = (uint32_t)w * kSlice * sizeof(int32_t);
    mbar_arrive_expect_tx(bar, vb + cb);
    bulk_g2s(buf, p.val + e0, vb, bar);
    bulk_g2s(buf + (size_t)wmax * kSlice * sizeof(double), p.col + e0, cb, bar);
}

// k_reg with the slice stream moved off the register file: each warp bulk-copies (TMA) its
// slice's values and columns into shared memory before anything else, the block then loads
// y^0 = x_J while the copies are in flight, and every lane reads its row's entries from
// shared memory (conflict-free: lane-contiguous). Local entries then live in registers for
// the k sweeps; only the dependent x gathers of the off-block part touch L2/HBM.
template <bool ASYNC, int WLR>
__global__ void __launch_bounds__(1024, 1) k_reg_tma(KP p) {
    if (*(volatile int *)&p.state->stop) return;
    extern __shared__ __align__(128) unsigned char smraw[];
    __shared__ __align__(8) uint64_t bars[32];
    const int R = p.R;
    const int wmax = p.wmax;
    const int64_t l = blockIdx.x;
    const int64_t TS = l * (int64_t)R;
    const int nrows = (int)min((int64_t)R, p.n - TS);
    const int nsl = (nrows + kSlice - 1) / kSlice;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t sl = l * p.spb + warp;
    unsigned char *buf = smraw + (size_t)warp * slice_buf_bytes(wmax);
    double *y0 = reinterpret_cast<double *>(smraw + (size_t)(blockDim.x >> 5) * slice_buf_bytes(wmax));
    double *y1 = y0 + R;
    const bool has_slice = warp < nsl;
    int w = 0, wo = 0, wl = 0;
    if (has_slice) {
        const int sw = p.sw[sl];
        wl = sw & 0xffff;
        wo = sw >> 16;
        w = wl + wo;
        if (lane == 0) {
            mbar_init(&bars[warp], 1);
            fence_mbar_init();
            issue_slice(p, sl, w, buf, &bars[warp], wmax);
        }
    }
    // y^0 = x_J while the slice streams in (Alg. 1: "read x from global memory")
    for (int i = threadIdx.x; i < nrows; i += blockDim.x) y0[i] = ldx<ASYNC>(p.x_in + TS + i);
    __syncthreads();

    constexpr int NP = WLR / 2;
    double lv[WLR];
    uint32_t lc[NP];
    double s = 0.0, rr = 0.0, bb = 0.0;
    const int loc = warp * kSlice + lane;
    const bool ok = has_slice && loc < nrows;
#pragma unroll
    for (int e = 0; e < WLR; ++e) lv[e] = 0.0;
#pragma unroll
    for (int e = 0; e < NP; ++e) lc[e] = 0;
    if (has_slice) {
        mbar_wait(&bars[warp], 0);
        const double *sv = reinterpret_cast<const double *>(buf) + lane;
        const int32_t *sc = reinterpret_cast<const int32_t *>(buf + (size_t)wmax * kSlice * sizeof(double)) + lane;
        if (ok) {
            const double bi = p.b[TS + loc];
            bb = bi * bi;
            // a3: off-block part with the x gathers batched U at a time
            double acc = bi;
            for (int e0 = 0; e0 < wo; e0 += 2 * U) {
                double xv[2 * U];
#pragma unroll
                for (int u = 0; u < 2 * U; ++u)
                    if (e0 + u < wo) xv[u] = ldx<ASYNC>(p.x_in + sc[(e0 + u) * kSlice]);
#pragma unroll
                for (int u = 0; u < 2 * U; ++u)
                    if (e0 + u < wo) acc -= sv[(e0 + u) * kSlice] * xv[u];
            }
            s = acc;
#pragma unroll
            for (int e = 0; e < WLR; ++e) {
                if (e < wl) {
                    lv[e] = sv[(wo + e) * kSlice];
                    lc[e >> 1] |= (uint32_t)sc[(wo + e) * kSlice] << (16 * (e & 1));
                }
            }
            // first local sweep = residual (a5)
#pragma unroll
            for (int e = 0; e < WLR; ++e) acc -= lv[e] * y0[(lc[e >> 1] >> (16 * (e & 1))) & 0xffff];
            lv[0] = 1.0 / lv[0];
            rr = acc * acc;
            y1[loc] = y0[loc] + lv[0] * acc;
        }
    }
    __syncthreads();
    // a4: sweeps 2..k, direct form, off-block part frozen
    for (int t = 1; t < p.k; ++t) {
        const double *yi = (t & 1) ? y1 : y0;
        double *yo = (t & 1) ? y0 : y1;
        if (ok) {
            double acc = s;
#pragma unroll
            for (int e = 1; e < WLR; ++e) acc -= lv[e] * yi[(lc[e >> 1] >> (16 * (e & 1))) & 0xffff];
            yo[loc] = lv[0] * acc;
        }
        __syncthreads();
    }
    const double *yk = (p.k & 1) ? y1 : y0;
    for (int i = threadIdx.x; i < nrows; i += blockDim.x) stx<ASYNC>(p.x_out + TS + i, yk[i]);
    reduce_finalize<ASYNC ? kAsync : kSync>(rr, bb, p);
}

// Persistent k_reg_tma: block c sweeps subdomains l = c, c + G, c + 2G, ... (G = blocks in the
// grid) and, while it runs the k local sweeps of subdomain l, the bulk copies of subdomain
// l + G's slices are already streaming into the other half of a double-buffered slice area —
// the HBM stream never waits for the on-chip sweeps. One residual reduction
// per block per launch instead of one per subdomain.
template <bool ASYNC, int WLR>
__global__ void __launch_bounds__(1024, 1) k_block_pers(KP p) {
    if (*(volatile int *)&p.state->stop) return;
    extern __shared__ __align__(128) unsigned char smraw[];
    __shared__ __align__(8) uint64_t bars[2][32];
    const int R = p.R;
    const int wmax = p.wmax;
    const int W = blockDim.x >> 5;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t sbb = slice_buf_bytes(wmax);
    unsigned char *buf[2] = {smraw + (size_t)warp * sbb, smraw + (size_t)(W + warp) * sbb};
    double *y0 = reinterpret_cast<double *>(smraw + (size_t)2 * W * sbb);
    double *y1 = y0 + R;
    const int64_t G = gridDim.x;
    const int64_t q = (p.n + R - 1) / R;
    auto nsl_of = [&](int64_t l) { return (int)((min((int64_t)R, p.n - l * R) + kSlice - 1) / kSlice); };
    // Subdomain order. Sync-block: static round robin (the per-block partial sums, and so the
    // residual, are then bitwise reproducible). Async: a device work queue, so subdomains are
    // claimed in increasing order by whichever block is free — a monotone processing front, which
    // is what lets later blocks see this iteration's values of earlier ones (eq. 4's shift
    // s(k+1, j) < 0: the block Gauss-Seidel flavour of P:209).
    // double-buffered: claim i+1 is written to slot (i+1) & 1 while slow threads may still be
    // reading claim i from the other slot (compute-sanitizer racecheck, round 2)
    __shared__ long long s_next[2];
    if (threadIdx.x == 0) s_next[0] = ASYNC ? (long long)atomicAdd(&p.state->work, 1ull) : (long long)blockIdx.x;
    __syncthreads();
    int64_t l = s_next[0];
    if (lane == 0) {
        mbar_init(&bars[0][warp], 1);
        mbar_init(&bars[1][warp], 1);
        fence_mbar_init();
        if (l < q && warp < nsl_of(l)) {
            const int64_t sl = l * p.spb + warp;
            const int sw = p.sw[sl];
            issue_slice(p, sl, (sw & 0xffff) + (sw >> 16), buf[0], &bars[0][warp], wmax);
        }
    }
    constexpr int NP = WLR / 2;
    double rr = 0.0, bb = 0.0;
    int i = 0;
    for (int64_t ln; l < q; l = ln, ++i) {
        const int st = i & 1;
        const int64_t TS = l * (int64_t)R;
        const int nrows = (int)min((int64_t)R, p.n - TS);
        const int nsl = (nrows + kSlice - 1) / kSlice;
        if (threadIdx.x == 0)
            s_next[(i + 1) & 1] = ASYNC ? (long long)atomicAdd(&p.state->work, 1ull) : (long long)(l + G);
        __syncthreads();
        ln = s_next[(i + 1) & 1];
        if (lane == 0 && ln < q && warp < nsl_of(ln)) {  // prefetch the next subdomain's slice
            fence_proxy_async_smem();
            const int64_t sl = ln * p.spb + warp;
            const int sw = p.sw[sl];
            issue_slice(p, sl, (sw & 0xffff) + (sw >> 16), buf[st ^ 1], &bars[st ^ 1][warp], wmax);
        }
        for (int r = threadIdx.x; r < nrows; r += blockDim.x) y0[r] = ldx<ASYNC>(p.x_in + TS + r);
        __syncthreads();
        double lv[WLR];
        uint32_t lc[NP];
        double s = 0.0;
        const int loc = warp * kSlice + lane;
        const bool has_slice = warp < nsl;
        const bool ok = has_slice && loc < nrows;
#pragma unroll
        for (int e = 0; e < WLR; ++e) lv[e] = 0.0;
#pragma unroll
        for (int e = 0; e < NP; ++e) lc[e] = 0;
        if (has_slice) {
            const int sw = p.sw[l * p.spb + warp];
            const int wl = sw & 0xffff, wo = sw >> 16;
            mbar_wait(&bars[st][warp], (i >> 1) & 1);
            const double *sv = reinterpret_cast<const double *>(buf[st]) + lane;
            const int32_t *sc =
                reinterpret_cast<const int32_t *>(buf[st] + (size_t)wmax * kSlice * sizeof(double)) + lane;
            if (ok) {
                const double bi = p.b[TS + loc];
                bb += bi * bi;
                double acc = bi;
                for (int e0 = 0; e0 < wo; e0 += 2 * U) {
                    double xv[2 * U];
#pragma unroll
                    for (int u = 0; u < 2 * U; ++u)
                        if (e0 + u < wo) xv[u] = ldx<ASYNC>(p.x_in + sc[(e0 + u) * kSlice]);
#pragma unroll
                    for (int u = 0; u < 2 * U; ++u)
                        if (e0 + u < wo) acc -= sv[(e0 + u) * kSlice] * xv[u];
                }
                s = acc;
#pragma unroll
                for (int e = 0; e < WLR; ++e) {
                    if (e < wl) {
                        lv[e] = sv[(wo + e) * kSlice];
                        lc[e >> 1] |= (uint32_t)sc[(wo + e) * kSlice] << (16 * (e & 1));
                    }
                }
#pragma unroll
                for (int e = 0; e < WLR; ++e) acc -= lv[e] * y0[(lc[e >> 1] >> (16 * (e & 1))) & 0xffff];
                lv[0] = 1.0 / lv[0];
                rr += acc * acc;
                y1[loc] = y0[loc] + lv[0] * acc;
            }
        }
        __syncthreads();
        for (int t = 1; t < p.k; ++t) {
            const double *yi = (t & 1) ? y1 : y0;
            double *yo = (t & 1) ? y0 : y1;
            if (ok) {
                double acc = s;
#pragma unroll
                for (int e = 1; e < WLR; ++e) acc -= lv[e] * yi[(lc[e >> 1] >> (16 * (e & 1))) & 0xffff];
                yo[loc] = lv[0] * acc;
            }
            __syncthreads();
        }
        const double *yk = (p.k & 1) ? y1 : y0;
        for (int r = threadIdx.x; r < nrows; r += blockDim.x) stx<ASYNC>(p.x_out + TS + r, yk[r]);
        __syncthreads();
    }
    reduce_finalize<ASYNC ? kAsync : kSync>(rr, bb, p);
}

// ---------------------------------------------------------------------------------------------
// k_block_stage: the staged block sweep (R = 128-class subdomains). Persistent blocks; everything one subdomain needs —
// its slices' values and columns (one contiguous range of the layout), b_J, x_J (= y^0), and
// the slices' metadata — arrives in one shared-memory STAGE through six bulk copies (TMA) that
// complete on one mbarrier. Two stages: while the block sweeps subdomain l out of one stage,
// the next subdomain streams into the other. Block thread 0 claims subdomains and loads the
// range bounds one subdomain further ahead, so no thread ever waits on a dependent global load
// except the off-block x gathers (a3). x_J may be bulk-copied early even in async mode: within
// one launch only the block that claimed subdomain l writes x_J.
// Requirements (host checks): rows_per_block % 128 == 0 (spb % 4 == 0), spb <= 32, <= WLR
// local entries per row, 16-byte aligned b / x.
struct StageGeom {
    uint32_t vcap;    // entries per stage (spb * 32 * wmax)
    uint32_t o_col, o_b, o_x, o_sptr, o_sw, bytes;
};

__host__ __device__ __forceinline__ StageGeom stage_geom(int R, int spb, int wmax) {
    StageGeom g;
    g.vcap = (uint32_t)spb * kSlice * (uint32_t)wmax;
    g.o_col = g.vcap * 8;
    g.o_b = g.o_col + g.vcap * 4;
    g.o_x = g.o_b + (uint32_t)R * 8;
    g.o_sptr = g.o_x + (uint32_t)R * 8;
    g.o_sw = g.o_sptr + (uint32_t)spb * 8;
    g.bytes = (g.o_sw + (uint32_t)spb * 4 + 127) & ~127u;
    return g;
}

__device__ __forceinline__ unsigned long long globaltimer_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

// Thread 0: the state reset leaves t_first = ~0, t_last = 0; every block of a single-launch
// kernel lowers t_first at its start and raises t_last at its exit.
__device__ __forceinline__ unsigned long long ld_relaxed_u64(const unsigned long long *a) {
    unsigned long long w;
    asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(w) : "l"(a) : "memory");
    return w;
}
__device__ __forceinline__ void stamp_first(DevState *S) { atomicMin(&S->t_first, globaltimer_ns()); }
__device__ __forceinline__ void stamp_last(DevState *S) { atomicMax(&S->t_last, globaltimer_ns()); }

// Thread 0 of a block that finished a subdomain of global iteration m (MULTI): add its
// residual contribution to iteration m's accumulators; the block finishing the q-th subdomain
// of iteration m evaluates rel_res_m (an estimate: each subdomain saw x as it stood) and
// applies the stopping rule (a7).
// A block's claims increase monotonically, so it is done with iteration m when its next claim
// belongs to a later iteration: it then publishes its (count, sum r^2, sum b^2) for m once —
// three atomics and one fence per block per global iteration, not per subdomain.
__device__ __forceinline__ void iteration_publish(const KP &p, long long m, unsigned int cnt, double t0, double t1,
                                                  int64_t q) {
    DevState *S = p.state;
    const int slot = (int)(m % kSlots);
    atomicAdd(&S->ss[slot], t0);
    atomicAdd(&S->bs[slot], t1);
    // the count is an acq_rel atomic: it releases this block's sums and, for the block that
    // completes the iteration, acquires every other block's (no separate gpu-scope fences)
    unsigned int c;
    asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], %2;" : "=r"(c) : "l"(&S->done[slot]), "r"(cnt)
                 : "memory");
    if (c + cnt != (unsigned int)q) return;
    const double ss = __longlong_as_double(
        (long long)atomicExch(reinterpret_cast<unsigned long long *>(&S->ss[slot]), 0ull));
    const double bsq = __longlong_as_double(
        (long long)atomicExch(reinterpret_cast<unsigned long long *>(&S->bs[slot]), 0ull));
    atomicExch(&S->done[slot], 0u);
    const double bn = sqrt(bsq);
    const double rel = bn != 0.0 ? sqrt(ss) / bn : 0.0;
    atomicMax(&S->iters_done, m + 1);
    S->bnorm = bn;
    S->last_rel = rel;
    if (p.hist) p.hist[m] = rel;
    bool stop = false;
    if (bn == 0.0) {
        S->diverged = 2;
        stop = true;
    } else if (!isfinite(rel) || rel > 1e30) {
        S->diverged = 1;
        stop = true;
    } else if (rel <= S->tol && S->stop == 0) {
        S->stop_iter = m + 1;
        stop = true;
    }
    if (stop && S->stop == 0) {
        S->stop = 1;
        // close the queue: later claims see w >= w_end; remember where to resume
        const unsigned long long old = atomicMax(&S->work, (unsigned long long)p.w_end);
        if (old < (unsigned long long)p.w_end) S->work_resume = old;
    }
}

// MULTI (async only): the fully asynchronous solver — ONE launch runs every global iteration.
// Claim w from the device queue means subdomain w mod q of global iteration w / q (R7); there
// is no grid-wide synchronisation at all, so a block may sweep subdomain l of iteration m+1
// while another still sweeps a neighbour in iteration m (eq. 3's bounded shift).
// When the last subdomain of iteration m finishes, its block turns the accumulated residual
// estimate into rel_res_m and raises the stop flag if it meets tol; blocks stop claiming.
// ---------------------------------------------------------------------------------------------
// k_block_pipe: the per-launch staged sweep with a DEEPER pipeline. The matrix slab of a
// subdomain is only needed until its local entries are in registers (end of phase 1), so the
// slab buffer is refilled with subdomain l+2 right then, while l's k-1 local sweeps and l+1's
// whole sweep still run: the HBM stream stays busy through the sweeps (N4: with one subdomain
// of look-ahead the local sweeps were not hidden, 2.2 -> 2.9 ms/iteration on C5 for k 1 -> 5).
// Buffers: two slab buffers (values, columns) and three small row slots [b -> y1 | x -> y0 |
// slice metadata] (b_i is read once, then its slot holds y1_i).
struct PipeGeom {
    uint32_t vcap, vc_bytes, o_x, o_sptr, o_sw, bx_bytes, o_bx;
};

__host__ __device__ __forceinline__ PipeGeom pipe_geom(int R, int spb, int wmax) {
    PipeGeom g;
    g.vcap = (uint32_t)spb * kSlice * (uint32_t)wmax;
    g.vc_bytes = (g.vcap * 12 + 127) & ~127u;  // values (8 B) then columns (4 B)
    g.o_x = (uint32_t)R * 8;
    g.o_sptr = g.o_x + (uint32_t)R * 8;
    g.o_sw = g.o_sptr + (uint32_t)spb * 8;
    g.bx_bytes = (g.o_sw + (uint32_t)spb * 4 + 127) & ~127u;
    g.o_bx = 2 * g.vc_bytes;
    return g;
}

// Issue path. Subdomains are claimed statically (block c sweeps l_j = c + j G, G = grid), so
// every thread knows l_j without communication. Issuing a stage was a ~300-instruction dependent
// chain on one thread (64-bit address arithmetic and uniform-register moves around six bulk
// copies) that every other warp waited for at the next sweep barrier — about a fifth of the
// launch (ncu source-level stall sampling, profiles/). It is now split over four warps, each
// issuing its share right after the barrier that frees the slab buffer:
//   warp 0  mbarrier arrive.expect_tx (before that barrier, off the critical path) + values
//   warp 1  columns + L2 prefetch of the subdomain's ghost x ranges (its a3 gathers)
//   warp 2  b_J and x_J
//   warp 3  slice metadata + cp.async of the bounds/ghost ranges of l_{i+4} into a 4-slot ring
// The arrive.expect_tx of l_{i+2} is posted before the barrier that precedes every copy of
// l_{i+2}, so no copy completes bytes before its phase expects them.
template <bool ASYNC, int WLR, bool EXT = false>
__global__ void __launch_bounds__(WLR > 12 ? 256 : (WLR > 8 ? 512 : 1024), 1) k_block_pipe(KP p) {
    if (*(volatile const int *)p.stop) return;
    extern __shared__ __align__(128) unsigned char smraw[];
    __shared__ __align__(8) uint64_t bars[3];
    __shared__ __align__(16) int64_t bnd[4][2];                // [j % 4]: E0, E1 of l_j
    __shared__ __align__(16) int32_t gsm[4][2 * kGhostRanges];  // [j % 4]: ghost ranges of l_j
    const int R = p.R, spb = p.spb;
    const PipeGeom g = pipe_geom(R, spb, p.wmax);
    const int64_t q = (p.n + R - 1) / R;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const Claims C = claims_of(p, q);
    auto lof = [&](long long j) { return C.l0 + j * C.step; };
    auto nsl_of = [&](long long l) { return (int)((min((int64_t)R, p.n - (int64_t)l * R) + kSlice - 1) / kSlice); };
    auto stage_bytes = [&](long long l, int64_t E0, int64_t E1) -> uint32_t {
        const int nrows = (int)min((int64_t)R, p.n - (int64_t)l * R);
        const uint32_t nsl = (uint32_t)((nrows + kSlice - 1) / kSlice);
        return (uint32_t)(E1 - E0) * 12 + ((uint32_t)nrows & ~1u) * 16 + ((nsl * 8 + 15) & ~15u) +
               ((nsl * 4 + 15) & ~15u);
    };
    // part w (0..3) of the stage of l_j (see above); one lane per warp
    auto issue_part = [&](int w, long long j, const int64_t *bd, const int32_t *gr) {
        const long long l = lof(j);
        if (l >= C.lend) return;
        const int vs = (int)(j & 1), bs = (int)(j % 3);
        const int64_t TS = l * (int64_t)R;
        unsigned char *V = smraw + (size_t)vs * g.vc_bytes;
        unsigned char *B = smraw + g.o_bx + (size_t)bs * g.bx_bytes;
        fence_proxy_async_smem();
        if (w == 0) {
            bulk_g2s_hint(V, p.val + bd[0], (uint32_t)(bd[1] - bd[0]) * 8, &bars[bs], policy_evict_first());
        } else if (w == 1) {
            bulk_g2s_hint(V + (size_t)g.vcap * 8, p.col + bd[0], (uint32_t)(bd[1] - bd[0]) * 4, &bars[bs],
                          policy_evict_first());
            if (gr) prefetch_ghost_x(p.x_in, gr, kGhostRanges);
        } else if (w == 2) {
            const uint32_t trows = (uint32_t)min((int64_t)R, p.n - TS) & ~1u;
            if (trows) {
                bulk_g2s_hint(B, p.b + TS, trows * 8, &bars[bs], policy_evict_first());
                bulk_g2s(B + g.o_x, p.x_in + TS, trows * 8, &bars[bs]);
            }
        } else {
            const uint32_t nsl = (uint32_t)nsl_of(l);
            bulk_g2s(B + g.o_sptr, p.sptr + l * spb, (nsl * 8 + 15) & ~15u, &bars[bs]);
            bulk_g2s(B + g.o_sw, p.sw + l * spb, (nsl * 4 + 15) & ~15u, &bars[bs]);
        }
    };
    // warp 3 lane 0: bounds and ghost ranges of l_j into ring slot j % 4 (one cp.async group)
    auto fetch_ring = [&](long long j) {
        const long long l = lof(j);
        if (l >= C.lend) return;
        const int r = (int)(j & 3);
        asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(&bnd[r][0])), "l"(p.sptr + l * spb)
                     : "memory");
        asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(&bnd[r][1])),
                     "l"(p.sptr + l * spb + nsl_of(l))
                     : "memory");
        if (p.gr) {
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(&gsm[r][0])),
                         "l"(p.gr + 2 * l * kGhostRanges)
                         : "memory");
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(&gsm[r][4])),
                         "l"(p.gr + 2 * l * kGhostRanges + 4)
                         : "memory");
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
    };
    if (threadIdx.x == 0) {  // prologue: stages of l_0 and l_1, ring slots of l_2 and l_3
        for (int j = 0; j < 3; ++j) mbar_init(&bars[j], 1);
        fence_mbar_init();
        for (int j = 0; j < 4; ++j) {
            const long long l = lof(j);
            if (l >= C.lend) break;
            bnd[j][0] = p.sptr[l * spb];
            bnd[j][1] = p.sptr[l * spb + nsl_of(l)];
            for (int t = 0; t < 2 * kGhostRanges; ++t) gsm[j][t] = p.gr ? p.gr[2 * l * kGhostRanges + t] : 0;
        }
        for (int j = 0; j < 2; ++j) {
            const long long l = lof(j);
            if (l >= C.lend) break;
            mbar_arrive_expect_tx(&bars[j], stage_bytes(l, bnd[j][0], bnd[j][1]));
            for (int w = 0; w < 4; ++w) issue_part(w, j, bnd[j], j == 1 && p.gr ? gsm[j] : nullptr);
        }
    }
    __syncthreads();

    constexpr int NP = WLR / 2;
    double rr = 0.0, bb = 0.0;
    for (int i = 0;; ++i) {
        const int vs = i & 1, bs = i % 3;
        const long long l = lof(i);
        if (l >= C.lend) break;
        unsigned char *V = smraw + (size_t)vs * g.vc_bytes;
        unsigned char *B = smraw + g.o_bx + (size_t)bs * g.bx_bytes;
        const int64_t TS = l * (int64_t)R;
        const int nrows = (int)min((int64_t)R, p.n - TS);
        const int nsl = (nrows + kSlice - 1) / kSlice;
        double *y1 = reinterpret_cast<double *>(B);  // b, then y1
        double *y0 = reinterpret_cast<double *>(B + g.o_x);
        mbar_wait(&bars[bs], (i / 3) & 1);
        if (nrows & 1) {  // odd tail of the last subdomain: not bulk-copied
            if (threadIdx.x == 0) y0[nrows - 1] = ldx<ASYNC>(p.x_in + TS + nrows - 1);
            __syncthreads();
        }
        double lv[WLR];
        uint32_t lc[NP];
        double s = 0.0;
        const int loc = warp * kSlice + lane;
        const bool ok = warp < nsl && loc < nrows;
        const bool fz = EXT && ok && p.frozen && p.frozen[TS + loc];  // N1
#pragma unroll
        for (int e = 0; e < WLR; ++e) lv[e] = 0.0;
#pragma unroll
        for (int e = 0; e < NP; ++e) lc[e] = 0;
        if (ok) {
            const int64_t *ssp = reinterpret_cast<const int64_t *>(B + g.o_sptr);
            const int sw = reinterpret_cast<const int32_t *>(B + g.o_sw)[warp];
            const int wl = sw & 0xffff, wo = sw >> 16;
            const int64_t off = ssp[warp] - ssp[0] + lane;
            const double *sv = reinterpret_cast<const double *>(V) + off;
            const int32_t *sc = reinterpret_cast<const int32_t *>(V + (size_t)g.vcap * 8) + off;
            const double bi = loc < (nrows & ~1) ? y1[loc] : p.b[TS + loc];
            bb += bi * bi;
            double acc = bi;
            // a3: off-block part, x as it stands (gathers batched)
            for (int e0 = 0; e0 < wo; e0 += 2 * U) {
                double xv[2 * U];
#pragma unroll
                for (int u = 0; u < 2 * U; ++u)
                    if (e0 + u < wo) xv[u] = ldx<ASYNC>(p.x_in + sc[(e0 + u) * kSlice]);
#pragma unroll
                for (int u = 0; u < 2 * U; ++u)
                    if (e0 + u < wo) acc -= sv[(e0 + u) * kSlice] * xv[u];
            }
            s = acc;
#pragma unroll
            for (int e = 0; e < WLR; ++e) {
                if (e < wl) {
                    lv[e] = sv[(wo + e) * kSlice];
                    lc[e >> 1] |= (uint32_t)sc[(wo + e) * kSlice] << (16 * (e & 1));
                }
            }
            // first local sweep; its correction numerator is the residual (a5)
#pragma unroll
            for (int e = 0; e < WLR; ++e) acc -= lv[e] * y0[(lc[e >> 1] >> (16 * (e & 1))) & 0xffff];
            lv[0] = 1.0 / lv[0];
            rr += acc * acc;
            // y1 takes b's slot: only this thread ever read b[loc]
            if (EXT) y1[loc] = ext_update(y0[loc], y0[loc] + lv[0] * acc, fz, p.tau);
            else y1[loc] = y0[loc] + lv[0] * acc;
        }
        // post the byte count of l_{i+2}'s stage before the barrier that frees its buffers, so
        // that no copy of it can complete bytes before its phase expects them
        if (threadIdx.x == 0 && lof(i + 2) < C.lend) {
            const int r = (i + 2) & 3;
            mbar_arrive_expect_tx(&bars[(i + 2) % 3], stage_bytes(lof(i + 2), bnd[r][0], bnd[r][1]));
        }
        __syncthreads();
        if (warp < 4 && lane == 0) {  // the slab buffer is free: stream l_{i+2} into it
            const int r = (i + 2) & 3;
            issue_part(warp, i + 2, bnd[r], p.gr ? gsm[r] : nullptr);
            if (warp == 3) fetch_ring(i + 4);  // into slot i % 4 (l_i's, no longer read)
        }
        // a4: sweeps 2..k, direct form, off-block part frozen
        for (int t = 1; t < p.k; ++t) {
            const double *yi = (t & 1) ? y1 : y0;
            double *yo = (t & 1) ? y0 : y1;
            if (ok) {
                double acc = s;
#pragma unroll
                for (int e = 1; e < WLR; ++e) acc -= lv[e] * yi[(lc[e >> 1] >> (16 * (e & 1))) & 0xffff];
                if (EXT) yo[loc] = ext_update(yi[loc], lv[0] * acc, fz, p.tau);
                else yo[loc] = lv[0] * acc;
            }
            if (t + 1 < p.k) __syncthreads();  // the write-back reads only the thread's own row
        }
        // ring slot of l_{i+3} complete before the barrier below publishes it (the newest group,
        // l_{i+4}, may stay in flight)
        if (warp == 3 && lane == 0) asm volatile("cp.async.wait_group 1;" ::: "memory");
        // a6: write back
        const double *yk = (p.k & 1) ? y1 : y0;
        for (int r = threadIdx.x; r < nrows; r += blockDim.x) stx<ASYNC>(p.x_out + TS + r, yk[r]);
        __syncthreads();
    }
    if (warp == 3 && lane == 0) asm volatile("cp.async.wait_all;" ::: "memory");
    reduce_finalize<ASYNC ? kAsync : kSync>(rr, bb, p);
}

// ---------------------------------------------------------------------------------------------
// k_block_duo: the pipelined sweep for large subdomains with TWO resident blocks per SM. With one
// 1024-thread block per SM (k_block_pipe at R = 1024), every block-wide barrier of a subdomain
// (after its gathers, after each local sweep) idles the SM's memory pipeline until the slowest
// warp arrives (ncu: barrier stalls were the top reason). Here a block of R/2 threads sweeps a
// subdomain with two rows per thread (slices w and w + R/64 of warp w), and its shared memory
// holds ONE matrix slab (values, columns, slice metadata) plus the y double buffer, so two
// blocks fit per SM and one block's barriers are covered by the other's work. b_J and x_J are
// read with coalesced loads (their ranges are bulk-prefetched into L2 one subdomain ahead), so
// y^0 = x_J is written to shared memory by each thread and the first sweep follows the barrier
// that also frees the slab. The slab of the next subdomain is issued right after that barrier,
// split over four warps as in k_block_pipe; its mbarrier byte count is posted before it.
// Subdomains are claimed statically (claims_of: round robin or contiguous chunks).
// Phase timing of k_block_duo (a profiling build only: -DBAR_PROFILE_DUO, tools/duo_phase_probe.py):
// lane 0 of warps 0 (slab issuer), 3 (b/x, ring and prefetch issuer) and nw - 1 (rows only) sums
// clock64 deltas between the marks over the launch; added into g_duo_prof[0..2][8] at the end.
// Row 3 (thread 0): [0] sum and [1] max over blocks of the block's %globaltimer span (ns) from
// kernel entry to the end of its last subdomain, [2] the latest end, [3] the earliest entry
// (ns, against ~0 initial values: min via atomicMin on ~end), [4] blocks.
#ifdef BAR_PROFILE_DUO
__device__ unsigned long long g_duo_prof[4][8];
#define DUO_PROF_DECL                                                                         \
    const int prof_w = warp == 0 ? 0 : warp == 3 ? 1 : warp == nw - 1 ? 2 : -1;              \
    long long prof_t[8] = {0, 0, 0, 0, 0, 0, 0, 0}, prof_last = clock64();
#define DUO_PROF_ENTRY                \
    unsigned long long prof_t0;       \
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(prof_t0));
#define DUO_PROF_MARK(i)                         \
    if (prof_w >= 0 && lane == 0) {              \
        const long long now = clock64();         \
        prof_t[i] += now - prof_last;            \
        prof_last = now;                         \
    }
#define DUO_PROF_FLUSH                                                                          \
    if (prof_w >= 0 && lane == 0)                                                               \
        for (int i = 0; i < 8; ++i) atomicAdd(&g_duo_prof[prof_w][i], (unsigned long long)prof_t[i]); \
    if (threadIdx.x == 0) {                                                                     \
        unsigned long long t_end;                                                               \
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_end));                               \
        atomicAdd(&g_duo_prof[3][0], t_end - prof_t0);                                          \
        atomicMax(&g_duo_prof[3][1], t_end - prof_t0);                                          \
        atomicMax(&g_duo_prof[3][2], t_end);                                                    \
        atomicMax(&g_duo_prof[3][3], ~prof_t0);                                                 \
        atomicAdd(&g_duo_prof[3][4], 1ull);                                                     \
    }
#else
#define DUO_PROF_ENTRY
#define DUO_PROF_DECL
#define DUO_PROF_MARK(i)
#define DUO_PROF_FLUSH
#endif

struct DuoGeom {
    uint32_t vcap, o_col, o_dict, o_sptr, o_sw, o_ya, o_yb, o_xs, o_bj, o_xj, bytes;
};

// coded: the column block holds 1-byte codes and is followed by the subdomain's dictionary
// (<= kDictMax int32 offsets); otherwise int32 columns. xs_len > 0 (staged gathers): a buffer
// of xs_len doubles for the subdomain's off-block x intervals.
__host__ __device__ __forceinline__ DuoGeom duo_geom(int R, int spb, int wmax, bool coded = false, int xs_len = 0,
                                                     bool bx = false) {
    DuoGeom g;
    g.vcap = (uint32_t)spb * kSlice * (uint32_t)wmax;
    g.o_col = g.vcap * 8;
    g.o_dict = (g.o_col + g.vcap * (coded ? 1 : 4) + 15) & ~15u;
    g.o_sptr = (g.o_dict + (coded ? kDictMax * 4 : 0) + 15) & ~15u;
    g.o_sw = g.o_sptr + (((uint32_t)spb * 8 + 15) & ~15u);
    g.o_ya = (g.o_sw + (((uint32_t)spb * 4 + 15) & ~15u) + 127) & ~127u;
    g.o_yb = g.o_ya + (uint32_t)R * 8;
    g.o_xs = g.o_yb + (uint32_t)R * 8;
    g.o_bj = g.o_xs + (uint32_t)xs_len * 8;  // bx: b_J and x_J staged with the slab
    g.o_xj = g.o_bj + (bx ? (uint32_t)R * 8 : 0u);
    g.bytes = g.o_xj + (bx ? (uint32_t)R * 8 : 0u);
    return g;
}

// CODED: 0 int32 columns; 1 coded columns, off-block x gathered entry by entry from global
// memory (relaxed loads); 2 coded columns with STAGED gathers: at the start of each subdomain the
// block copies its off-block x intervals (Layout::iv, at most kMaxIv, x "as it stands", relaxed
// loads, one coalesced pass) into shared memory, and phase 1 reads x there (Layout::sdict).
// BX: b_J and x_J ride with the slab (two more bulk copies on the slab's mbarrier) instead of
// per-row global loads in phase 1. x_J of l_{j+1} is read when its slab is issued, during l_j's
// sweeps: only the block that sweeps l_{j+1} writes those rows in this launch (static claims), so
// the bulk read races with no write. Requires even n (16-byte copies end inside b and x).
// WOR > 0 (coded columns, <= WOR off-block entries per row): phase 1 fully unrolled over the
// off-block entries in three stages — (A) both rows' codes, offsets and all their gathers issued,
// (C) the off-block sums, (B) the local entries into registers — with one 64-bit row base per row
// and 32-bit offsets (the generic loop re-derived a 64-bit address per entry and exposed one
// gather latency per row). WOR = 4 (3D stencils at R = two grid lines); measured on B200 (round
// 2, tools/kernel_ab.py, same box): C5 async 2.35 vs 2.50 ms, sync-block 2.32 vs 2.39 ms per
// launch. With up to 8 off-block entries (2D 9-point, C4) the 16 gathered values of two rows
// spill at 64 registers and one row at a time is no faster than the generic loop (0.359 / 0.378
// vs 0.346 ms), so WOR = 8 is not built.
template <bool ASYNC, int WLR, bool EXT = false, int CODED = 0, bool BX = false, int WOR = 0>
__global__ void __launch_bounds__(512, 2) k_block_duo(KP p) {
    DUO_PROF_ENTRY
    if (*(volatile const int *)p.stop) return;
    extern __shared__ __align__(128) unsigned char smraw[];
    __shared__ __align__(8) uint64_t bar;
    __shared__ __align__(16) int64_t bnd[4][2];                // [j % 4]: E0, E1 of l_j
    __shared__ __align__(16) int32_t gsm[4][2 * kGhostRanges];  // [j % 4]: ghost ranges of l_j
    __shared__ __align__(16) int32_t dbd[4][2];                 // [j % 4]: dictionary D0, D1 (CODED)
    __shared__ __align__(16) int32_t ivs[CODED == 2 ? 4 : 1][4 * kMaxIv];  // [j % 4]: x intervals of l_j
    const int R = p.R, spb = p.spb;
    const DuoGeom g = duo_geom(R, spb, p.wmax, CODED != 0, CODED == 2 ? p.xs_len : 0, BX);
    const int64_t q = (p.n + R - 1) / R;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int nw = blockDim.x >> 5;  // = spb / 2
    double *ya = reinterpret_cast<double *>(smraw + g.o_ya);
    double *yb = reinterpret_cast<double *>(smraw + g.o_yb);
    const Claims C = claims_of(p, q);
    auto lof = [&](long long j) { return C.l0 + j * C.step; };
    auto nsl_of = [&](long long l) { return (int)((min((int64_t)R, p.n - (int64_t)l * R) + kSlice - 1) / kSlice); };
    auto slab_bytes = [&](long long l, const int64_t *bd, const int32_t *db) -> uint32_t {
        const uint32_t nsl = (uint32_t)nsl_of(l);
        const uint32_t colb = CODED ? (uint32_t)(bd[1] - bd[0]) + (uint32_t)(db[1] - db[0]) * 4
                                    : (uint32_t)(bd[1] - bd[0]) * 4;
        const uint32_t bx = BX ? 2u * 8u * (uint32_t)min((int64_t)R, p.n - (int64_t)l * R) : 0u;
        return (uint32_t)(bd[1] - bd[0]) * 8 + colb + ((nsl * 8 + 15) & ~15u) + ((nsl * 4 + 15) & ~15u) + bx;
    };
    // part w of the issue for l_j (slab) and the L2 prefetches of what l_j / l_{j+1} read directly
    // (w = 3: b_J and x_J; the ghost ranges are prefetched separately, ghost_prefetch)
    auto issue_part = [&](int w, long long j) {
        const long long l = lof(j);
        if (l >= C.lend) return;
        const int64_t *bd = bnd[j & 3];
        if (w == 3) {  // what l_j's first phase reads directly: b_J, x_J and its ghost x ranges
            const int64_t TS = l * (int64_t)R;
            const uint32_t nrows = (uint32_t)min((int64_t)R, p.n - TS);
            if (BX) {  // b_J, x_J with the slab; only the ghost ranges are prefetched into L2
                fence_proxy_async_smem();
                bulk_g2s_hint(smraw + g.o_bj, p.b + TS, nrows * 8, &bar, policy_evict_first());
                bulk_g2s(smraw + g.o_xj, p.x_in + TS, nrows * 8, &bar);
                return;
            }
            const uintptr_t b0 = reinterpret_cast<uintptr_t>(p.b + TS) & ~(uintptr_t)15;
            const uintptr_t b1 = (reinterpret_cast<uintptr_t>(p.b + TS + nrows) + 15) & ~(uintptr_t)15;
            bulk_prefetch_l2_hint(reinterpret_cast<const void *>(b0), (uint32_t)(b1 - b0), policy_evict_first());
            const uintptr_t x0 = reinterpret_cast<uintptr_t>(p.x_in + TS) & ~(uintptr_t)15;
            const uintptr_t x1 = (reinterpret_cast<uintptr_t>(p.x_in + TS + nrows) + 15) & ~(uintptr_t)15;
            bulk_prefetch_l2(reinterpret_cast<const void *>(x0), (uint32_t)(x1 - x0));
            return;
        }
        fence_proxy_async_smem();
        const uint32_t ne = (uint32_t)(bd[1] - bd[0]);
        if (w == 0) {
            bulk_g2s_hint(smraw, p.val + bd[0], ne * 8, &bar, policy_evict_first());
        } else if (w == 1) {
            if (CODED) {
                const int32_t *db = dbd[j & 3];
                bulk_g2s_hint(smraw + g.o_col, p.codes + bd[0], ne, &bar, policy_evict_first());
                bulk_g2s(smraw + g.o_dict, (CODED == 2 ? p.sdict : p.dict) + db[0], (uint32_t)(db[1] - db[0]) * 4,
                         &bar);
            } else {
                bulk_g2s_hint(smraw + g.o_col, p.col + bd[0], ne * 4, &bar, policy_evict_first());
            }
        } else {
            const uint32_t nsl = (uint32_t)nsl_of(l);
            bulk_g2s(smraw + g.o_sptr, p.sptr + l * spb, (nsl * 8 + 15) & ~15u, &bar);
            bulk_g2s(smraw + g.o_sw, p.sw + l * spb, (nsl * 4 + 15) & ~15u, &bar);
            // the slab after this one into L2 already: a second slab buffer, in L2 instead of
            // shared memory, so HBM keeps streaming while both blocks of the SM sweep locally
            if (p.slab_ahead && lof(j + 1) < C.lend) {
                const int64_t *bn = bnd[(j + 1) & 3];
                const uint32_t nn = (uint32_t)(bn[1] - bn[0]);
                bulk_prefetch_l2(p.val + bn[0], nn * 8);
                if (CODED) bulk_prefetch_l2(p.codes + bn[0], (nn + 15) & ~15u);
                else bulk_prefetch_l2(p.col + bn[0], nn * 4);
            }
        }
    };
    // warp 3 lane 0: bounds and ghost ranges of l_j into ring slot j % 4 (one cp.async group)
    auto fetch_ring = [&](long long j) {
        const long long l = lof(j);
        if (l >= C.lend) return;
        const int r = (int)(j & 3);
        asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(&bnd[r][0])), "l"(p.sptr + l * spb)
                     : "memory");
        asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(&bnd[r][1])),
                     "l"(p.sptr + l * spb + nsl_of(l))
                     : "memory");
        if (p.gr) {
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(&gsm[r][0])),
                         "l"(p.gr + 2 * l * kGhostRanges)
                         : "memory");
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(&gsm[r][4])),
                         "l"(p.gr + 2 * l * kGhostRanges + 4)
                         : "memory");
        }
        if (CODED) {
            asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(&dbd[r][0])), "l"(p.dptr + l)
                         : "memory");
            asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(&dbd[r][1])), "l"(p.dptr + l + 1)
                         : "memory");
        }
        if (CODED == 2) {
#pragma unroll
            for (int t = 0; t < kMaxIv; ++t)
                asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(&ivs[r & 3][4 * t])),
                             "l"(p.iv + 4 * (l * kMaxIv + t))
                             : "memory");
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
    };
    if (threadIdx.x == 0) {  // prologue: ring slots of l_0 .. l_2, the slab of l_0
        mbar_init(&bar, 1);
        fence_mbar_init();
        for (int j = 0; j < 3; ++j) {
            const long long l = lof(j);
            if (l >= C.lend) break;
            bnd[j][0] = p.sptr[l * spb];
            bnd[j][1] = p.sptr[l * spb + nsl_of(l)];
            for (int t = 0; t < 2 * kGhostRanges; ++t) gsm[j][t] = p.gr ? p.gr[2 * l * kGhostRanges + t] : 0;
            if (CODED) {
                dbd[j][0] = p.dptr[l];
                dbd[j][1] = p.dptr[l + 1];
            }
            if (CODED == 2)
                for (int t = 0; t < 4 * kMaxIv; ++t) ivs[j & 3][t] = p.iv[4 * l * kMaxIv + t];
        }
        mbar_arrive_expect_tx(&bar, slab_bytes(lof(0), bnd[0], dbd[0]));
        for (int w = 0; w < 4; ++w) issue_part(w, 0);
        if (p.gr && lof(0) < C.lend) prefetch_ghost_x(p.x_in, gsm[0], kGhostRanges);
    }
    // the issue after the slab is freed, split over warps so that no warp's share holds up the
    // barrier after the first sweep: roles 0..3 the slab parts (issue_part), 4 the ghost-range L2
    // prefetch, 5 the ring of bounds (cp.async, always the same thread: its groups are per thread)
    constexpr int kRoles = 6;
    const int ring_warp = (kRoles - 1) % nw;
    double *xs = reinterpret_cast<double *>(smraw + g.o_xs);
    const uint32_t sxs = smem_u32(xs);
    if (CODED == 2)  // slots past a subdomain's intervals are read (times 0) by padding entries
        for (int t = threadIdx.x; t < p.xs_len; t += blockDim.x) xs[t] = 0.0;
    __syncthreads();

    constexpr int NP = WLR / 2;
    double rr = 0.0, bb = 0.0;
    DUO_PROF_DECL
    for (int i = 0;; ++i) {
        const long long l = lof(i);
        if (l >= C.lend) break;
        const int64_t TS = l * (int64_t)R;
        const int nrows = (int)min((int64_t)R, p.n - TS);
        const int nsl = (nrows + kSlice - 1) / kSlice;
        DUO_PROF_MARK(7)
        if (CODED == 2) {  // a3 staged: the off-block x intervals, as they stand, into shared memory
            const int32_t *iv = ivs[i & 3];
#pragma unroll
            for (int t = 0; t < kMaxIv; ++t) {
                const int32_t lo = iv[4 * t], len = iv[4 * t + 1], base = iv[4 * t + 2];
                for (int u = threadIdx.x; u < len; u += blockDim.x) xs[base + u] = ldx<ASYNC>(p.x_in + lo + u);
            }
            __syncthreads();
        }
        mbar_wait(&bar, i & 1);
        DUO_PROF_MARK(0)
        double lv[2][WLR];
        uint32_t lc[2][NP];
        double s[2] = {0.0, 0.0};
#pragma unroll
        for (int h = 0; h < 2; ++h) {
#pragma unroll
            for (int e = 0; e < WLR; ++e) lv[h][e] = 0.0;
#pragma unroll
            for (int e = 0; e < NP; ++e) lc[h][e] = 0;
        }
        auto row_of = [&](int h) { return (warp + h * nw) * kSlice + lane; };  // local row of slice h
        // a2/a3: b_i and x_i (direct, L2-prefetched; x_i -> y^0), the off-block part with x as
        // it stands, the local entries into registers
        const int64_t *ssp = reinterpret_cast<const int64_t *>(smraw + g.o_sptr);
        const uint32_t sb = smem_u32(smraw);
        if constexpr (WOR > 0) {
            static_assert(CODED == 1, "the unrolled phase 1 reads coded columns");
            const uint32_t ad = sb + g.o_dict;
            uint32_t av[2], ac[2];
            int wl[2], wo[2];
            double xv[2][WOR], bi[2], xj[2];
            // (A) offsets and gathers of row h (x as it stands)
            auto stage_a = [&](int h) {
                const int sl = warp + h * nw, loc = row_of(h);
                const bool v = sl < nsl && loc < nrows;
                const int sw = v ? lds_s32(sb + g.o_sw + 4 * sl) : 0;
                wl[h] = sw & 0xffff;
                wo[h] = sw >> 16;
                const uint32_t off = v ? (uint32_t)(ssp[sl] - ssp[0]) + lane : 0u;
                av[h] = sb + off * 8;
                ac[h] = sb + g.o_col + off;
                BAR_CHECK(!v || (off + (uint32_t)(wo[h] + wl[h] - 1) * kSlice + 1) * 8 <= g.o_col, "duo slab values");
                BAR_CHECK(!v || off + (uint32_t)(wo[h] + wl[h] - 1) * kSlice + 1 <= g.o_dict - g.o_col, "duo slab codes");
                const double *xr = p.x_in + (TS + loc);
#pragma unroll
                for (int e = 0; e < WOR; ++e)
                    xv[h][e] = e < wo[h] ? ldx<ASYNC>(xr + lds_s32(ad + 4 * lds_u8(ac[h] + e * kSlice))) : 0.0;
                bi[h] = !v ? 0.0 : BX ? lds_f64(sb + g.o_bj + 8u * loc) : p.b[TS + loc];
                xj[h] = !v ? 0.0 : BX ? lds_f64(sb + g.o_xj + 8u * loc) : ldx<ASYNC>(xr);
            };
            // (B) local entries of row h into registers, branch-free (slots past wl read in-bounds
            // shared memory, zeroed)
            auto stage_b = [&](int h) {
                const int loc = row_of(h);
#pragma unroll
                for (int e = 0; e < WLR; ++e) {
                    const bool ok = e < wl[h];
                    BAR_CHECK(av[h] + (uint32_t)(wo[h] + e) * kSlice * 8 + 8 - sb <= dyn_smem_bytes(), "duo local value read");
                    BAR_CHECK(ac[h] + (uint32_t)(wo[h] + e) * kSlice + 1 - sb <= dyn_smem_bytes(), "duo local code read");
                    const double v = lds_f64(av[h] + (wo[h] + e) * kSlice * 8);
                    const uint32_t c = (uint32_t)(loc + lds_s32(ad + 4 * lds_u8(ac[h] + (wo[h] + e) * kSlice))) & 0xffffu;
                    lv[h][e] = ok ? v : 0.0;
                    lc[h][e >> 1] |= (ok ? c : 0u) << (16 * (e & 1));
                }
            };
            // (C) s_i = b_i - sum_{j not in J} a_ij x_j; y^0 = x_J
            auto stage_c = [&](int h) {
                const int sl = warp + h * nw, loc = row_of(h);
                double acc = bi[h];
#pragma unroll
                for (int e = 0; e < WOR; ++e)
                    if (e < wo[h]) acc -= lds_f64(av[h] + e * kSlice * 8) * xv[h][e];
                s[h] = acc;
                if (sl < nsl && loc < nrows) ya[loc] = xj[h];
                bb += bi[h] * bi[h];
            };
            // both rows' gathers in flight together; the local entries after the sums, so the
            // gathered values and the local entries are never live at once (64 registers)
            stage_a(0);
            stage_a(1);
            stage_c(0);
            stage_c(1);
            stage_b(0);
            stage_b(1);
        } else
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int sl = warp + h * nw, loc = row_of(h);
            if (sl >= nsl || loc >= nrows) continue;
            const int sw = lds_s32(sb + g.o_sw + 4 * sl);
            const int wl = sw & 0xffff, wo = sw >> 16;
            const uint32_t off = (uint32_t)(ssp[sl] - ssp[0]) + lane;
            const uint32_t av = sb + off * 8, ac = sb + g.o_col + off * (CODED ? 1 : 4), ad = sb + g.o_dict;
            // stored column of entry e: global for off-block entries, local index for local ones
            // (CODED: the offset d = col - row from the subdomain's dictionary)
            auto dcol = [&](int e) -> int32_t {
                return CODED ? lds_s32(ad + 4 * lds_u8(ac + e * kSlice)) : lds_s32(ac + e * kSlice * 4);
            };
            const double bi = BX ? lds_f64(sb + g.o_bj + 8u * loc) : p.b[TS + loc];
            ya[loc] = BX ? lds_f64(sb + g.o_xj + 8u * loc) : ldx<ASYNC>(p.x_in + TS + loc);
            double acc = bi;
            for (int e0 = 0; e0 < wo; e0 += U) {
                double xv[U];
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    if (e0 + u >= wo) continue;
                    if (CODED == 2) xv[u] = lds_f64(sxs + 8u * (uint32_t)(loc + dcol(e0 + u)));
                    else xv[u] = ldx<ASYNC>(p.x_in + (CODED ? TS + loc : 0) + dcol(e0 + u));
                }
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (e0 + u < wo) acc -= lds_f64(av + (e0 + u) * kSlice * 8) * xv[u];
            }
            s[h] = acc;
            // local entries, branch-free: slots past wl read in-bounds shared memory (the regions
            // after the slab) and are zeroed (value 0, column 0)
#pragma unroll
            for (int e = 0; e < WLR; ++e) {
                const bool ok = e < wl;
                const double v = lds_f64(av + (wo + e) * kSlice * 8);
                const uint32_t c = (uint32_t)((CODED ? loc : 0) + dcol(wo + e)) & 0xffffu;
                lv[h][e] = ok ? v : 0.0;
                lc[h][e >> 1] |= (ok ? c : 0u) << (16 * (e & 1));
            }
            bb += bi * bi;
        }
        DUO_PROF_MARK(1)
        // post the byte count of l_{i+1}'s slab before the barrier that frees the buffer
        if (threadIdx.x == 0 && lof(i + 1) < C.lend)
            mbar_arrive_expect_tx(&bar, slab_bytes(lof(i + 1), bnd[(i + 1) & 3], dbd[(i + 1) & 3]));
        __syncthreads();
        DUO_PROF_MARK(2)
        if (lane == 0) {  // the slab is free: stream l_{i+1} into it
            for (int r = warp; r < kRoles; r += nw) {
                if (r < 4) {
                    issue_part(r, i + 1);
                } else if (r == 4) {
                    if (p.gr && lof(i + 1) < C.lend) prefetch_ghost_x(p.x_in, gsm[(i + 1) & 3], kGhostRanges);
                } else {
                    fetch_ring(i + 3);  // into slot (i + 3) % 4 (l_{i-1}'s, no longer read)
                    // ring slot of l_{i+2} complete; the next barrier publishes it (thread 0 reads
                    // it before the first barrier of the next subdomain)
                    asm volatile("cp.async.wait_group 1;" ::: "memory");
                }
            }
        }
        DUO_PROF_MARK(3)
        // first local sweep in the correction form; its numerator is the residual (a5)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int loc = row_of(h);
            if (warp + h * nw >= nsl || loc >= nrows) continue;
            double acc = s[h];
#pragma unroll
            for (int e = 0; e < WLR; ++e) acc -= lv[h][e] * ya[(lc[h][e >> 1] >> (16 * (e & 1))) & 0xffff];
            lv[h][0] = 1.0 / lv[h][0];
            rr += acc * acc;
            const double xo = ya[loc];
            if (EXT) yb[loc] = ext_update(xo, xo + lv[h][0] * acc, p.frozen && p.frozen[TS + loc], p.tau);
            else yb[loc] = xo + lv[h][0] * acc;
        }
        DUO_PROF_MARK(4)
        // every thread writes back exactly its own two rows, so the last sweep needs no barrier
        // before the write-back (the barrier after it guards the buffers' reuse)
        if (p.k > 1) __syncthreads();
        DUO_PROF_MARK(5)
        // a4: sweeps 2..k, direct form, off-block part frozen
        if (EXT) {
            for (int t = 1; t < p.k; ++t) {
                const double *yi = (t & 1) ? yb : ya;
                double *yo = (t & 1) ? ya : yb;
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    const int loc = row_of(h);
                    if (warp + h * nw >= nsl || loc >= nrows) continue;
                    double acc = s[h];
#pragma unroll
                    for (int e = 1; e < WLR; ++e) acc -= lv[h][e] * yi[(lc[h][e >> 1] >> (16 * (e & 1))) & 0xffff];
                    yo[loc] = ext_update(yi[loc], lv[h][0] * acc, p.frozen && p.frozen[TS + loc], p.tau);
                }
                if (t + 1 < p.k) __syncthreads();
            }
        } else {
            // straight-line: row addresses and y indices hoisted out of the sweep loop, rows past
            // the subdomain's end (partial last subdomain) computed on zeroed entries and not stored
            const uint32_t ya_s = smem_u32(ya), yb_s = smem_u32(yb);
            uint32_t yoff[2][WLR], sto[2];
            bool vh[2];
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                vh[h] = warp + h * nw < nsl && row_of(h) < nrows;
                sto[h] = 8u * (uint32_t)row_of(h);
#pragma unroll
                for (int e = 1; e < WLR; ++e) yoff[h][e] = 8u * ((lc[h][e >> 1] >> (16 * (e & 1))) & 0xffffu);
            }
            for (int t = 1; t < p.k; ++t) {
                const uint32_t yi = (t & 1) ? yb_s : ya_s, yo = (t & 1) ? ya_s : yb_s;
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    double acc = s[h];
#pragma unroll
                    for (int e = 1; e < WLR; ++e) acc -= lv[h][e] * lds_f64(yi + yoff[h][e]);
                    if (vh[h]) sts_f64(yo + sto[h], lv[h][0] * acc);
                }
                if (t + 1 < p.k) __syncthreads();
            }
        }
        DUO_PROF_MARK(6)
        // a6: write back (the thread's own two rows)
        double *yk = (p.k & 1) ? yb : ya;
        for (int r = threadIdx.x; r < nrows; r += blockDim.x) stx<ASYNC>(p.x_out + TS + r, yk[r]);
        if (p.k == 1) {
            __syncthreads();  // publishes the ring slot; guards ya against the next phase 1
        } else if (p.k & 1) {
            // no barrier: the next subdomain's y^0 goes into this one's final buffer yk, of which
            // each thread writes only its own rows (already written back above), while threads
            // still in the last sweep read only the other buffer; the barrier after sweep 1
            // published the ring slot
            yb = ya;
            ya = yk;
        }
    }
    DUO_PROF_FLUSH
    if (warp == ring_warp && lane == 0) asm volatile("cp.async.wait_all;" ::: "memory");
    reduce_finalize<ASYNC ? kAsync : kSync>(rr, bb, p);
}

// Per-launch staged sweep (one global iteration per launch).
template <bool ASYNC, int WLR, bool EXT = false>
__global__ void __launch_bounds__(WLR > 12 ? 256 : (WLR > 8 ? 512 : 1024), 1) k_block_stage(KP p) {
    if (*(volatile int *)&p.state->stop) return;
    extern __shared__ __align__(128) unsigned char smraw[];
    __shared__ __align__(8) uint64_t bars[2];
    __shared__ long long stage_l[2];
    const int R = p.R, spb = p.spb;
    const StageGeom g = stage_geom(R, spb, p.wmax);
    double *y1 = reinterpret_cast<double *>(smraw + 2 * (size_t)g.bytes);
    const int64_t q = (p.n + R - 1) / R;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t G = gridDim.x;

    // ---- thread 0: subdomain claims and stage issue ----
    long long claims = 0;
    auto claim = [&]() -> long long {
        if (ASYNC && !p.static_claims) return (long long)atomicAdd(&p.state->work, 1ull);
        return (long long)blockIdx.x + (claims++) * G;
    };
    auto issue = [&](long long l, int st, int64_t E0, int64_t E1) {
        stage_l[st] = l;
        if (l >= q) return;
        const int64_t TS = l * (int64_t)R;
        const int nrows = (int)min((int64_t)R, p.n - TS);
        const int nsl = (nrows + kSlice - 1) / kSlice;
        const uint32_t trows = (uint32_t)nrows & ~1u;
        const uint32_t nb_sptr = ((uint32_t)nsl * 8 + 15) & ~15u, nb_sw = ((uint32_t)nsl * 4 + 15) & ~15u;
        const uint32_t ne = (uint32_t)(E1 - E0);
        unsigned char *S = smraw + (size_t)st * g.bytes;
        fence_proxy_async_smem();
        mbar_arrive_expect_tx(&bars[st], ne * 12 + trows * 16 + nb_sptr + nb_sw);
        bulk_g2s(S, p.val + E0, ne * 8, &bars[st]);
        bulk_g2s(S + g.o_col, p.col + E0, ne * 4, &bars[st]);
        if (trows) {
            bulk_g2s(S + g.o_b, p.b + TS, trows * 8, &bars[st]);
            bulk_g2s(S + g.o_x, p.x_in + TS, trows * 8, &bars[st]);
        }
        bulk_g2s(S + g.o_sptr, p.sptr + l * spb, nb_sptr, &bars[st]);
        bulk_g2s(S + g.o_sw, p.sw + l * spb, nb_sw, &bars[st]);
    };
    auto bounds = [&](long long l, int64_t &E0, int64_t &E1) {
        if (l >= q) return;
        const int nsl = (int)((min((int64_t)R, p.n - (int64_t)l * R) + kSlice - 1) / kSlice);
        E0 = p.sptr[l * spb];
        E1 = p.sptr[l * spb + nsl];
    };
    // Thread 0 keeps a three-deep claim pipeline so neither the work-queue atomic nor the range
    // loads are waited on in the iteration that issues them: at iteration i it issues the stage
    // of l_next (bounds loaded during i-1), loads the bounds of l_next2 (claimed during i-1) and
    // claims a new subdomain.
    // Ghost-range entries travel to shared memory by cp.async one iteration before their x
    // ranges are prefetched into L2, two subdomains ahead of the gathers (a3) that read them.
    __shared__ __align__(16) int32_t gsm[2 * kGhostRanges];
    long long l_next = 0, l_next2 = 0;
    int64_t e0n = 0, e1n = 0;
    if (threadIdx.x == 0) {
        mbar_init(&bars[0], 1);
        mbar_init(&bars[1], 1);
        fence_mbar_init();
        const long long l0 = claim();
        int64_t e0 = 0, e1 = 0;
        bounds(l0, e0, e1);
        issue(l0, 0, e0, e1);
        l_next = claim();
        bounds(l_next, e0n, e1n);
        if (p.gr && l_next < q) prefetch_ghost_x(p.x_in, p.gr + 2 * l_next * kGhostRanges, kGhostRanges);
        l_next2 = claim();
        fetch_ghost_entry(p, l_next2, q, gsm);
    }
    __syncthreads();

    constexpr int NP = WLR / 2;
    double rr = 0.0, bb = 0.0;
    for (int i = 0;; ++i) {
        const int st = i & 1;
        const long long l = stage_l[st];
        if (l >= q) break;
        if (threadIdx.x == 0) {  // stream the next subdomain into the other stage
            issue(l_next, st ^ 1, e0n, e1n);
            if (p.gr && l_next2 < q) {
                asm volatile("cp.async.wait_all;" ::: "memory");
                prefetch_ghost_x(p.x_in, gsm, kGhostRanges);
            }
            l_next = l_next2;
            bounds(l_next, e0n, e1n);
            l_next2 = l_next < q ? claim() : q;
            fetch_ghost_entry(p, l_next2, q, gsm);
        }
        unsigned char *S = smraw + (size_t)st * g.bytes;
        const int64_t TS = l * (int64_t)R;
        const int nrows = (int)min((int64_t)R, p.n - TS);
        const int nsl = (nrows + kSlice - 1) / kSlice;
        double *y0 = reinterpret_cast<double *>(S + g.o_x);
        const double *sb = reinterpret_cast<const double *>(S + g.o_b);
        mbar_wait(&bars[st], (i >> 1) & 1);
        if (nrows & 1) {  // odd tail of the last subdomain: not bulk-copied
            if (threadIdx.x == 0) y0[nrows - 1] = ldx<ASYNC>(p.x_in + TS + nrows - 1);
            __syncthreads();
        }
        double lv[WLR];
        uint32_t lc[NP];
        double s = 0.0;
        const int loc = warp * kSlice + lane;
        const bool ok = warp < nsl && loc < nrows;
        const bool fz = EXT && ok && p.frozen && p.frozen[TS + loc];  // N1
#pragma unroll
        for (int e = 0; e < WLR; ++e) lv[e] = 0.0;
#pragma unroll
        for (int e = 0; e < NP; ++e) lc[e] = 0;
        if (ok) {
            const int64_t *ssp = reinterpret_cast<const int64_t *>(S + g.o_sptr);
            const int sw = reinterpret_cast<const int32_t *>(S + g.o_sw)[warp];
            const int wl = sw & 0xffff, wo = sw >> 16;
            const int64_t off = ssp[warp] - ssp[0] + lane;
            const double *sv = reinterpret_cast<const double *>(S) + off;
            const int32_t *sc = reinterpret_cast<const int32_t *>(S + g.o_col) + off;
            const double bi = loc < (nrows & ~1) ? sb[loc] : p.b[TS + loc];
            bb += bi * bi;
            double acc = bi;
            // a3: off-block part, x as it stands (gathers batched)
            for (int e0 = 0; e0 < wo; e0 += 2 * U) {
                double xv[2 * U];
#pragma unroll
                for (int u = 0; u < 2 * U; ++u)
                    if (e0 + u < wo) xv[u] = ldx<ASYNC>(p.x_in + sc[(e0 + u) * kSlice]);
#pragma unroll
                for (int u = 0; u < 2 * U; ++u)
                    if (e0 + u < wo) acc -= sv[(e0 + u) * kSlice] * xv[u];
            }
            s = acc;
#pragma unroll
            for (int e = 0; e < WLR; ++e) {
                if (e < wl) {
                    lv[e] = sv[(wo + e) * kSlice];
                    lc[e >> 1] |= (uint32_t)sc[(wo + e) * kSlice] << (16 * (e & 1));
                }
            }
            // first local sweep; its correction numerator is the residual (a5)
#pragma unroll
            for (int e = 0; e < WLR; ++e) acc -= lv[e] * y0[(lc[e >> 1] >> (16 * (e & 1))) & 0xffff];
            lv[0] = 1.0 / lv[0];
            rr += acc * acc;
            if (EXT) y1[loc] = ext_update(y0[loc], y0[loc] + lv[0] * acc, fz, p.tau);
            else y1[loc] = y0[loc] + lv[0] * acc;
        }
        __syncthreads();
        // a4: sweeps 2..k, direct form, off-block part frozen
        for (int t = 1; t < p.k; ++t) {
            const double *yi = (t & 1) ? y1 : y0;
            double *yo = (t & 1) ? y0 : y1;
            if (ok) {
                double acc = s;
#pragma unroll
                for (int e = 1; e < WLR; ++e) acc -= lv[e] * yi[(lc[e >> 1] >> (16 * (e & 1))) & 0xffff];
                if (EXT) yo[loc] = ext_update(yi[loc], lv[0] * acc, fz, p.tau);
                else yo[loc] = lv[0] * acc;
            }
            __syncthreads();
        }
        // a6: write back
        const double *yk = (p.k & 1) ? y1 : y0;
        for (int r = threadIdx.x; r < nrows; r += blockDim.x) stx<ASYNC>(p.x_out + TS + r, yk[r]);
        __syncthreads();
    }
    reduce_finalize<ASYNC ? kAsync : kSync>(rr, bb, p);
}


// w = m*q + l without a 64-bit integer division (a long dependent chain on the critical warp):
// w < 2^53 is exact in fp64, the quotient estimate is off by at most one and is corrected.
__device__ __forceinline__ void divmod_q(long long w, int64_t q, double inv_q, long long &m, long long &l) {
    m = (long long)((double)w * inv_q);
    l = w - m * q;
    if (l < 0) {
        --m;
        l += q;
    } else if (l >= q) {
        ++m;
        l -= q;
    }
}

// State of the block's thread 0 (claims, stage issue, residual publication). Kept in shared
// memory, not registers: every thread would otherwise reserve the registers it occupies.
struct T0State {
    long long claims, pub_m;
    double pub_ss, pub_bs;
    unsigned int pub_cnt;
};

template <bool ASYNC, int WLR, bool MULTI>
__global__ void __launch_bounds__(WLR > 12 ? 256 : (WLR > 8 ? 512 : 1024), 1) k_block_stage_m(KP p) {
    if (!MULTI && *(volatile int *)&p.state->stop) return;
    if (MULTI && threadIdx.x == 0) stamp_first(p.state);
    extern __shared__ __align__(128) unsigned char smraw[];
    __shared__ __align__(8) uint64_t bars[2];
    __shared__ long long stage_w[2];    // claim held by each stage (>= wend: none)
    __shared__ long long stage_sub[2];  // its subdomain index
    __shared__ long long stage_m[2];    // its global iteration (MULTI)
    __shared__ double sred[2][32];
    __shared__ T0State t0;
    const int R = p.R, spb = p.spb;
    const StageGeom g = stage_geom(R, spb, p.wmax);
    double *y1 = reinterpret_cast<double *>(smraw + 2 * (size_t)g.bytes);
    const int64_t q = (p.n + R - 1) / R;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const long long wend = MULTI ? p.w_end : q;  // claims >= wend end the launch
    const double inv_q = MULTI ? 1.0 / (double)q : 0.0;

    // ---- thread 0 only: subdomain claims and stage issue ----
    auto claim = [&]() -> long long {
        if (MULTI) {  // a stop request moves the queue to w_end, so no flag needs to be polled
            const long long w = (long long)atomicAdd(&p.state->work, 1ull);
            return w < wend ? w : wend;
        }
        if (ASYNC) return (long long)atomicAdd(&p.state->work, 1ull);
        return (long long)blockIdx.x + (t0.claims++) * (long long)gridDim.x;
    };
    auto issue = [&](long long w, int st, int64_t E0, int64_t E1) {
        stage_w[st] = w;
        if (w >= wend) return;
        long long l = w, m = 0;
        if (MULTI) divmod_q(w, q, inv_q, m, l);
        stage_sub[st] = l;
        stage_m[st] = m;
        const int64_t TS = l * (int64_t)R;
        const int nrows = (int)min((int64_t)R, p.n - TS);
        const int nsl = (nrows + kSlice - 1) / kSlice;
        const uint32_t trows = (uint32_t)nrows & ~1u;
        const uint32_t nb_sptr = ((uint32_t)nsl * 8 + 15) & ~15u, nb_sw = ((uint32_t)nsl * 4 + 15) & ~15u;
        const uint32_t ne = (uint32_t)(E1 - E0);
        unsigned char *S = smraw + (size_t)st * g.bytes;
        const bool bulk_x = !(MULTI && p.fresh_xj);
        fence_proxy_async_smem();
        mbar_arrive_expect_tx(&bars[st], ne * 12 + trows * (bulk_x ? 16 : 8) + nb_sptr + nb_sw);
        bulk_g2s(S, p.val + E0, ne * 8, &bars[st]);
        bulk_g2s(S + g.o_col, p.col + E0, ne * 4, &bars[st]);
        if (trows) {
            bulk_g2s(S + g.o_b, p.b + TS, trows * 8, &bars[st]);
            if (bulk_x) bulk_g2s(S + g.o_x, p.x_in + TS, trows * 8, &bars[st]);
        }
        bulk_g2s(S + g.o_sptr, p.sptr + l * spb, nb_sptr, &bars[st]);
        bulk_g2s(S + g.o_sw, p.sw + l * spb, nb_sw, &bars[st]);
    };
    auto bounds = [&](long long w, int64_t &E0, int64_t &E1) {
        if (w >= wend) return;
        long long l = w, m = 0;
        if (MULTI) divmod_q(w, q, inv_q, m, l);
        const int nsl = (int)((min((int64_t)R, p.n - (int64_t)l * R) + kSlice - 1) / kSlice);
        E0 = p.sptr[l * spb];
        E1 = p.sptr[l * spb + nsl];
    };
    // Thread 0 keeps a three-deep claim pipeline so neither the work-queue atomic nor the range
    // loads are waited on in the iteration that issues them: at iteration i it issues the stage
    // of l_next (bounds loaded during i-1), loads the bounds of l_next2 (claimed during i-1) and
    // claims a new subdomain. These four stay in registers: storing a load or atomic result to
    // shared memory would wait for it.
    long long l_next = 0, l_next2 = 0;
    int64_t e0n = 0, e1n = 0;
    if (threadIdx.x == 0) {
        t0.claims = 0;
        t0.pub_m = -1;
        t0.pub_cnt = 0;
        t0.pub_ss = t0.pub_bs = 0.0;
        mbar_init(&bars[0], 1);
        mbar_init(&bars[1], 1);
        fence_mbar_init();
        const long long l0 = claim();
        int64_t e0 = 0, e1 = 0;
        bounds(l0, e0, e1);
        issue(l0, 0, e0, e1);
        l_next = claim();
        bounds(l_next, e0n, e1n);
        l_next2 = claim();
    }
    __syncthreads();

    constexpr int NP = WLR / 2;
    double rr = 0.0, bb = 0.0;
    for (int i = 0;; ++i) {
        const int st = i & 1;
        const long long wcur = stage_w[st];
        if (wcur >= wend) break;
        const long long l = MULTI ? stage_sub[st] : wcur;
        if (MULTI) rr = bb = 0.0;  // per-subdomain residual contribution
        if (threadIdx.x == 0) {  // stream the next subdomain into the other stage
            issue(l_next, st ^ 1, e0n, e1n);
            l_next = l_next2;
            bounds(l_next, e0n, e1n);
            l_next2 = l_next < wend ? claim() : wend;
        }
        unsigned char *S = smraw + (size_t)st * g.bytes;
        const int64_t TS = l * (int64_t)R;
        const int nrows = (int)min((int64_t)R, p.n - TS);
        const int nsl = (nrows + kSlice - 1) / kSlice;
        double *y0 = reinterpret_cast<double *>(S + g.o_x);
        const double *sb = reinterpret_cast<const double *>(S + g.o_b);
        mbar_wait(&bars[st], (i >> 1) & 1);
        if (MULTI && p.fresh_xj) {  // few subdomains per block: x_J must not be prefetched
            for (int r = threadIdx.x; r < nrows; r += blockDim.x) y0[r] = ldx<ASYNC>(p.x_in + TS + r);
            __syncthreads();
        } else if (nrows & 1) {  // odd tail of the last subdomain: not bulk-copied
            if (threadIdx.x == 0) y0[nrows - 1] = ldx<ASYNC>(p.x_in + TS + nrows - 1);
            __syncthreads();
        }
        double lv[WLR];
        uint32_t lc[NP];
        double s = 0.0;
        const int loc = warp * kSlice + lane;
        const bool ok = warp < nsl && loc < nrows;
#pragma unroll
        for (int e = 0; e < WLR; ++e) lv[e] = 0.0;
#pragma unroll
        for (int e = 0; e < NP; ++e) lc[e] = 0;
        if (ok) {
            const int64_t *ssp = reinterpret_cast<const int64_t *>(S + g.o_sptr);
            const int sw = reinterpret_cast<const int32_t *>(S + g.o_sw)[warp];
            const int wl = sw & 0xffff, wo = sw >> 16;
            const int64_t off = ssp[warp] - ssp[0] + lane;
            const double *sv = reinterpret_cast<const double *>(S) + off;
            const int32_t *sc = reinterpret_cast<const int32_t *>(S + g.o_col) + off;
            const double bi = loc < (nrows & ~1) ? sb[loc] : p.b[TS + loc];
            bb += bi * bi;
            double acc = bi;
            // a3: off-block part, x as it stands (gathers batched)
            for (int e0 = 0; e0 < wo; e0 += 2 * U) {
                double xv[2 * U];
#pragma unroll
                for (int u = 0; u < 2 * U; ++u)
                    if (e0 + u < wo) xv[u] = ldx<ASYNC>(p.x_in + sc[(e0 + u) * kSlice]);
#pragma unroll
                for (int u = 0; u < 2 * U; ++u)
                    if (e0 + u < wo) acc -= sv[(e0 + u) * kSlice] * xv[u];
            }
            s = acc;
#pragma unroll
            for (int e = 0; e < WLR; ++e) {
                if (e < wl) {
                    lv[e] = sv[(wo + e) * kSlice];
                    lc[e >> 1] |= (uint32_t)sc[(wo + e) * kSlice] << (16 * (e & 1));
                }
            }
            // first local sweep; its correction numerator is the residual (a5)
#pragma unroll
            for (int e = 0; e < WLR; ++e) acc -= lv[e] * y0[(lc[e >> 1] >> (16 * (e & 1))) & 0xffff];
            lv[0] = 1.0 / lv[0];
            rr += acc * acc;
            y1[loc] = y0[loc] + lv[0] * acc;
        }
        __syncthreads();
        // a4: sweeps 2..k, direct form, off-block part frozen
        for (int t = 1; t < p.k; ++t) {
            const double *yi = (t & 1) ? y1 : y0;
            double *yo = (t & 1) ? y0 : y1;
            if (ok) {
                double acc = s;
#pragma unroll
                for (int e = 1; e < WLR; ++e) acc -= lv[e] * yi[(lc[e >> 1] >> (16 * (e & 1))) & 0xffff];
                yo[loc] = lv[0] * acc;
            }
            __syncthreads();
        }
        // a6: write back
        const double *yk = (p.k & 1) ? y1 : y0;
        for (int r = threadIdx.x; r < nrows; r += blockDim.x) stx<ASYNC>(p.x_out + TS + r, yk[r]);
        if (MULTI) {
            const double wr = warp_sum(rr), wb = warp_sum(bb);
            if (lane == 0) {
                sred[0][warp] = wr;
                sred[1][warp] = wb;
            }
        }
        __syncthreads();
        if (MULTI && warp == 0) {
            const int W = blockDim.x >> 5;
            const double a0 = warp_sum(lane < W ? sred[0][lane] : 0.0);
            const double a1 = warp_sum(lane < W ? sred[1][lane] : 0.0);
            if (lane == 0) {
                const long long m = stage_m[st];
                if (m != t0.pub_m && t0.pub_cnt) {
                    iteration_publish(p, t0.pub_m, t0.pub_cnt, t0.pub_ss, t0.pub_bs, q);
                    t0.pub_cnt = 0;
                    t0.pub_ss = t0.pub_bs = 0.0;
                }
                t0.pub_m = m;
                ++t0.pub_cnt;
                t0.pub_ss += a0;
                t0.pub_bs += a1;
            }
        }
    }
    if (MULTI && threadIdx.x == 0 && t0.pub_cnt) iteration_publish(p, t0.pub_m, t0.pub_cnt, t0.pub_ss, t0.pub_bs, q);
    if (MULTI && threadIdx.x == 0) stamp_last(p.state);
    if (!MULTI) reduce_finalize<ASYNC ? kAsync : kSync>(rr, bb, p);
}

// The stopping rule of iteration m from its sum of r_i^2 (lazy / tagged publication).
__device__ __forceinline__ void lazy_rule(DevState *S, long long m, double ss, double bn, double *hist) {
    const double rel = bn != 0.0 ? sqrt(ss) / bn : 0.0;
    atomicMax(&S->iters_done, m + 1);
    S->bnorm = bn;
    S->last_rel = rel;
    if (hist) hist[m] = rel;
    bool stop = false;
    if (bn == 0.0) {
        S->diverged = 2;
        stop = true;
    } else if (!isfinite(rel) || rel > 1e30) {
        S->diverged = 1;
        stop = true;
    } else if (rel <= S->tol) {
        // evaluations may complete out of order: the first iteration that met tol wins
        atomicMin(reinterpret_cast<unsigned long long *>(&S->stop_iter), (unsigned long long)(m + 1));
        stop = true;
    }
    if (stop) atomicExch(&S->stop, 1);
}

// k_block_resident<.., LAZY>: warp 0 of block m % q evaluates iteration m once all q partials are
// in ring[m % kSlots] (LAZY = 1: thread 0 polls the slot's counter with relaxed loads, then an
// acquire fence before the CTA barrier that hands the evaluation to the warp): fixed-order sums
// over the blocks (lane-strided, then the shuffle tree), the stopping rule, iters_done, and the
// slot's counter reset for iteration m + kSlots. TAGGED (LAZY = 2; this function only on the
// lead-wait path, the regular evaluation sums the words warp 0 already holds): the ring words
// carry the iteration and launch epoch in their 12 low mantissa bits (the partial keeps 40 bits of
// mantissa, a relative 1e-12 of the estimate); they are summed with the tag cleared, and ||b|| is
// the one the x^(0) residual stored before the launch.
template <bool TAGGED>
__device__ __noinline__ void lazy_evaluate(const KP &p, long long m, int64_t q, int lane, double bnorm0) {
    DevState *S = p.state;
    const int slot = (int)(m % kSlots);
    const double *row = p.ring + (int64_t)slot * q;
    double ss = 0.0, bsq = 0.0;
    for (int64_t c = lane; c < q; c += kSlice) {
        if (TAGGED) {
            unsigned long long w;
            asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(w) : "l"(row + c) : "memory");
            ss += __longlong_as_double((long long)(w & ~0xFFFull));
        } else {
            ss += __ldcg(row + c);
            bsq += __ldcg(p.bsum_arr + c);
        }
    }
    ss = warp_sum(ss);
    if (!TAGGED) bsq = warp_sum(bsq);
    if (lane != 0) return;
    if (!TAGGED) S->done[slot] = 0u;
    lazy_rule(S, m, ss, TAGGED ? bnorm0 : sqrt(bsq), p.hist);
}

// Phase timing of k_block_resident's thread 0 (a profiling build only: -DBAR_PROFILE_RESIDENT):
// clock64 deltas between the marks, summed over the launch, added per block into g_res_prof.
#ifdef BAR_PROFILE_RESIDENT
__device__ unsigned long long g_res_prof[8];
#define BAR_PROF_DECL long long prof_t[6] = {0, 0, 0, 0, 0, 0}, prof_last = clock64();
#define BAR_PROF_MARK(i)                            \
    if (threadIdx.x == 0) {                         \
        const long long now = clock64();            \
        prof_t[i] += now - prof_last;               \
        prof_last = now;                            \
    }
#define BAR_PROF_FLUSH                                                                  \
    if (threadIdx.x == 0)                                                               \
        for (int i = 0; i < 6; ++i) atomicAdd(&g_res_prof[i], (unsigned long long)prof_t[i]);
#else
#define BAR_PROF_DECL
#define BAR_PROF_MARK(i)
#define BAR_PROF_FLUSH
#endif

// k_block_resident: the fully asynchronous solve for systems whose subdomains all fit on the
// device at once (q <= co-resident blocks; C1-C3). Block c OWNS subdomain c for the whole launch,
// the paper's picture taken literally: one thread block per subdomain, iterating with no
// synchronisation with the other blocks (Alg. 1, eq. 3). Everything that does not change between
// iterations is loaded ONCE: the block's local entries and 1/a_ii in registers, its off-block
// entries in shared memory, b_i in a register, and x_J stays in shared memory (only this block
// ever writes it). A global iteration is then: gather the off-block x as it stands (relaxed
// loads), k local sweeps, relaxed write-back of x_J, residual publication for iteration m
// (iteration_publish: the block completing iteration m evaluates rel_res_m and stops the solve).
// Blocks stop on the stop flag (read one iteration ahead, so its latency is hidden) or after
// max_global_iters sweeps; state->res_sweeps counts the sweeps for the host's accounting. A block
// may run at most p.lead (<= 48) iterations ahead of the last completed one (the 64 residual
// slots; P:109's bounded delay), waiting otherwise. The kernel relies on all q blocks being
// resident at once; if they are not (other work on the device holds SMs), a waiting block
// times out after ~2 ms, raises state->aborted and the stop flag, every block exits, and the
// host continues the solve from the current iterate with per-launch kernels (R12).
// Words of a tagged ring row each lane of warp 0 holds (k_block_resident<.., 2>): 8 (q <= 256) in
// the 256 / 512-thread variants, 2 (q <= 64) in the 1024-thread ones (64 registers).
__host__ __device__ constexpr int resident_pend(int wlr) { return wlr > 8 ? 8 : 2; }

// LAZY: 0 blocking publication (iteration_publish), 1 ring + counter (release reduction),
// 2 tagged ring words (q <= 32 resident_pend): a block's partial and its iteration tag in ONE relaxed 64-bit
// store, so publishing needs no release fence (which waited for every write of the block,
// x included, to reach L2: ~1 K cycles per iteration); warp 0 of the evaluating block loads the
// q words one iteration ahead (<= 8 per lane) and votes on their tags.
template <int WLR, int LAZY = 0>
__global__ void __launch_bounds__(WLR > 12 ? 256 : (WLR > 8 ? 512 : 1024), 1) k_block_resident(KP p) {
    extern __shared__ __align__(128) unsigned char smraw[];
    __shared__ double sred[2][32];
    __shared__ int go;
    __shared__ long long eval_m;  // LAZY: iteration warp 0 evaluates in this pass (-1: none)
    if (threadIdx.x == 0) stamp_first(p.state);
    const int R = p.R, spb = p.spb;
    const int64_t q = (p.n + R - 1) / R;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t l = blockIdx.x, TS = l * (int64_t)R;
    const int nrows = (int)min((int64_t)R, p.n - TS);
    const int nsl = (nrows + kSlice - 1) / kSlice;
    const int loc = warp * kSlice + lane;
    const bool ok = warp < nsl && loc < nrows;
    double *const ybase = reinterpret_cast<double *>(smraw);  // y buffer c at ybase + c R
    auto ybuf = [&](int c) { return ybase + (c ? R : 0); };
    // off-block entries of the subdomain: values then columns, slice-major as in the layout
    double *ov = reinterpret_cast<double *>(smraw) + 2 * R;
    const int64_t E0 = p.sptr[l * spb];
    const int ocap = p.wmax * spb * kSlice;
    int32_t *oc = reinterpret_cast<int32_t *>(ov + ocap);
    constexpr int NP = WLR / 2;
    double lv[WLR];
    uint32_t lc[NP];
    double bi = 0.0;
    int wo = 0;
    uint32_t ooff = 0;
#pragma unroll
    for (int e = 0; e < WLR; ++e) lv[e] = 0.0;
#pragma unroll
    for (int e = 0; e < NP; ++e) lc[e] = 0;
    if (ok) {  // once per launch: matrix rows into registers / shared memory, x_J and b_i
        const int64_t so = p.sptr[l * spb + warp];
        const int sw = p.sw[l * spb + warp];
        const int wl = sw & 0xffff;
        wo = sw >> 16;
        ooff = (uint32_t)(so - E0) + lane;
        for (int e = 0; e < wo; ++e) {
            ov[ooff + e * kSlice] = p.val[so + e * kSlice + lane];
            oc[ooff + e * kSlice] = p.col[so + e * kSlice + lane];
        }
#pragma unroll
        for (int e = 0; e < WLR; ++e) {
            if (e < wl) {
                lv[e] = p.val[so + (int64_t)(wo + e) * kSlice + lane];
                lc[e >> 1] |= (uint32_t)p.col[so + (int64_t)(wo + e) * kSlice + lane] << (16 * (e & 1));
            }
        }
        bi = p.b[TS + loc];
        ybase[loc] = ldx<true>(p.x_in + TS + loc);
    }
    const double dinv = ok ? 1.0 / lv[0] : 0.0;  // lv[0] = a_ii stays for the correction form
    // sum of b_i^2 of the block (the same every iteration)
    double bsum;
    {
        const double wb = warp_sum(bi * bi);
        if (lane == 0) sred[1][warp] = wb;
        __syncthreads();
        const int W = blockDim.x >> 5;
        bsum = 0.0;
        for (int w = 0; w < W; ++w) bsum += sred[1][w];
    }
    // LAZY publication: block c stores its partial of iteration m into ring[m % kSlots][c] and
    // bumps done[m % kSlots] with a release reduction (no returned value, nothing to wait for);
    // iteration m is evaluated by block m % q once it sees all q contributions (a relaxed load
    // issued one iteration ahead; acquire fence when complete): fixed-order sum of the ring row
    // and of the blocks' sum b_i^2, then the stopping rule as in iteration_publish (lazy_evaluate)
    long long next_eval = p.m0 + (((long long)blockIdx.x - p.m0) % q + q) % q;  // first m >= m0 with m % q == c
    unsigned int dv_ld = 0;
    if (LAZY && threadIdx.x == 0)
        asm volatile("st.relaxed.gpu.global.f64 [%0], %1;" ::"l"(p.bsum_arr + blockIdx.x), "d"(bsum) : "memory");
    // LAZY == 2: the launch's epoch, ||b|| from the x^(0) residual, the words of slot next_eval
    const unsigned int ep = LAZY == 2 ? *(volatile unsigned int *)&p.state->epoch : 0u;
    const double bnorm0 = LAZY == 2 ? *(volatile double *)&p.state->bnorm : 0.0;
    auto tag_of = [&](long long mm) -> unsigned long long {
        return ((unsigned long long)(ep & 0xFu) << 8) | ((unsigned long long)mm & 0xFFull);
    };
    constexpr int PEND = resident_pend(WLR);  // words per lane: q <= 32 PEND (registers)
    unsigned long long pend[PEND];
#pragma unroll
    for (int j = 0; j < PEND; ++j) pend[j] = ~0ull;  // no tag matches
    // thread 0's slow path (lead wait): are all q words of iteration mm's slot tagged mm?
    auto tags_ready = [&](long long mm) -> bool {  // (batches of 8 loads in flight)
        const unsigned long long *row = reinterpret_cast<const unsigned long long *>(p.ring) + (mm % kSlots) * q;
        BAR_CHECK(mm >= 0, "tags_ready iteration");
        bool all = true;
        for (int64_t c0 = 0; c0 < q && all; c0 += 8) {
            unsigned long long w[8];
#pragma unroll
            for (int u = 0; u < 8; ++u)
                w[u] = c0 + u < q ? ld_relaxed_u64(row + c0 + u) : tag_of(mm);
#pragma unroll
            for (int u = 0; u < 8; ++u) all = all && (w[u] & 0xFFFull) == tag_of(mm);
        }
        return all;
    };
    int cur = 0;
    // Gathers one iteration ahead (the 256-thread variants have the registers): a row's off-block
    // x values for iteration m + 1 are loaded right after its write-back of iteration m — x "as
    // it stands" a few hundred cycles earlier than at the next sweep, which eq. 3 allows — so their
    // L2 latency overlaps the residual publication and the next iteration's start instead of
    // opening the sweep
    constexpr int GPRE = WLR > 12 ? 16 : 0;
    const bool pre = GPRE > 0 && p.gather_ahead && wo <= GPRE;
    double xg[GPRE > 0 ? GPRE : 1];
    auto issue_gathers = [&]() {
#pragma unroll
        for (int e = 0; e < GPRE; ++e)
            if (e < wo) xg[e] = ldx<true>(p.x_in + oc[ooff + e * kSlice]);
    };
    if (pre && ok) issue_gathers();
    // thread 0: the stop flag, loaded one iteration ahead of its use (k_init_check may have raised
    // it before the launch: x^(0) already meets tol)
    int stop_seen = threadIdx.x == 0 ? *(volatile int *)&p.state->stop : 0, stop_ld = 0;
    long long done_ld = p.m0;  // thread 0: iters_done, loaded one iteration ahead of its use
    unsigned long long sweeps = 0;
    BAR_PROF_DECL
    for (long long m = p.m0;;) {
        BAR_PROF_MARK(0)
        if (threadIdx.x == 0) {
            // every block sweeps exactly max_global_iters = w_end / q times unless the solve stops
            int g = m < p.w_end / q && !stop_seen;
            // LAZY: this block's pending evaluation, if all q partials of that iteration are in
            // (dv_ld / the tagged words: loaded one iteration ahead); evaluated by warp 0 after the
            // barrier below
            if (LAZY) {
                eval_m = -1;
                if (LAZY == 1 && next_eval < m && dv_ld == (unsigned int)q) {
                    if (LAZY == 1) asm volatile("fence.acq_rel.gpu;" ::: "memory");
                    eval_m = next_eval;
                    dv_ld = 0;
                }
            }
            // bounded lead over the last completed iteration (p.lead sweeps; residual slots are
            // reused mod 64). The lead is checked against iters_done as loaded one iteration ago
            // and only re-read (waited on) when exceeded. The wait is itself bounded (~2 ms of
            // %globaltimer): a lagging block that long behind is not resident, so the launch gives
            // up (aborted + stop) instead of waiting on work that cannot run. LAZY: the iteration
            // the others wait for may be the one this block evaluates — then stop waiting, let
            // warp 0 evaluate it, and come back (go = 2) before sweeping
            if (g && m - done_ld > p.lead) {
                if (LAZY && eval_m >= 0) {
                    g = 2;
                } else {
                    const unsigned long long t0c = globaltimer_ns();
                    while (g && m - *(volatile long long *)&p.state->iters_done > p.lead) {
                        if (*(volatile int *)&p.state->stop) g = 0;
                        else if (globaltimer_ns() - t0c > 2000000ull) {
                            atomicExch(&p.state->aborted, 1);
                            atomicExch(&p.state->stop, 1);
                            g = 0;
                        } else if (LAZY && next_eval < m &&
                                   (LAZY == 2 ? tags_ready(next_eval)
                                              : *(volatile unsigned int *)&p.state->done[next_eval % kSlots] ==
                                                    (unsigned int)q)) {
                            if (LAZY == 1) asm volatile("fence.acq_rel.gpu;" ::: "memory");
                            eval_m = next_eval;
                            g = 2;
                            break;
                        }
                    }
                }
            }
            go = g;
        }
        __syncthreads();
        if (LAZY && eval_m >= 0) {  // every thread advances next_eval (warp 0 votes with it)
            if (warp == 0) lazy_evaluate<LAZY == 2>(p, eval_m, q, lane, bnorm0);
            next_eval = eval_m + q;
        }
        if (!go) break;
        // LAZY == 2: warp 0 loads the words of iteration next_eval (already swept and published
        // by this block) now and votes on them at the end of this iteration, so the other blocks
        // have had this whole iteration to publish theirs
        const bool pend_issued = LAZY == 2 && go == 1 && next_eval < m;
        BAR_CHECK(!pend_issued || (next_eval >= 0 && q <= 32 * PEND), "tagged pending words");
        if (LAZY == 2 && warp == 0 && pend_issued) {
            const unsigned long long *row =
                reinterpret_cast<const unsigned long long *>(p.ring) + (next_eval % kSlots) * q;
#pragma unroll
            for (int j = 0; j < PEND; ++j)
                if (lane + 32 * j < q)
                    asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(pend[j]) : "l"(row + lane + 32 * j) : "memory");
        }
        if (LAZY && go == 2) {  // evaluated for the waiting blocks; re-check the lead
            __syncthreads();
            continue;
        }
        BAR_PROF_MARK(1)
        ++sweeps;
        if (threadIdx.x == 0) {  // issued now, consumed at the next iteration's start
            asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(stop_ld) : "l"(&p.state->stop));
            asm volatile("ld.relaxed.gpu.global.s64 %0, [%1];" : "=l"(done_ld) : "l"(&p.state->iters_done));
        }
        const double *y0 = ybuf(cur);
        double *y1 = ybuf(cur ^ 1);
        double s = bi, rr = 0.0;
        if (ok && pre) {  // a3 from the values gathered one iteration ahead
#pragma unroll
            for (int e = 0; e < GPRE; ++e)
                if (e < wo) s -= ov[ooff + e * kSlice] * xg[e];
        } else if (ok) {
            // a3: off-block part, x as it stands
            for (int e0 = 0; e0 < wo; e0 += 2 * U) {
                double xv[2 * U];
#pragma unroll
                for (int u = 0; u < 2 * U; ++u)
                    if (e0 + u < wo) xv[u] = ldx<true>(p.x_in + oc[ooff + (e0 + u) * kSlice]);
#pragma unroll
                for (int u = 0; u < 2 * U; ++u)
                    if (e0 + u < wo) s -= ov[ooff + (e0 + u) * kSlice] * xv[u];
            }
        }
        if (ok) {
            // first local sweep in the correction form: its numerator is r_i (a5)
            double acc = s;
#pragma unroll
            for (int e = 0; e < WLR; ++e) acc -= lv[e] * y0[(lc[e >> 1] >> (16 * (e & 1))) & 0xffff];
            rr = acc * acc;
            y1[loc] = y0[loc] + dinv * acc;
        }
        __syncthreads();
        BAR_PROF_MARK(2)
        for (int t = 1; t < p.k; ++t) {  // a4: sweeps 2..k, direct form, off-block part frozen
            const double *yi = ybuf(cur ^ (t & 1));
            double *yo = ybuf(cur ^ ((t + 1) & 1));
            if (ok) {
                double acc = s;
#pragma unroll
                for (int e = 1; e < WLR; ++e) acc -= lv[e] * yi[(lc[e >> 1] >> (16 * (e & 1))) & 0xffff];
                yo[loc] = dinv * acc;
            }
            __syncthreads();
        }
        BAR_PROF_MARK(3)
        cur ^= p.k & 1;
        if (ok) stx<true>(p.x_out + TS + loc, ybuf(cur)[loc]);  // a6
        if (pre && ok) issue_gathers();  // for the next iteration
        const double wr = warp_sum(rr);
        if (lane == 0) sred[0][warp] = wr;
        __syncthreads();
        BAR_PROF_MARK(4)
        if (LAZY == 2 && warp == 0 && pend_issued) {  // evaluate iteration next_eval if all q words are in
            bool r = true;
#pragma unroll
            for (int j = 0; j < PEND; ++j)
                if (lane + 32 * j < q) r = r && (pend[j] & 0xFFFull) == tag_of(next_eval);
            if (__all_sync(0xffffffffu, r)) {
                double ss = 0.0;
#pragma unroll
                for (int j = 0; j < PEND; ++j)
                    if (lane + 32 * j < q) ss += __longlong_as_double((long long)(pend[j] & ~0xFFFull));
                ss = warp_sum(ss);
                if (lane == 0) lazy_rule(p.state, next_eval, ss, bnorm0, p.hist);
                next_eval += q;  // warp 0 only: the other warps never read it in this variant
            }
        }
        if (threadIdx.x == 0) {
            const int W = blockDim.x >> 5;
            double a0 = 0.0;
            for (int w = 0; w < W; ++w) a0 += sred[0][w];
            if (LAZY == 2) {
                const int slot = (int)(m % kSlots);
                const unsigned long long w = ((unsigned long long)__double_as_longlong(a0) & ~0xFFFull) | tag_of(m);
                asm volatile("st.relaxed.gpu.global.b64 [%0], %1;" ::"l"(p.ring + (int64_t)slot * q + blockIdx.x),
                             "l"(w)
                             : "memory");
            } else if (LAZY) {
                const int slot = (int)(m % kSlots);
                asm volatile("st.relaxed.gpu.global.f64 [%0], %1;" ::"l"(p.ring + (int64_t)slot * q + blockIdx.x),
                             "d"(a0)
                             : "memory");
                asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(&p.state->done[slot]) : "memory");
                if (next_eval <= m)  // consumed at the next iteration's start
                    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];"
                                 : "=r"(dv_ld)
                                 : "l"(&p.state->done[next_eval % kSlots]));
            } else {
                iteration_publish(p, m, 1u, a0, bsum, q);
            }
            stop_seen = stop_ld;
        }
        BAR_PROF_MARK(5)
        ++m;
    }
    if (threadIdx.x == 0) atomicAdd(&p.state->res_sweeps, sweeps);
    // The exact residual ||b - A x||_2 of the iterate the solve returns (a5, the confirming
    // residual of a7), fused: once every block has stopped sweeping (a grid barrier — all q blocks
    // are co-resident; bounded by ~2 ms of %globaltimer like the lead wait, after which the host
    // runs the residual kernel instead), each block forms r_i = b_i - sum_j a_ij x_j for its rows
    // from the matrix entries it already holds (off-block x as written, x_J from shared memory),
    // and the last block sums the q partials in block order (own ticket and ring row 0, so a
    // partial pass leaves the residual kernel's state untouched; ring row kSlots).
    if (LAZY && p.fuse_residual) {
        __shared__ int fuse_go;
        if (threadIdx.x == 0) {
            asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(&p.state->fuse_arrive) : "memory");
            const unsigned long long t0c = globaltimer_ns();
            int okb = 1;
            for (;;) {
                unsigned int a;
                asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(a) : "l"(&p.state->fuse_arrive) : "memory");
                if (a >= (unsigned int)q) break;
                if (globaltimer_ns() - t0c > 2000000ull) {
                    okb = 0;
                    break;
                }
            }
            fuse_go = okb && !*(volatile int *)&p.state->aborted;
        }
        __syncthreads();
        if (fuse_go) {
            double r2 = 0.0;
            if (ok) {
                double s = bi;
                for (int e0 = 0; e0 < wo; e0 += 2 * U) {
                    double xv[2 * U];
#pragma unroll
                    for (int u = 0; u < 2 * U; ++u)
                        if (e0 + u < wo) xv[u] = ldx<true>(p.x_in + oc[ooff + (e0 + u) * kSlice]);
#pragma unroll
                    for (int u = 0; u < 2 * U; ++u)
                        if (e0 + u < wo) s -= ov[ooff + (e0 + u) * kSlice] * xv[u];
                }
                const double *yf = ybuf(cur);
#pragma unroll
                for (int e = 0; e < WLR; ++e) s -= lv[e] * yf[(lc[e >> 1] >> (16 * (e & 1))) & 0xffff];
                r2 = s * s;
            }
            const double wr = warp_sum(r2);
            if (lane == 0) sred[0][warp] = wr;
            __syncthreads();
            __shared__ bool fuse_last;
            if (threadIdx.x == 0) {
                const int W = blockDim.x >> 5;
                double a0 = 0.0;
                for (int w = 0; w < W; ++w) a0 += sred[0][w];
                asm volatile("st.relaxed.gpu.global.f64 [%0], %1;" ::"l"(p.ring + kSlots * q + blockIdx.x), "d"(a0)
                             : "memory");
                unsigned int tk;
                asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(tk) : "l"(&p.state->fuse_ticket) : "memory");
                fuse_last = tk == (unsigned int)q - 1;
            }
            __syncthreads();
            if (fuse_last) {
                double s0 = 0.0, s1 = 0.0;
                for (int64_t i = threadIdx.x; i < q; i += blockDim.x) {
                    double v0, v1;
                    asm volatile("ld.relaxed.gpu.global.f64 %0, [%1];" : "=d"(v0) : "l"(p.ring + kSlots * q + i) : "memory");
                    asm volatile("ld.relaxed.gpu.global.f64 %0, [%1];" : "=d"(v1) : "l"(p.bsum_arr + i) : "memory");
                    s0 += v0;
                    s1 += v1;
                }
                s0 = warp_sum(s0);
                s1 = warp_sum(s1);
                __syncthreads();
                if (lane == 0) {
                    sred[0][warp] = s0;
                    sred[1][warp] = s1;
                }
                __syncthreads();
                if (threadIdx.x == 0) {
                    const int W = blockDim.x >> 5;
                    double ss = 0.0, bsq = 0.0;
                    for (int w = 0; w < W; ++w) {
                        ss += sred[0][w];
                        bsq += sred[1][w];
                    }
                    apply_stop_rule(p.state, ss, bsq, true, nullptr);
                    p.state->exact_fused = 1;
                }
            }
        }
    }
    if (threadIdx.x == 0) stamp_last(p.state);
    BAR_PROF_FLUSH
}

// Jacobi (eq. 2) and the standalone residual, persistent warps: warp g handles slices
// g, g + G, g + 2G, ... (G = warps in the grid) and keeps the next slice's bulk copy in flight
// (two slice buffers per warp) while computing the current one.
template <bool RESIDUAL_ONLY>
__global__ void __launch_bounds__(256, 4) k_rowwise_tma(KP p) {
    if (!RESIDUAL_ONLY && *(volatile int *)&p.state->stop) return;
    extern __shared__ __align__(128) unsigned char smraw[];
    __shared__ __align__(8) uint64_t bars[8][2];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int wmax = p.wmax;
    const uint32_t bb_bytes = slice_buf_bytes(wmax);
    unsigned char *buf[2] = {smraw + (size_t)(2 * warp) * bb_bytes, smraw + (size_t)(2 * warp + 1) * bb_bytes};
    const int64_t G = (int64_t)gridDim.x * 8;
    int64_t sl = (int64_t)blockIdx.x * 8 + warp;
    if (lane == 0) {
        mbar_init(&bars[warp][0], 1);
        mbar_init(&bars[warp][1], 1);
        fence_mbar_init();
        if (sl < p.nslices) {
            const int w = p.sw[sl];
            issue_slice(p, sl, (w & 0xffff) + (w >> 16), buf[0], &bars[warp][0], wmax);
        }
    }
    __syncwarp();
    double rr = 0.0, bb = 0.0;
    for (int i = 0; sl < p.nslices; ++i, sl += G) {
        const int st = i & 1;
        const int64_t nx = sl + G;
        if (lane == 0 && nx < p.nslices) {
            fence_proxy_async_smem();
            const int w = p.sw[nx];
            issue_slice(p, nx, (w & 0xffff) + (w >> 16), buf[st ^ 1], &bars[warp][st ^ 1], wmax);
        }
        const int sw = p.sw[sl];
        const int wl = sw & 0xffff, wo = sw >> 16, w = wl + wo;
        const int64_t l = sl / p.spb;
        const int64_t TS = l * (int64_t)p.R;
        const int64_t loc = (sl - l * p.spb) * kSlice + lane;
        const int64_t row = TS + loc;
        mbar_wait(&bars[warp][st], (i >> 1) & 1);
        if (loc < p.R && row < p.n) {
            const double *sv = reinterpret_cast<const double *>(buf[st]) + lane;
            const int32_t *sc = reinterpret_cast<const int32_t *>(buf[st] + (size_t)wmax * kSlice * sizeof(double)) + lane;
            const double bi = p.b[row];
            bb += bi * bi;
            double acc = bi, dinv = 0.0;
            for (int e0 = 0; e0 < w; e0 += 2 * U) {
                double xv[2 * U];
#pragma unroll
                for (int u = 0; u < 2 * U; ++u) {
                    const int e = e0 + u;
                    if (e < w) xv[u] = __ldg(p.x_in + (e < wo ? 0 : TS) + sc[e * kSlice]);
                }
#pragma unroll
                for (int u = 0; u < 2 * U; ++u) {
                    const int e = e0 + u;
                    if (e < w) {
                        const double a = sv[e * kSlice];
                        if (e == wo) dinv = 1.0 / a;
                        acc -= a * xv[u];
                    }
                }
            }
            rr += acc * acc;
            if (!RESIDUAL_ONLY) {
                const double xi = __ldg(p.x_in + row);
                p.x_out[row] = ext_update(xi, xi + dinv * acc, p.frozen && p.frozen[row], p.tau);
            }
        }
        __syncwarp();
    }
    reduce_finalize<RESIDUAL_ONLY ? kResidual : kSync>(rr, bb, p);
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
            double s, res, dinv;
            row_pass<false, false, false>(p.val + base, p.col + base, wo, wo + wl, p.x_in, p.x_in + TS, bi, s, res,
                                          dinv, nullptr, nullptr, 0);
            rr = res * res;
            if (!RESIDUAL_ONLY) {
                const double xi = __ldg(p.x_in + row);
                p.x_out[row] = ext_update(xi, xi + dinv * res, p.frozen && p.frozen[row], p.tau);
            }
        }
    }
    reduce_finalize<RESIDUAL_ONLY ? kResidual : kSync>(rr, bb, p);
}

__global__ void k_init_state(DevState *S, double tol) {
    S->counter = 0;
    S->stop = 0;
    S->diverged = 0;
    S->aborted = 0;
    S->iter = 0;
    S->conv_iter = -1;
    S->tol = tol;
    S->last_rel = -1.0;
    S->exact_rel = -1.0;
    S->work = 0;
    S->iters_done = 0;
    S->stop_iter = -1;
    S->work_resume = 0;
    S->res_sweeps = 0;
    S->t_first = ~0ull;
    S->t_last = 0;
    S->fuse_arrive = 0;
    S->fuse_ticket = 0;
    S->exact_fused = 0;
    S->epoch += 1;
    for (int i = 0; i < kSlots; ++i) {
        S->done[i] = 0;
        S->ss[i] = 0.0;
        S->bs[i] = 0.0;
    }
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
    p.tau = 1.0;
    p.frozen = nullptr;
    // measured on B200 (round 1, tools/kernel_ab.py): the L2 prefetch of the gather ranges pays
    // for large subdomains (C5, R = 1024: 2.78 vs 2.87 ms per sync-block-(5) launch) and costs
    // for small ones (C4, R = 128: 0.45 vs 0.41 ms), whose ranges are 1 KB
    const int gp = L.tune.ghost_prefetch;
    p.gr = (gp ? gp > 0 : L.R >= 512) ? L.gr : nullptr;
    p.grid_cap = L.tune.grid_cap > 0 ? L.tune.grid_cap : 0;
    p.slab_ahead = L.tune.slab_prefetch > 0 ? 1 : 0;
    return p;
}

// Launch caches per (kernel, device): the dynamic shared-memory attribute (cudaFuncSetAttribute
// applies to the current device only) and the occupancy query results. Guarded by g_launch_mu.
struct FnState {
    size_t attr = 0, c_smem = 0;
    int c_threads = 0, occ = 0;
};
std::map<std::pair<const void *, int>, FnState> g_fn;

FnState &fn_state(const void *fn) {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) {
        cudaGetLastError();
        dev = 0;
    }
    return g_fn[{fn, dev}];
}

template <class F>
cudaError_t ensure_smem(F *fn, size_t smem) {
    FnState &s = fn_state(reinterpret_cast<const void *>(fn));
    if (smem > s.attr) {
        cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        s.attr = smem;
    }
    return cudaSuccess;
}

// Co-resident blocks of fn per SM at (threads, smem); 0 if the query fails or nothing fits.
template <class F>
int occupancy(F *fn, int threads, size_t smem) {
    FnState &s = fn_state(reinterpret_cast<const void *>(fn));
    if (s.c_smem != smem || s.c_threads != threads) {
        int o = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, fn, threads, smem) != cudaSuccess) {
            cudaGetLastError();
            o = 0;
        }
        s.occ = o;
        s.c_smem = smem;
        s.c_threads = threads;
    }
    return s.occ;
}

template <bool ASYNC, bool STAGE>
cudaError_t launch_block_t(const KP &p, int threads, size_t smem, unsigned grid, cudaStream_t st) {
    std::lock_guard<std::recursive_mutex> lk(g_launch_mu);
    cudaError_t e = ensure_smem(k_block<ASYNC, STAGE>, smem);
    if (e != cudaSuccess) return e;
    k_block<ASYNC, STAGE><<<grid, threads, smem, st>>>(p);
    return cudaGetLastError();
}

// Block geometry: one 32-row slice per warp and pass; local entries staged in shared memory
// when they fit (otherwise re-read through L1/L2 in every sweep).
template <bool ASYNC, int WLR, int RPT>
cudaError_t launch_reg_t(const KP &p, const Layout &L, cudaStream_t st) {
    const int W = (L.spb + RPT - 1) / RPT;
    k_reg<ASYNC, WLR, RPT><<<(unsigned)L.q, W * kSlice, 2 * (size_t)L.R * sizeof(double), st>>>(p);
    return cudaGetLastError();
}

template <bool ASYNC, int RPT>
cudaError_t launch_reg_w(const KP &p, const Layout &L, cudaStream_t st) {
    if (L.max_wl <= 4) return launch_reg_t<ASYNC, 4, RPT>(p, L, st);
    if (L.max_wl <= 6) return launch_reg_t<ASYNC, 6, RPT>(p, L, st);
    return launch_reg_t<ASYNC, 8, RPT>(p, L, st);
}

template <bool ASYNC, int WLR>
cudaError_t launch_reg_tma_t(const KP &p, const Layout &L, size_t smem, cudaStream_t st) {
    std::lock_guard<std::recursive_mutex> lk(g_launch_mu);
    cudaError_t e = ensure_smem(k_reg_tma<ASYNC, WLR>, smem);
    if (e != cudaSuccess) return e;
    k_reg_tma<ASYNC, WLR><<<(unsigned)L.q, L.spb * kSlice, smem, st>>>(p);
    return cudaGetLastError();
}

// Persistent grid: every block that fits on the device at once (at least one per SM), capped by
// the subdomain count and the tuning's grid cap.
int64_t persistent_grid(int per_sm, const KP &p, const Layout &L) {
    int64_t g = (int64_t)(per_sm < 1 ? 1 : per_sm) * L.sms;
    if (p.grid_cap > 0 && g > p.grid_cap) g = p.grid_cap;
    const int64_t nsub = p.l_end > 0 ? p.l_end - p.l_begin : L.q;
    return g < nsub ? g : nsub;
}

template <bool ASYNC, int WLR>
cudaError_t launch_pers_t(const KP &p, const Layout &L, size_t smem, cudaStream_t st) {
    std::lock_guard<std::recursive_mutex> lk(g_launch_mu);
    auto kfn = k_block_pers<ASYNC, WLR>;
    cudaError_t e = ensure_smem(kfn, smem);
    if (e != cudaSuccess) return e;
    const int64_t g = persistent_grid(occupancy(kfn, L.spb * kSlice, smem), p, L);
    kfn<<<(unsigned)g, L.spb * kSlice, smem, st>>>(p);
    return cudaGetLastError();
}

template <bool ASYNC, int WLR, bool MULTI>
cudaError_t launch_stage_m(const KP &p, const Layout &L, size_t smem, cudaStream_t st) {
    const bool ext = !MULTI && (p.frozen != nullptr || p.tau != 1.0);  // N1 / N3 requested
    auto kfn = MULTI ? k_block_stage_m<true, WLR, true>
                     : (ext ? k_block_stage<ASYNC, WLR, true> : k_block_stage<ASYNC, WLR, false>);
    std::lock_guard<std::recursive_mutex> lk(g_launch_mu);
    cudaError_t e = ensure_smem(kfn, smem);
    if (e != cudaSuccess) return e;
    const int64_t g = persistent_grid(occupancy(kfn, L.spb * kSlice, smem), p, L);
    KP pp = p;
    // a block prefetches x_J two claims ahead; with fewer than ~3 claims of other blocks in
    // between, that could predate the subdomain's own previous update
    pp.fresh_xj = MULTI && L.q < 4 * g;
    kfn<<<(unsigned)g, L.spb * kSlice, smem, st>>>(pp);
    return cudaGetLastError();
}

template <bool ASYNC, int WLR>
cudaError_t launch_pipe_t(const KP &p, const Layout &L, size_t smem, cudaStream_t st) {
    const bool ext = p.frozen != nullptr || p.tau != 1.0;
    auto kfn = ext ? k_block_pipe<ASYNC, WLR, true> : k_block_pipe<ASYNC, WLR, false>;
    std::lock_guard<std::recursive_mutex> lk(g_launch_mu);
    cudaError_t e = ensure_smem(kfn, smem);
    if (e != cudaSuccess) return e;
    const int64_t g = persistent_grid(occupancy(kfn, L.spb * kSlice, smem), p, L);
    kfn<<<(unsigned)g, L.spb * kSlice, smem, st>>>(p);
    return cudaGetLastError();
}

// Name of the coded k_block_duo variant (Layout::last_kernel, bench roofline.kernel): wo4 = the
// unrolled phase 1, bx = b_J, x_J with the slab.
const char *duo_coded_name(bool async, bool bx, int wor) {
    static const char *names[2][2][2] = {
        {{"k_block_duo<sync,coded>", "k_block_duo<sync,coded,wo4>"},
         {"k_block_duo<sync,coded,bx>", "k_block_duo<sync,coded,wo4,bx>"}},
        {{"k_block_duo<async,coded>", "k_block_duo<async,coded,wo4>"},
         {"k_block_duo<async,coded,bx>", "k_block_duo<async,coded,wo4,bx>"}}};
    return names[async][bx][wor == 4 ? 1 : 0];
}

template <bool ASYNC, int WLR>
cudaError_t launch_duo_t(const KP &p, const Layout &L, size_t smem, cudaStream_t st, size_t smem_bx = 0) {
    const bool ext = p.frozen != nullptr || p.tau != 1.0;
    const int coded = p.codes == nullptr ? 0 : (p.sdict != nullptr ? 2 : 1);
    // unrolled phase 1 (WOR) for the coded layouts with <= 4 off-block entries per row
    const int wor = coded == 1 && !ext && L.tune.unroll_off >= 0 && L.max_wo <= 4 ? 4 : 0;
    auto kfn = coded == 2 ? (ext ? k_block_duo<ASYNC, WLR, true, 2> : k_block_duo<ASYNC, WLR, false, 2>)
               : coded == 1 ? (ext ? k_block_duo<ASYNC, WLR, true, 1>
                               : wor == 4 ? k_block_duo<ASYNC, WLR, false, 1, false, 4>
                                          : k_block_duo<ASYNC, WLR, false, 1>)
                            : (ext ? k_block_duo<ASYNC, WLR, true, 0> : k_block_duo<ASYNC, WLR, false, 0>);
    const int threads = L.spb / 2 * kSlice;
    std::lock_guard<std::recursive_mutex> lk(g_launch_mu);
    cudaError_t e = ensure_smem(kfn, smem);
    if (e != cudaSuccess) return e;
    const int occ = occupancy(kfn, threads, smem);
    // b_J / x_J staged with the slab (coded layout, no EXT) where that keeps the blocks per SM
    if (smem_bx > 0 && coded == 1 && !ext) {
        auto kbx = wor == 4 ? k_block_duo<ASYNC, WLR, false, 1, true, 4>
                   : k_block_duo<ASYNC, WLR, false, 1, true>;
        if (ensure_smem(kbx, smem_bx) == cudaSuccess && occupancy(kbx, threads, smem_bx) >= occ) {
            L.last_kernel = duo_coded_name(ASYNC, true, wor);
            const int64_t g = persistent_grid(occ, p, L);
            kbx<<<(unsigned)g, threads, smem_bx, st>>>(p);
            return cudaGetLastError();
        }
        cudaGetLastError();
    }
    if (coded == 1 && !ext) L.last_kernel = duo_coded_name(ASYNC, false, wor);
    const int64_t g = persistent_grid(occ, p, L);
    kfn<<<(unsigned)g, threads, smem, st>>>(p);
    return cudaGetLastError();
}

// k_block_resident for a single-launch async solve when all q subdomains fit on the device at
// once (grid = q blocks co-resident); tuning.resident = -1 keeps the work-queue kernel.
template <int WLR>
bool launch_resident_t(const KP &p, const Layout &L, cudaStream_t st, cudaError_t &err) {
    if (L.tune.resident < 0) return false;
    const int threads = L.spb * kSlice;
    const size_t smem = 2 * (size_t)L.R * sizeof(double) + (size_t)L.max_w * threads * 12;
    if (smem > kSmemMax) return false;
    std::lock_guard<std::recursive_mutex> lk(g_launch_mu);
    if (ensure_smem(k_block_resident<WLR>, smem) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    // every subdomain's block must fit at once (if other work keeps some of them from being
    // resident, the kernel aborts and the host continues with per-launch kernels: DESIGN.md R12)
    if ((int64_t)occupancy(k_block_resident<WLR>, threads, smem) * L.sms < L.q) return false;
    L.last_kernel = "k_block_resident<async>";
    // lead: 48 by default, the loosest bound the residual ring allows (kSlots = 64 slots), i.e. as
    // close to "no inter-block synchronisation" as the bookkeeping gets. Round 1 measured lead 3
    // ahead (C2 51 vs 56-59 iterations with lead 40); with the lazy publication of round 2 the
    // bound no longer matters (B200, tools/kernel_ab.py, medians of 3 x 41 solves, lead 3 / 8 /
    // 16 / 48: C1 0.157 / 0.157 / 0.157 / 0.157 ms with 29 / 28 / 28 / 28 iterations, C2 0.220 /
    // 0.219 / 0.219 / 0.221 ms with 52 / 53 / 53 / 53, C3 0.182 / 0.182 / 0.181 / 0.181 ms, 27)
    KP pp = p;
    pp.lead = L.tune.lead > 0 ? std::min(48, L.tune.lead) : 48;
    pp.fuse_residual = p.ring && L.tune.lazy_publish >= 0 && L.tune.fuse_residual >= 0;
    pp.gather_ahead = L.tune.gather_ahead >= 0;
    // tagged publication (LAZY = 2) while warp 0 can hold the q words, by default in the
    // 256-thread variants (rows with > 12 local entries): there it is faster (C1 0.104 vs 0.122 ms,
    // C3 0.161 vs 0.172); in the 512-thread variant of C2 it was not (0.209 vs 0.202 ms) and cost
    // iterations (56-57 vs 53-54: without the counter's release fence the x stores of an iteration
    // are not drained before the next sweep), so the others keep the counter unless lazy_publish = 2
    if (p.ring && L.tune.lazy_publish >= 0) {
        const bool tagged = L.q <= 32 * resident_pend(WLR) &&
                            (L.tune.lazy_publish == 2 || (L.tune.lazy_publish == 0 && WLR > 12));
        auto kfn = tagged ? k_block_resident<WLR, 2> : k_block_resident<WLR, 1>;
        if (ensure_smem(kfn, smem) != cudaSuccess) {
            cudaGetLastError();
            return false;
        }
        kfn<<<(unsigned)L.q, threads, smem, st>>>(pp);
    } else {
        k_block_resident<WLR><<<(unsigned)L.q, threads, smem, st>>>(pp);
    }
    err = cudaGetLastError();
    return true;
}

template <bool ASYNC, int WLR>
cudaError_t launch_stage_t(const KP &p, const Layout &L, size_t smem, cudaStream_t st) {
    if (ASYNC && p.w_end > 0) {
        cudaError_t e = cudaSuccess;
        if (launch_resident_t<WLR>(p, L, st, e)) return e;
        L.last_kernel = "k_block_stage_m<async>";
        return launch_stage_m<true, WLR, true>(p, L, smem, st);
    }
    return launch_stage_m<ASYNC, WLR, false>(p, L, smem, st);
}

// Whether the staged (TMA) block kernels apply to this layout and these vectors.
bool staged_ok(const KP &p, const Layout &L) {
    const bool aligned = ((uintptr_t)p.b % 16 == 0) && ((uintptr_t)p.x_in % 16 == 0);
    const bool geom_ok = L.spb % 4 == 0 && L.R % 2 == 0 &&
                         ((L.spb <= 32 && L.max_wl <= 8) || (L.spb <= 16 && L.max_wl <= 12) || (L.spb <= 8 && L.max_wl <= 16));
    const size_t stage_smem = 2 * (size_t)stage_geom(L.R, L.spb, L.max_w).bytes + (size_t)L.R * sizeof(double);
    return aligned && geom_ok && stage_smem <= kSmemMax;
}

// Kernel choice for one block-sweep launch (async / sync-block / Jacobi), in order:
//   k_block_duo    two blocks per SM, <= 4 local entries per row, R >= 256 (C4, C5; coded
//                  columns when the layout has them); async always, sync when the pipelined
//                  kernel would hold a whole SM
//   k_block_pipe   persistent, two subdomains of look-ahead (R >= 256 or sync-block k >= 3)
//   k_block_stage  persistent, whole-subdomain TMA stages; with p.w_end > 0 (single launch for
//                  all iterations): k_block_resident when every subdomain fits on the device at
//                  once (C1-C3), else the work-queue k_block_stage_m
//   k_block_pers   persistent, double-buffered TMA slice stream
//   k_reg_tma  subdomains of <= 1024 rows with <= 8 local entries per row: TMA-streamed slices,
//              register-resident local entries
//   k_reg      same without TMA (tuning.kernel = 2, for comparison)
//   k_block    anything else: local entries staged in shared memory when they fit, else
//              re-read through L1/L2 each sweep (tuning.kernel = 1 forces it)
// The choice depends only on the layout, the vectors' alignment and the handle's bar_tuning.
template <bool ASYNC>
cudaError_t launch_block(KP p, const Layout &L, cudaStream_t st) {
    const bar_tuning &T = L.tune;
    const int kind = T.kernel;  // 0 auto, 1 k_block, 2 k_reg, 3 k_reg_tma, 4 k_block_pers
    p.wlmax = L.max_wl;
    p.wmax = L.max_w;
    // async subdomain order of the per-launch kernels: static claims by default. Measured on
    // B200 (round 1): the device work queue's atomic claims cost 0.6 ms/iteration on some boxes
    // (C5 k=5: 3.57 vs 2.91 ms) and converged no faster (59 vs 57 global iterations).
    p.static_claims = T.async_queue != 1;
    // async claim order of k_block_pipe / k_block_duo: contiguous chunks by default. Measured on
    // B200 (round 1, tools/kernel_ab.py, async-(5) to 1e-10): C5 (R = 1024) 44 global iterations
    // vs 59 with round robin, C4 (R = 512) 63 vs 105 — each block sweeps its chunk in order, so
    // the neighbouring lines / planes below a subdomain already hold this iteration's values.
    // (sync modes: the order does not change the iterates; round robin)
    p.claim_chunk = T.async_order == 0 ? (ASYNC ? 1 : 0) : (T.async_order == 1 ? 1 : 0);
    p.fronts = T.async_order == 3 ? (T.fronts > 0 ? T.fronts : 8) : 0;
    const size_t tma_smem = (size_t)L.spb * slice_buf_bytes(L.max_w) + 2 * (size_t)L.R * sizeof(double);
    const size_t pers_smem = tma_smem + (size_t)L.spb * slice_buf_bytes(L.max_w);
    const size_t stage_smem = 2 * (size_t)stage_geom(L.R, L.spb, L.max_w).bytes + (size_t)L.R * sizeof(double);
    const bool aligned = ((uintptr_t)p.b % 16 == 0) && ((uintptr_t)p.x_in % 16 == 0);
    // bulk-copy sources must be 16-byte aligned: b/x at l*R rows (R even), ptr/sw at l*spb
    const bool geom_ok = L.spb % 4 == 0 && L.R % 2 == 0 &&
                         ((L.spb <= 32 && L.max_wl <= 8) || (L.spb <= 16 && L.max_wl <= 12) || (L.spb <= 8 && L.max_wl <= 16));
    const PipeGeom pg = pipe_geom(L.R, L.spb, L.max_w);
    const size_t pipe_smem = 2 * (size_t)pg.vc_bytes + 3 * (size_t)pg.bx_bytes;
    // measured on B200 (round 1, tools/local_iters.py, kernel_ab.py): the two-ahead pipeline wins
    // for sync-block (C5: 2.64 vs 3.51 ms/iteration) and, since async claims are static (no
    // work-queue atomic on the issuing thread), for async and Jacobi with R >= 256 too (C5:
    // 2.65 vs 3.35 and 2.58 vs 2.69 ms; C4 at R = 256: 0.38 vs 0.42 ms); with R = 128 (C4) the
    // one-ahead kernel is 2% faster for async.
    const bool pipe_on = (T.pipe ? T.pipe > 0 : ((!ASYNC && p.k >= 3) || L.R >= 256)) &&
                         (!ASYNC || p.static_claims);  // the pipeline claims statically
    // two-blocks-per-SM variant (k_block_duo) where the pipelined kernel holds a whole SM (C5
    // sync modes, B200 round 1, tools/kernel_ab.py: Jacobi 2.45 vs 2.58 ms, sync-block-(5) 2.56-2.67
    // vs 2.67 ms per launch); coded columns (Layout::codes, 1 byte per entry instead of 4) when
    // the layout has them
    const bool coded = L.codes != nullptr && T.coded >= 0;
    // staged gathers (CODED = 2, tuning.coded = 2) where every subdomain's off-block columns fit
    // its x intervals. Not the default: measured on B200 (round 2, tools/kernel_ab.py, async-(5))
    // C4 0.474 vs 0.335 ms and C5 2.83 vs 2.42 ms per launch against the entry-by-entry relaxed
    // gathers (one more barrier per subdomain; on C4 the buffer costs a block per SM; on C5 each
    // ghost value is used once, so staging adds shared-memory traffic and saves no global loads)
    const bool staged = coded && L.sdict != nullptr && L.xs_len > 0 && T.coded == 2;
    const size_t duo_smem = duo_geom(L.R, L.spb, L.max_w, coded, staged ? (int)L.xs_len : 0).bytes;
    const bool duo_fits = L.spb % 2 == 0 && L.spb >= 8 && L.max_wl <= 4 && 2 * (duo_smem + 2048) <= 228 * 1024;
    // Async: two blocks per SM whenever they fit (C5 R = 1024: 2.69 vs 2.93 ms per launch with
    // chunked claims; C4 R = 512: 0.40 vs 0.52 ms). With round-robin claims the 2 x 148
    // subdomains in flight (303K rows on C5) exceeded the plane coupling distance (262K) and cost
    // global iterations (63 vs 59); chunked claims do not depend on the window.
    const bool duo_on = (T.duo ? T.duo > 0 : ((ASYNC && p.claim_chunk) || pipe_smem > 113 * 1024)) && duo_fits &&
                        (!ASYNC || p.static_claims);
    if (kind == 0 && duo_on && p.w_end == 0 && geom_ok && aligned) {
        L.last_kernel = staged  ? (ASYNC ? "k_block_duo<async,staged>" : "k_block_duo<sync,staged>")
                        : coded ? (ASYNC ? "k_block_duo<async,coded>" : "k_block_duo<sync,coded>")
                                : (ASYNC ? "k_block_duo<async>" : "k_block_duo<sync>");
        KP pc = p;
        if (coded) {
            pc.codes = L.codes;
            pc.dict = L.dict;
            pc.dptr = L.dptr;
        }
        if (staged) {
            pc.sdict = L.sdict;
            pc.iv = L.iv;
            pc.xs_len = (int32_t)L.xs_len;
        }
        // b_J / x_J with the slab: n even (every subdomain's rows then end on a 16-byte boundary)
        const size_t bx_smem = (coded && !staged && L.n % 2 == 0 && T.stage_bx >= 0)
                                   ? duo_geom(L.R, L.spb, L.max_w, true, 0, true).bytes
                                   : 0;
        return launch_duo_t<ASYNC, 4>(pc, L, duo_smem, st, bx_smem);  // two rows per thread: <= 4 local entries
    }
    if (kind == 0 && pipe_on && p.w_end == 0 && geom_ok && aligned && pipe_smem <= kSmemMax) {
        L.last_kernel = ASYNC ? "k_block_pipe<async>" : "k_block_pipe<sync>";
        if (L.max_wl <= 4) return launch_pipe_t<ASYNC, 4>(p, L, pipe_smem, st);
        if (L.max_wl <= 6) return launch_pipe_t<ASYNC, 6>(p, L, pipe_smem, st);
        if (L.max_wl <= 8) return launch_pipe_t<ASYNC, 8>(p, L, pipe_smem, st);
        if (L.max_wl <= 12) return launch_pipe_t<ASYNC, 12>(p, L, pipe_smem, st);  // <= 512 threads
        return launch_pipe_t<ASYNC, 16>(p, L, pipe_smem, st);
    }
    if (p.l_end > 0) return cudaErrorNotSupported;  // subdomain ranges: k_block_duo / k_block_pipe only
    if (kind == 0 && geom_ok && aligned && stage_smem <= kSmemMax) {
        L.last_kernel = ASYNC ? "k_block_stage<async>" : "k_block_stage<sync>";
        if (L.max_wl <= 4) return launch_stage_t<ASYNC, 4>(p, L, stage_smem, st);
        if (L.max_wl <= 6) return launch_stage_t<ASYNC, 6>(p, L, stage_smem, st);
        if (L.max_wl <= 8) return launch_stage_t<ASYNC, 8>(p, L, stage_smem, st);
        if (L.max_wl <= 12) return launch_stage_t<ASYNC, 12>(p, L, stage_smem, st);  // <= 512 threads
        return launch_stage_t<ASYNC, 16>(p, L, stage_smem, st);  // <= 256 threads per block
    }
    if (p.w_end > 0) return cudaErrorNotSupported;  // no persistent multi-iteration kernel here
    const bool ext = p.frozen != nullptr || p.tau != 1.0;  // N1/N3: only k_block_stage and k_block
    if (!ext && (kind == 0 || kind == 4) && L.spb <= 32 && L.max_wl <= 8 && pers_smem <= kSmemBudget) {
        L.last_kernel = ASYNC ? "k_block_pers<async>" : "k_block_pers<sync>";
        if (L.max_wl <= 4) return launch_pers_t<ASYNC, 4>(p, L, pers_smem, st);
        if (L.max_wl <= 6) return launch_pers_t<ASYNC, 6>(p, L, pers_smem, st);
        return launch_pers_t<ASYNC, 8>(p, L, pers_smem, st);
    }
    if (!ext && (kind == 0 || kind == 3) && L.spb <= 32 && L.max_wl <= 8 && tma_smem <= kSmemBudget) {
        L.last_kernel = ASYNC ? "k_reg_tma<async>" : "k_reg_tma<sync>";
        if (L.max_wl <= 4) return launch_reg_tma_t<ASYNC, 4>(p, L, tma_smem, st);
        if (L.max_wl <= 6) return launch_reg_tma_t<ASYNC, 6>(p, L, tma_smem, st);
        return launch_reg_tma_t<ASYNC, 8>(p, L, tma_smem, st);
    }
    if (!ext && kind != 1 && L.spb <= 32 && L.max_wl <= 8) {
        L.last_kernel = ASYNC ? "k_reg<async>" : "k_reg<sync>";
        return launch_reg_w<ASYNC, 1>(p, L, st);
    }
    L.last_kernel = ASYNC ? "k_block<async>" : "k_block<sync>";
    const size_t row_bytes = 3 * (size_t)L.R * sizeof(double);  // y0, y1, s
    const size_t stage_bytes = (size_t)L.max_wl * L.spb * kSlice * (sizeof(double) + sizeof(int32_t));
    const bool stage = row_bytes + stage_bytes <= kSmemBudget;
    const size_t smem = row_bytes + (stage ? stage_bytes : 0);
    int W = L.spb < 32 ? L.spb : 32;
    if (T.warps >= 1 && T.warps <= 32) W = T.warps < L.spb ? T.warps : L.spb;
    if (stage) return launch_block_t<ASYNC, true>(p, W * 32, smem, (unsigned)L.q, st);
    return launch_block_t<ASYNC, false>(p, W * 32, smem, (unsigned)L.q, st);
}

// Persistent grid for the rowwise kernels: as many 256-thread blocks as fit on the device at
// once (two slice buffers per warp), capped by the number of 8-slice groups.
bool rowwise_tma_ok(const Layout &L) { return 16 * (size_t)slice_buf_bytes(L.max_w) <= kSmemBudget; }

template <bool RES>
cudaError_t launch_rowwise(KP p, const Layout &L, cudaStream_t st) {
    p.wmax = L.max_w;
    if (!rowwise_tma_ok(L) || L.tune.kernel == 2) {
        if (!RES) L.last_kernel = "k_rowwise<jacobi>";
        k_rowwise<RES><<<(unsigned)((L.nslices + 7) / 8), 256, 0, st>>>(p);
        return cudaGetLastError();
    }
    const size_t smem = 16 * (size_t)slice_buf_bytes(L.max_w);
    const int64_t grid = rowwise_grid(L);
    std::lock_guard<std::recursive_mutex> lk(g_launch_mu);
    cudaError_t e = ensure_smem(k_rowwise_tma<RES>, smem);
    if (e != cudaSuccess) return e;
    if (!RES) L.last_kernel = "k_rowwise_tma<jacobi>";
    k_rowwise_tma<RES><<<(unsigned)grid, 256, smem, st>>>(p);
    return cudaGetLastError();
}

}  // namespace

int64_t rowwise_grid(const Layout &L) {
    if (L.rw_grid >= 0) return L.rw_grid;
    const int64_t groups = (L.nslices + 7) / 8;
    if (!rowwise_tma_ok(L)) return L.rw_grid = groups;
    const size_t smem = 16 * (size_t)slice_buf_bytes(L.max_w);
    std::lock_guard<std::recursive_mutex> lk(g_launch_mu);
    int a = 0, b = 0;
    if (ensure_smem(k_rowwise_tma<true>, smem) == cudaSuccess && ensure_smem(k_rowwise_tma<false>, smem) == cudaSuccess) {
        a = occupancy(k_rowwise_tma<true>, 256, smem);
        b = occupancy(k_rowwise_tma<false>, 256, smem);
    }
    cudaGetLastError();
    int64_t per_sm = a < b ? a : b;  // the same grid for both (deterministic reductions)
    if (per_sm < 1) per_sm = 1;
    const int64_t g = per_sm * L.sms;
    return L.rw_grid = (g < groups ? g : groups);
}

int64_t num_blocks_for(const Layout &L, bar_mode mode) {
    int64_t rowwise = rowwise_grid(L);
    int64_t legacy = (L.nslices + 7) / 8;
    if (legacy > rowwise) rowwise = legacy;
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
    p.dist_out = a.dist_out;
    p.frozen = a.frozen;
    p.tau = a.tau;
    p.w_end = 0;
    p.l_begin = a.l_begin;
    p.l_end = a.l_end;
    p.stop = a.stop ? a.stop : &a.state->stop;
    if (mode == BAR_MODE_JACOBI) {
        // Jacobi (eq. 2) is sync-block-(1) for any R, with the same per-row arithmetic
        // (off-block entries, then local ones, diagonal included): use the staged stream
        if (a.L->tune.jacobi_rowwise != 1 && staged_ok(p, *a.L)) {
            p.k = 1;
            return launch_block<false>(p, *a.L, st);
        }
        if (p.l_end > 0) return cudaErrorNotSupported;
        return launch_rowwise<false>(p, *a.L, st);
    }
    if (mode == BAR_MODE_ASYNC) return launch_block<true>(p, *a.L, st);
    return launch_block<false>(p, *a.L, st);
}

cudaError_t launch_async_multi(const SweepArgs &a, long long w_end, cudaStream_t st) {
    KP p = make_kp(*a.L);
    p.b = a.b;
    p.x_in = a.x_in;
    p.x_out = a.x_out;
    p.k = a.k;
    p.state = a.state;
    p.partials = a.partials;
    p.hist = a.hist;
    p.dist_out = a.dist_out;
    p.frozen = a.frozen;
    p.tau = a.tau;
    p.w_end = w_end > 0 ? w_end : 1;
    p.m0 = a.m0;
    p.stop = &a.state->stop;
    p.ring = a.ring;
    p.bsum_arr = a.bsum_arr;
    return launch_block<true>(p, *a.L, st);
}

cudaError_t launch_residual(const Layout &L, const double *b, const double *x, DevState *state, double *partials,
                            cudaStream_t st, double *dist_out, bool init_check) {
    KP p = make_kp(L);
    p.b = b;
    p.x_in = x;
    p.state = state;
    p.partials = partials;
    p.dist_out = dist_out;
    p.init_check = init_check && dist_out == nullptr ? 1 : 0;
    return launch_rowwise<true>(p, L, st);
}

__global__ void k_pack(const double *__restrict__ x_own, const int32_t *__restrict__ idx, int64_t cnt,
                       double *__restrict__ out) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cnt; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = x_own[idx[i]];
}

cudaError_t launch_pack(const double *x_own, const int32_t *idx, int64_t cnt, double *out, cudaStream_t st) {
    if (cnt <= 0) return cudaSuccess;
    int64_t blocks = (cnt + 255) / 256;
    if (blocks > 4096) blocks = 4096;
    k_pack<<<(unsigned)blocks, 256, 0, st>>>(x_own, idx, cnt, out);
    return cudaGetLastError();
}

// Rank-ordered sum of the gathered per-rank [sum r^2, sum b^2]: every rank computes the same
// bits, so every rank takes the same stopping decision.
__global__ void k_dist_decide(DevState *S, const double *__restrict__ g, int nranks, int residual_only) {
    if (!residual_only && S->stop) return;  // queued iterations after the stop: sweeps were skipped
    double ss = 0.0, bsq = 0.0;
    for (int r = 0; r < nranks; ++r) {
        ss += g[2 * r];
        bsq += g[2 * r + 1];
    }
    apply_stop_rule(S, ss, bsq, residual_only != 0, nullptr);
}

cudaError_t launch_dist_decide(DevState *state, const double *gathered, int nranks, bool residual_only,
                               cudaStream_t st) {
    k_dist_decide<<<1, 1, 0, st>>>(state, gathered, nranks, residual_only ? 1 : 0);
    return cudaGetLastError();
}

__global__ void k_resume_queue(DevState *S, int clear_slots) {
    if (clear_slots) {
        S->done[threadIdx.x] = 0u;
        S->ss[threadIdx.x] = 0.0;
        S->bs[threadIdx.x] = 0.0;
    }
    if (threadIdx.x == 0) {
        S->stop = 0;
        S->work = S->work_resume;
        S->fuse_arrive = 0;
        S->fuse_ticket = 0;
        S->exact_fused = 0;
        S->epoch += 1;
    }
}

cudaError_t launch_resume_queue(DevState *state, cudaStream_t st, bool clear_slots) {
    k_resume_queue<<<1, kSlots, 0, st>>>(state, clear_slots ? 1 : 0);
    return cudaGetLastError();
}

__global__ void __launch_bounds__(256) k_zero_start(KP p) {
    double s = 0.0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < p.n; i += (int64_t)gridDim.x * blockDim.x) {
        const double v = p.b[i];
        s += v * v;
    }
    reduce_finalize<kResidual>(s, s, p);  // exact_ss = ||b||^2, exact_rel = ||b|| / ||b||
}

cudaError_t launch_zero_start_residual(const Layout &L, const double *b, DevState *state, double *partials,
                                       cudaStream_t st, bool init_check) {
    KP p = make_kp(L);
    p.b = b;
    p.state = state;
    p.partials = partials;
    p.init_check = init_check ? 1 : 0;
    k_zero_start<<<(unsigned)rowwise_grid(L), 256, 0, st>>>(p);
    return cudaGetLastError();
}

__global__ void k_init_check(DevState *S) { init_check_rule(S); }

// After an aborted single-launch solve: continue counting global iterations from the completed
// ones with per-launch kernels (S->iter is the per-launch kernels' counter).
__global__ void k_continue_per_launch(DevState *S) {
    S->iter = S->iters_done;
    S->stop = 0;
    S->aborted = 0;
    S->counter = 0;
    S->work = 0;
}

cudaError_t launch_continue_per_launch(DevState *state, cudaStream_t st) {
    k_continue_per_launch<<<1, 1, 0, st>>>(state);
    return cudaGetLastError();
}

cudaError_t launch_init_check(DevState *state, cudaStream_t st) {
    k_init_check<<<1, 1, 0, st>>>(state);
    return cudaGetLastError();
}

cudaError_t launch_init_state(DevState *state, double tol, cudaStream_t st) {
    k_init_state<<<1, 1, 0, st>>>(state, tol);
    return cudaGetLastError();
}

}  // namespace bar

#ifdef BAR_PROFILE_DUO
extern "C" int bar_debug_duo_profile(unsigned long long *out32, int reset) {
    cudaMemcpyFromSymbol(out32, bar::g_duo_prof, sizeof(unsigned long long) * 32);
    if (reset) {
        unsigned long long z[32] = {};
        cudaMemcpyToSymbol(bar::g_duo_prof, z, sizeof(z));
    }
    return (int)cudaGetLastError();
}
#endif

#ifdef BAR_PROFILE_RESIDENT
extern "C" int bar_debug_resident_profile(unsigned long long *out8, int reset) {
    cudaMemcpyFromSymbol(out8, bar::g_res_prof, sizeof(unsigned long long) * 8);
    if (reset) {
        unsigned long long z[8] = {};
        cudaMemcpyToSymbol(bar::g_res_prof, z, sizeof(z));
    }
    return (int)cudaGetLastError();
}
#endif
