// layout.cu — CSR validation and conversion to the split sliced-ELL device layout
// (the layout itself is described in bar_internal.cuh / DESIGN.md).
//
// Runs once per bar_create_csr on the device (the 128M-row config has ~0.94G entries), outside
// every timed region ("initialisation ... subtracted").
#include <cub/cub.cuh>

#include <climits>
#include <cstdlib>

#include "bar_internal.cuh"

namespace bar {
namespace {

enum : int { kErrBadCsr = 1, kErrZeroDiag = 2, kErrNonFinite = 4 };

__device__ __forceinline__ void slice_row(int64_t s, int32_t R, int32_t spb, int64_t n, int64_t &row, bool &valid,
                                          int64_t &TS, int lane) {
    int64_t l = s / spb;
    int64_t j = s - l * spb;
    TS = l * (int64_t)R;
    int64_t nrows = min((int64_t)R, n - TS);
    int64_t loc = j * kSlice + lane;
    valid = loc < nrows;
    row = TS + loc;
}

// Per row: validate and count local (column inside the row's subdomain, diagonal included)
// and off-block entries.
// Columns may range over [col_lo, col_hi) with col_lo <= 0: a multi-GPU rank numbers its
// ghost columns below its first row negatively (order-preserving local numbering, dist.cu).
__global__ void k_validate_count(int64_t n, int64_t nnz, const int32_t *__restrict__ rowptr,
                                 const int32_t *__restrict__ col, const double *__restrict__ val, int32_t R,
                                 int64_t col_lo, int64_t col_hi, int32_t *__restrict__ nloc,
                                 int32_t *__restrict__ noff, int *__restrict__ err) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    int32_t a = rowptr[i], e = rowptr[i + 1];
    if (a < 0 || e < a || e > nnz) {
        atomicOr(err, kErrBadCsr);
        nloc[i] = 1;
        noff[i] = 0;
        return;
    }
    int64_t TS = (i / R) * (int64_t)R;
    int64_t TE = min(TS + (int64_t)R, n);
    int cl = 0, co = 0, bad = 0;
    bool diag = false;
    int64_t prev = col_lo - 1;
    for (int32_t p = a; p < e; ++p) {
        int64_t c = col[p];
        double v = val[p];
        if (c < col_lo || c >= col_hi || c <= prev) bad |= kErrBadCsr;
        prev = c;
        if (!isfinite(v)) bad |= kErrNonFinite;
        if (c == i) {
            diag = true;
            if (v == 0.0) bad |= kErrZeroDiag;
        }
        if (c >= TS && c < TE) ++cl; else ++co;
    }
    if (!diag) bad |= kErrBadCsr;
    if (bad) atomicOr(err, bad);
    nloc[i] = cl;
    noff[i] = co;
}

// Per slice (one warp): widths wl = max local count, wo = max off-block count.
__global__ void k_slice_widths(int64_t nslices, int64_t n, int32_t R, int32_t spb, const int32_t *__restrict__ nloc,
                               const int32_t *__restrict__ noff, int32_t *__restrict__ sw,
                               int64_t *__restrict__ ssize) {
    int64_t s = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / kSlice;
    int lane = threadIdx.x & (kSlice - 1);
    if (s >= nslices) return;
    int64_t row, TS;
    bool valid;
    slice_row(s, R, spb, n, row, valid, TS, lane);
    int wl = valid ? nloc[row] : 1;
    int wo = valid ? noff[row] : 0;
    for (int o = 16; o > 0; o >>= 1) {
        wl = max(wl, __shfl_xor_sync(0xffffffffu, wl, o));
        wo = max(wo, __shfl_xor_sync(0xffffffffu, wo, o));
    }
    if (lane == 0) {
        sw[s] = wl | (wo << 16);
        ssize[s] = (int64_t)kSlice * (wl + wo);
    }
}

// Per (slice, lane): write the lane's column of the slice — first the off-block entries
// ascending (global index), then the diagonal, then the other local entries ascending (local
// index), then padding (value 0, own row). Off-block first means one ascending pass over a row
// produces s_i = b_i - sum_off a_ij x_j before the local part starts (Alg. 1 line 3).
__global__ void k_fill(int64_t nslices, int64_t n, int32_t R, int32_t spb, const int32_t *__restrict__ rowptr,
                       const int32_t *__restrict__ col, const double *__restrict__ val,
                       const int64_t *__restrict__ sptr, const int32_t *__restrict__ sw,
                       double *__restrict__ oval, int32_t *__restrict__ ocol) {
    int64_t gt = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    int64_t s = gt / kSlice;
    int lane = (int)(gt & (kSlice - 1));
    if (s >= nslices) return;
    int64_t row, TS;
    bool valid;
    slice_row(s, R, spb, n, row, valid, TS, lane);
    int wl = sw[s] & 0xffff, wo = sw[s] >> 16;
    int64_t base = sptr[s] + lane;
    int64_t TE = min(TS + (int64_t)R, n);
    int32_t own_loc = valid ? (int32_t)(row - TS) : 0;
    int32_t own_glb = (int32_t)(valid ? row : TS);
    int el = 0, eo = 0;
    if (valid) {
        int32_t a = rowptr[row], e = rowptr[row + 1];
        for (int32_t p = a; p < e; ++p)  // diagonal -> first local entry
            if (col[p] == row) {
                oval[base + (int64_t)wo * kSlice] = val[p];
                ocol[base + (int64_t)wo * kSlice] = own_loc;
                el = 1;
            }
        for (int32_t p = a; p < e; ++p) {
            int64_t c = col[p];
            if (c == row) continue;
            if (c >= TS && c < TE) {
                oval[base + (int64_t)(wo + el) * kSlice] = val[p];
                ocol[base + (int64_t)(wo + el) * kSlice] = (int32_t)(c - TS);
                ++el;
            } else {
                oval[base + (int64_t)eo * kSlice] = val[p];
                ocol[base + (int64_t)eo * kSlice] = (int32_t)c;
                ++eo;
            }
        }
    }
    for (; eo < wo; ++eo) {
        oval[base + (int64_t)eo * kSlice] = 0.0;
        ocol[base + (int64_t)eo * kSlice] = own_glb;
    }
    for (; el < wl; ++el) {
        oval[base + (int64_t)(wo + el) * kSlice] = 0.0;
        ocol[base + (int64_t)(wo + el) * kSlice] = own_loc;
    }
}

// Per subdomain (one block): the off-block columns of a row i are grouped by their offset
// d = c - i; the (at most kGhostRanges) most frequent offsets, each used by at least a quarter of
// the subdomain's rows, give the x ranges [TS + d, TE + d) (clipped to the column range and to
// outside the subdomain itself) that the sweep kernels prefetch into L2 two subdomains ahead of
// the gathers that read them (a3): on stencils that is every off-block column; irregular
// matrices simply get fewer or no ranges. A locality hint only — no result depends on it.
constexpr int kOffSlots = 64;
__global__ void k_ghost_ranges(int64_t n, int32_t R, int64_t col_lo, int64_t col_hi,
                               const int32_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                               int32_t *__restrict__ gr) {
    __shared__ unsigned long long key[kOffSlots];
    __shared__ int cnt[kOffSlots];
    const unsigned long long kEmpty = ~0ull;
    for (int t = threadIdx.x; t < kOffSlots; t += blockDim.x) {
        key[t] = kEmpty;
        cnt[t] = 0;
    }
    __syncthreads();
    const int64_t l = blockIdx.x;
    const int64_t TS = l * (int64_t)R, TE = min(TS + (int64_t)R, n);
    for (int64_t i = TS + threadIdx.x; i < TE; i += blockDim.x) {
        for (int32_t p = rowptr[i]; p < rowptr[i + 1]; ++p) {
            const int64_t c = col[p];
            if (c >= TS && c < TE) continue;
            const unsigned long long k = (unsigned long long)(c - i);
            int h = (int)((k * 0x9E3779B97F4A7C15ull) >> 58);  // 6 bits
            for (int probe = 0; probe < kOffSlots; ++probe, h = (h + 1) & (kOffSlots - 1)) {
                unsigned long long old = atomicCAS(&key[h], kEmpty, k);
                if (old == kEmpty || old == k) {
                    atomicAdd(&cnt[h], 1);
                    break;
                }
            }
        }
    }
    __syncthreads();
    if (threadIdx.x != 0) return;
    const int nrows = (int)(TE - TS);
    int out = 0;
    bool used[kOffSlots];
    for (int t = 0; t < kOffSlots; ++t) used[t] = false;
    for (; out < kGhostRanges; ++out) {
        int best = -1;
        for (int t = 0; t < kOffSlots; ++t)
            if (!used[t] && key[t] != kEmpty && (best < 0 || cnt[t] > cnt[best])) best = t;
        if (best < 0 || 4 * cnt[best] < nrows) break;
        used[best] = true;
        const int64_t d = (int64_t)key[best];
        int64_t lo = max(TS + d, col_lo), hi = min(TE + d, col_hi);
        if (lo < TS && hi > TS) hi = TS;  // the subdomain's own x_J is staged anyway
        if (lo < TE && hi > TE) lo = TE;
        if (hi <= lo) { --out; continue; }
        gr[2 * (l * kGhostRanges + out)] = (int32_t)lo;
        gr[2 * (l * kGhostRanges + out) + 1] = (int32_t)(hi - lo);
    }
    for (; out < kGhostRanges; ++out) {
        gr[2 * (l * kGhostRanges + out)] = 0;
        gr[2 * (l * kGhostRanges + out) + 1] = 0;
    }
}

// Per subdomain (one block): the dictionary of its column offsets d = col - row (off-block
// entries store global columns, local ones col - TS; padding has d = 0), keyed by (d, local):
// an offset that is local for some rows of the subdomain and off-block for others (a 3D
// stencil's -512 in a two-line subdomain) gets two codes. dcount[l] = dictionary size, or -1 if
// it exceeds kDictMax (then no coded layout). Entries of the rows past n in the last subdomain
// are never read: code 0.
//
// Staged gathers: the off-block columns of the subdomain's real (non-padding) entries with
// offset d span [TS + d + loc_min(d), TS + d + loc_max(d)]; merged (gaps <= kIvGap), these
// spans give at most kMaxIv intervals of x that the sweep copies into shared memory once per
// visit (one pass of coalesced relaxed loads) instead of gathering entry by entry. sdict[code]
// is then, for an off-block code, the shared-memory index offset TS + d - lo_r + base_r of its
// interval r (x of entry (loc, code) at xs[loc + sdict[code]]), for a local code d itself, and
// 0 for off-block padding (value 0; xs[loc] is finite since the buffer holds >= R values).
// iv[l] = kMaxIv x (lo, len, base, 0); ivlen[l] = buffer length, or -1 when the subdomain's
// off-block columns do not fit kMaxIv intervals of total length <= kIvCap * R.
constexpr int kDictSlots = 2 * kDictMax;
constexpr int kIvGap = 16;
constexpr int kIvCap = 4;
__global__ void k_codes(int64_t n, int32_t R, int32_t spb, const int64_t *__restrict__ sptr,
                        const int32_t *__restrict__ sw, const int32_t *__restrict__ col, uint8_t *__restrict__ codes,
                        int32_t *__restrict__ dtmp, int32_t *__restrict__ stmp, int32_t *__restrict__ dcount,
                        int32_t *__restrict__ iv, int32_t *__restrict__ ivlen) {
    __shared__ long long key[kDictSlots];
    __shared__ int32_t code[kDictSlots];
    __shared__ int32_t mnl[kDictSlots], mxl[kDictSlots];
    __shared__ long long st[kDictMax], en[kDictMax];  // thread 0: spans of the off-block offsets
    __shared__ int overflow;
    const long long kEmpty = (long long)0x8000000000000000ull;
    for (int t = threadIdx.x; t < kDictSlots; t += blockDim.x) {
        key[t] = kEmpty;
        mnl[t] = INT32_MAX;
        mxl[t] = -1;
    }
    if (threadIdx.x == 0) overflow = 0;
    __syncthreads();
    const int64_t l = blockIdx.x, TS = l * (int64_t)R;
    const int nrows = (int)min((int64_t)R, n - TS);
    const int nsl = (nrows + kSlice - 1) / kSlice;
    auto slot_of = [&](long long k, bool insert) -> int {
        int h = (int)(((unsigned long long)k * 0x9E3779B97F4A7C15ull) >> 55) & (kDictSlots - 1);  // 9 bits
        for (int probe = 0; probe < kDictSlots; ++probe, h = (h + 1) & (kDictSlots - 1)) {
            const long long kk = key[h];
            if (kk == k) return h;
            if (kk == kEmpty) {
                if (!insert) return -1;
                const long long old = (long long)atomicCAS((unsigned long long *)&key[h], (unsigned long long)kEmpty,
                                                           (unsigned long long)k);
                if (old == kEmpty || old == k) return h;
            }
        }
        return -1;
    };
    for (int pass = 0; pass < 2; ++pass) {
        for (int j = 0; j < nsl; ++j) {
            const int64_t s = l * spb + j, E = sptr[s];
            const int wl = sw[s] & 0xffff, wo = sw[s] >> 16;
            for (int t = threadIdx.x; t < kSlice * (wl + wo); t += blockDim.x) {
                const int lane = t & (kSlice - 1), e = t / kSlice, loc = j * kSlice + lane;
                if (loc >= nrows) {
                    if (pass == 1) codes[E + t] = 0;
                    continue;
                }
                const int32_t c = col[E + t];
                const bool local = e >= wo;
                const int32_t d = local ? c - loc : (int32_t)(c - (TS + loc));
                const int h = slot_of(((long long)d << 1) | (local ? 1 : 0), pass == 0);
                if (h < 0) {
                    overflow = 1;
                    continue;
                }
                if (pass == 1) {
                    codes[E + t] = (uint8_t)code[h];
                    if (!local && (c < TS || c >= TS + nrows)) {  // a real off-block entry
                        atomicMin(&mnl[h], loc);
                        atomicMax(&mxl[h], loc);
                    }
                }
            }
        }
        __syncthreads();
        if (pass == 0 && threadIdx.x == 0) {
            int cnt = 0;
            for (int h = 0; h < kDictSlots; ++h) {
                if (key[h] == kEmpty) continue;
                if (cnt < kDictMax) dtmp[l * kDictMax + cnt] = (int32_t)(key[h] >> 1);
                code[h] = cnt++;
            }
            if (cnt == 0) dtmp[l * kDictMax + cnt++] = 0;
            if (cnt > kDictMax) overflow = 1;
            dcount[l] = overflow ? -1 : cnt;
        }
        __syncthreads();
        if (overflow) return;
    }
    if (threadIdx.x != 0) return;
    // intervals: spans of the real off-block offsets, sorted by start and merged
    int ns = 0;
    for (int h = 0; h < kDictSlots; ++h) {
        if (key[h] == kEmpty || (key[h] & 1) || mxl[h] < 0) continue;
        const long long d = key[h] >> 1;
        long long a = TS + d + mnl[h], b = TS + d + mxl[h] + 1;
        int i = ns++;
        while (i > 0 && st[i - 1] > a) {  // insertion sort by start
            st[i] = st[i - 1];
            en[i] = en[i - 1];
            --i;
        }
        st[i] = a;
        en[i] = b;
    }
    long long lo[kMaxIv], hi[kMaxIv];
    int ni = 0;
    bool ok = true;
    for (int i = 0; i < ns && ok; ++i) {
        if (ni > 0 && st[i] <= hi[ni - 1] + kIvGap) {
            if (en[i] > hi[ni - 1]) hi[ni - 1] = en[i];
        } else if (ni == kMaxIv) {
            ok = false;
        } else {
            lo[ni] = st[i];
            hi[ni] = en[i];
            ++ni;
        }
    }
    long long tot = 0;
    for (int r = 0; r < ni; ++r) tot += hi[r] - lo[r];
    if (tot > (long long)kIvCap * R) ok = false;
    long long base[kMaxIv];
    {
        long long acc = 0;
        for (int r = 0; r < ni; ++r) {
            base[r] = acc;
            acc += hi[r] - lo[r];
        }
    }
    for (int r = 0; r < kMaxIv; ++r) {
        int32_t *o = iv + 4 * (l * kMaxIv + r);
        o[0] = ok && r < ni ? (int32_t)lo[r] : 0;
        o[1] = ok && r < ni ? (int32_t)(hi[r] - lo[r]) : 0;
        o[2] = ok && r < ni ? (int32_t)base[r] : 0;
        o[3] = 0;
    }
    ivlen[l] = ok ? (int32_t)(tot > R ? tot : R) : -1;
    for (int h = 0; h < kDictSlots; ++h) {
        if (key[h] == kEmpty) continue;
        const long long d = key[h] >> 1;
        int32_t v = (int32_t)d;  // local code: the local offset
        if (!(key[h] & 1)) {
            v = 0;  // off-block padding only
            if (mxl[h] >= 0 && ok) {
                const long long a = TS + d + mnl[h];
                for (int r = 0; r < ni; ++r)
                    if (a >= lo[r] && a < hi[r]) v = (int32_t)(TS + d - lo[r] + base[r]);
            }
        }
        stmp[l * kDictMax + code[h]] = v;
    }
}

// Padded dictionary sizes (multiples of 4 int32 = 16 bytes, the bulk-copy granule).
__global__ void k_dict_pad(int64_t q, const int32_t *__restrict__ dcount, int32_t *__restrict__ dsize) {
    const int64_t l = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (l < q) dsize[l] = (dcount[l] + 3) & ~3;
    if (l == q) dsize[l] = 0;
}

__global__ void k_dict_compact(int64_t q, const int32_t *__restrict__ dtmp, const int32_t *__restrict__ stmp,
                               const int32_t *__restrict__ dcount, const int32_t *__restrict__ dptr,
                               int32_t *__restrict__ dict, int32_t *__restrict__ sdict) {
    const int64_t l = blockIdx.x;
    const int cnt = dcount[l], sz = dptr[l + 1] - dptr[l];
    for (int c = threadIdx.x; c < sz; c += blockDim.x) {
        dict[dptr[l] + c] = c < cnt ? dtmp[l * kDictMax + c] : 0;
        sdict[dptr[l] + c] = c < cnt ? stmp[l * kDictMax + c] : 0;
    }
}

template <class T>
cudaError_t dmalloc(T **p, size_t count) {
    return cudaMalloc((void **)p, sizeof(T) * (count ? count : 1));
}

}  // namespace

void free_layout(Layout &L) {
    cudaFree(L.val);
    cudaFree(L.col);
    cudaFree(L.sptr);
    cudaFree(L.sw);
    L.val = nullptr;
    L.col = nullptr;
    L.sptr = nullptr;
    L.sw = nullptr;
    cudaFree(L.gr);
    L.gr = nullptr;
    cudaFree(L.codes);
    cudaFree(L.dict);
    cudaFree(L.dptr);
    cudaFree(L.sdict);
    cudaFree(L.iv);
    L.codes = nullptr;
    L.dict = nullptr;
    L.dptr = nullptr;
    L.sdict = nullptr;
    L.iv = nullptr;
    L.dict_entries = 0;
    L.xs_len = 0;
}

// Coded columns (Layout::codes); leaves them NULL when a subdomain has more than kDictMax
// distinct offsets or memory is short (the kernels then read the int32 columns). With them, the
// staged-gather tables (Layout::sdict / iv / xs_len) when every subdomain's off-block columns fit
// its intervals (else xs_len = 0: the coded kernels gather from global memory).
static void build_codes(Layout &L, cudaStream_t st) {
    const int64_t q = L.q;
    int32_t *dtmp = nullptr, *stmp = nullptr, *dcount = nullptr, *dsize = nullptr, *ivlen = nullptr, *red = nullptr;
    void *tmp = nullptr;
    size_t tb = 0;
    int32_t mn = 0, total = 0, ivmin = -1, ivmax = 0;
    bool ok = false;
    if (cudaMalloc(&L.codes, (size_t)L.entries + 16) != cudaSuccess ||
        cudaMalloc(&dtmp, sizeof(int32_t) * (size_t)q * kDictMax) != cudaSuccess ||
        cudaMalloc(&stmp, sizeof(int32_t) * (size_t)q * kDictMax) != cudaSuccess ||
        cudaMalloc(&dcount, sizeof(int32_t) * (size_t)(q + 1)) != cudaSuccess ||
        cudaMalloc(&dsize, sizeof(int32_t) * (size_t)(q + 1)) != cudaSuccess ||
        cudaMalloc(&ivlen, sizeof(int32_t) * (size_t)(q + 1)) != cudaSuccess ||
        cudaMalloc(&red, sizeof(int32_t) * 2) != cudaSuccess ||
        cudaMalloc(&L.iv, sizeof(int32_t) * 4 * (size_t)q * kMaxIv) != cudaSuccess ||
        cudaMalloc(&L.dptr, sizeof(int32_t) * (size_t)(q + 1)) != cudaSuccess)
        goto out;
    k_codes<<<(unsigned)q, 256, 0, st>>>(L.n, L.R, L.spb, L.sptr, L.sw, L.col, L.codes, dtmp, stmp, dcount, L.iv,
                                        ivlen);
    if (cub::DeviceReduce::Min(nullptr, tb, dcount, dsize + q, q, st) != cudaSuccess) goto out;
    {
        size_t tb2 = 0;
        if (cub::DeviceScan::ExclusiveSum(nullptr, tb2, dsize, L.dptr, q + 1, st) != cudaSuccess) goto out;
        if (tb2 > tb) tb = tb2;
        if (cub::DeviceReduce::Max(nullptr, tb2, ivlen, red + 1, q, st) != cudaSuccess) goto out;
        if (tb2 > tb) tb = tb2;
    }
    if (cudaMalloc(&tmp, tb) != cudaSuccess) goto out;
    {
        size_t t = tb;
        if (cub::DeviceReduce::Min(tmp, t, dcount, dsize + q, q, st) != cudaSuccess) goto out;
        if (cudaMemcpyAsync(&mn, dsize + q, sizeof(int32_t), cudaMemcpyDeviceToHost, st) != cudaSuccess ||
            cudaStreamSynchronize(st) != cudaSuccess || mn < 1)
            goto out;
        t = tb;
        if (cub::DeviceReduce::Min(tmp, t, ivlen, red, q, st) != cudaSuccess) goto out;
        t = tb;
        if (cub::DeviceReduce::Max(tmp, t, ivlen, red + 1, q, st) != cudaSuccess) goto out;
        if (cudaMemcpyAsync(&ivmin, red, sizeof(int32_t), cudaMemcpyDeviceToHost, st) != cudaSuccess ||
            cudaMemcpyAsync(&ivmax, red + 1, sizeof(int32_t), cudaMemcpyDeviceToHost, st) != cudaSuccess)
            goto out;
        k_dict_pad<<<(unsigned)((q + 1 + 255) / 256), 256, 0, st>>>(q, dcount, dsize);
        t = tb;
        if (cub::DeviceScan::ExclusiveSum(tmp, t, dsize, L.dptr, q + 1, st) != cudaSuccess) goto out;
        if (cudaMemcpyAsync(&total, L.dptr + q, sizeof(int32_t), cudaMemcpyDeviceToHost, st) != cudaSuccess ||
            cudaStreamSynchronize(st) != cudaSuccess)
            goto out;
    }
    if (cudaMalloc(&L.dict, sizeof(int32_t) * (size_t)(total + 4)) != cudaSuccess ||
        cudaMalloc(&L.sdict, sizeof(int32_t) * (size_t)(total + 4)) != cudaSuccess)
        goto out;
    k_dict_compact<<<(unsigned)q, 64, 0, st>>>(q, dtmp, stmp, dcount, L.dptr, L.dict, L.sdict);
    ok = cudaStreamSynchronize(st) == cudaSuccess && cudaGetLastError() == cudaSuccess;
    L.dict_entries = total;
    L.xs_len = ivmin >= 0 ? ((ivmax + 1) & ~1) : 0;  // staged gathers for every subdomain, or none
out:
    cudaGetLastError();
    cudaFree(dtmp);
    cudaFree(stmp);
    cudaFree(dcount);
    cudaFree(dsize);
    cudaFree(ivlen);
    cudaFree(red);
    cudaFree(tmp);
    if (!ok) {
        cudaFree(L.codes);
        cudaFree(L.dict);
        cudaFree(L.dptr);
        cudaFree(L.sdict);
        cudaFree(L.iv);
        L.codes = nullptr;
        L.dict = nullptr;
        L.dptr = nullptr;
        L.sdict = nullptr;
        L.iv = nullptr;
        L.dict_entries = 0;
        L.xs_len = 0;
    }
}

static bar_status alloc_fail(cudaError_t e, const char *what) {
    if (e == cudaErrorMemoryAllocation) {
        cudaGetLastError();
        set_error(std::string("out of device memory: ") + what);
        return BAR_ERR_OOM;
    }
    return cuda_fail(e, what);
}

#define BAR_ALLOC(call)                                        \
    do {                                                       \
        cudaError_t _e = (call);                               \
        if (_e != cudaSuccess) { st_ = alloc_fail(_e, #call); goto done; } \
    } while (0)
#define BAR_CK(call)                                           \
    do {                                                       \
        cudaError_t _e = (call);                               \
        if (_e != cudaSuccess) { st_ = cuda_fail(_e, #call); goto done; } \
    } while (0)

bar_status build_layout(Layout &L, int64_t n, int64_t nnz, const int32_t *d_rowptr, const int32_t *d_col,
                        const double *d_val, int32_t R, cudaStream_t st, int64_t col_lo, int64_t col_hi) {
    if (col_hi < 0) col_hi = n;
    bar_status st_ = BAR_OK;
    int32_t *nloc = nullptr, *noff = nullptr;
    int *d_err = nullptr;
    int64_t *ssize = nullptr;
    void *tmp = nullptr;
    size_t tmp_bytes = 0, tmp2 = 0;
    int h_err = 0;
    int64_t *d_sum = nullptr;
    int64_t h_tot[2] = {0, 0};
    int h_w[2] = {0, 0};
    int64_t h_maxsz = 0;

    L.n = n;
    L.nnz = nnz;
    L.R = R;
    L.spb = (R + kSlice - 1) / kSlice;
    L.q = (n + R - 1) / R;
    {
        int64_t last_rows = n - (L.q - 1) * (int64_t)R;
        L.nslices = (L.q - 1) * (int64_t)L.spb + (last_rows + kSlice - 1) / kSlice;
    }
    const int TB = 256;
    int64_t nsl = L.nslices;

    BAR_ALLOC(dmalloc(&nloc, (size_t)n));
    BAR_ALLOC(dmalloc(&noff, (size_t)n));
    BAR_ALLOC(dmalloc(&d_err, 1));
    BAR_ALLOC(dmalloc(&ssize, (size_t)nsl + 1));
    BAR_ALLOC(dmalloc(&d_sum, 2));
    // +4 entries of slack: bulk copies round metadata ranges up to 16 bytes
    BAR_ALLOC(dmalloc(&L.sptr, (size_t)nsl + 5));
    BAR_ALLOC(dmalloc(&L.sw, (size_t)nsl + 4));
    BAR_CK(cudaMemsetAsync(L.sw + nsl, 0, 4 * sizeof(int32_t), st));
    BAR_CK(cudaMemsetAsync(L.sptr + nsl + 1, 0, 4 * sizeof(int64_t), st));
    BAR_CK(cudaMemsetAsync(d_err, 0, sizeof(int), st));

    k_validate_count<<<(unsigned)((n + TB - 1) / TB), TB, 0, st>>>(n, nnz, d_rowptr, d_col, d_val, R, col_lo,
                                                                  col_hi, nloc, noff, d_err);
    BAR_CK(cudaGetLastError());
    BAR_CK(cudaMemcpyAsync(&h_err, d_err, sizeof(int), cudaMemcpyDeviceToHost, st));
    BAR_CK(cudaStreamSynchronize(st));
    if (h_err & kErrBadCsr) { set_error("malformed CSR (rowptr/col/diagonal)"); st_ = BAR_ERR_BAD_CSR; goto done; }
    if (h_err & kErrNonFinite) { set_error("non-finite matrix value"); st_ = BAR_ERR_NONFINITE; goto done; }
    if (h_err & kErrZeroDiag) { set_error("zero diagonal entry"); st_ = BAR_ERR_ZERO_DIAG; goto done; }

    k_slice_widths<<<(unsigned)((nsl * kSlice + TB - 1) / TB), TB, 0, st>>>(nsl, n, R, L.spb, nloc, noff, L.sw,
                                                                           ssize);
    BAR_CK(cudaGetLastError());
    BAR_CK(cudaMemsetAsync(ssize + nsl, 0, sizeof(int64_t), st));
    // slice offsets: exclusive scan of slice sizes (nslices+1 entries -> sptr[nslices] = total)
    BAR_CK(cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, ssize, L.sptr, nsl + 1, st));
    BAR_CK(cub::DeviceReduce::Sum(nullptr, tmp2, nloc, d_sum + 1, n, st));
    if (tmp2 > tmp_bytes) tmp_bytes = tmp2;
    BAR_CK(cub::DeviceReduce::Max(nullptr, tmp2, nloc, (int32_t *)d_sum, n, st));
    if (tmp2 > tmp_bytes) tmp_bytes = tmp2;
    BAR_CK(cub::DeviceReduce::Max(nullptr, tmp2, ssize, d_sum, nsl, st));
    if (tmp2 > tmp_bytes) tmp_bytes = tmp2;
    BAR_ALLOC(cudaMalloc(&tmp, tmp_bytes));
    BAR_CK(cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, ssize, L.sptr, nsl + 1, st));
    BAR_CK(cudaMemcpyAsync(&h_tot[0], L.sptr + nsl, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    {
        // count local entries (int32 counts summed into int64)
        size_t tb = tmp_bytes;
        BAR_CK(cub::DeviceReduce::Sum(tmp, tb, nloc, d_sum + 1, n, st));
        BAR_CK(cudaMemcpyAsync(&h_tot[1], d_sum + 1, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
        tb = tmp_bytes;
        BAR_CK(cub::DeviceReduce::Max(tmp, tb, nloc, (int32_t *)d_sum, n, st));
        BAR_CK(cudaMemcpyAsync(&h_w[0], d_sum, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
        tb = tmp_bytes;
        BAR_CK(cub::DeviceReduce::Max(tmp, tb, noff, (int32_t *)d_sum, n, st));
        BAR_CK(cudaMemcpyAsync(&h_w[1], d_sum, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
        BAR_CK(cudaStreamSynchronize(st));
        tb = tmp_bytes;
        BAR_CK(cub::DeviceReduce::Max(tmp, tb, ssize, d_sum, nsl, st));
        BAR_CK(cudaMemcpyAsync(&h_maxsz, d_sum, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    }
    BAR_CK(cudaStreamSynchronize(st));
    L.max_w = (int)(h_maxsz / kSlice);
    {
        int dev = 0, sms = 0;
        if (cudaGetDevice(&dev) == cudaSuccess &&
            cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) == cudaSuccess && sms > 0)
            L.sms = sms;
    }
    L.entries = h_tot[0];
    L.local_entries = h_tot[1];
    L.max_wl = h_w[0];
    L.max_wo = h_w[1];
    if (L.max_wl > 0xffff || L.max_wo > 0x7fff) {
        set_error("a row has more than 32767 off-block or 65535 local entries");
        st_ = BAR_ERR_INVALID_ARG;
        goto done;
    }
    // +4 entries of slack so 16-byte vector loads past the last slice stay in bounds
    BAR_ALLOC(dmalloc(&L.val, (size_t)L.entries + 4));
    BAR_ALLOC(dmalloc(&L.col, (size_t)L.entries + 4));
    BAR_CK(cudaMemsetAsync(L.val + L.entries, 0, 4 * sizeof(double), st));
    BAR_CK(cudaMemsetAsync(L.col + L.entries, 0, 4 * sizeof(int32_t), st));
    k_fill<<<(unsigned)((nsl * kSlice + TB - 1) / TB), TB, 0, st>>>(nsl, n, R, L.spb, d_rowptr, d_col, d_val, L.sptr,
                                                                   L.sw, L.val, L.col);
    BAR_CK(cudaGetLastError());
    BAR_ALLOC(dmalloc(&L.gr, (size_t)L.q * kGhostRanges * 2));
    k_ghost_ranges<<<(unsigned)L.q, 256, 0, st>>>(n, R, col_lo, col_hi, d_rowptr, d_col, L.gr);
    BAR_CK(cudaGetLastError());
    BAR_CK(cudaStreamSynchronize(st));
    build_codes(L, st);

done:
    cudaFree(nloc);
    cudaFree(noff);
    cudaFree(d_err);
    cudaFree(ssize);
    cudaFree(d_sum);
    cudaFree(tmp);
    if (st_ != BAR_OK) free_layout(L);
    return st_;
}

}  // namespace bar
