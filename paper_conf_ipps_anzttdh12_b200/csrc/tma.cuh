// tma.cuh — sm_100a bulk-copy (TMA, cp.async.bulk -> SASS UBLKCP) and mbarrier helpers.
//
// A warp streams its 32-row slice of the sliced layout (values, then columns — each a contiguous,
// 128/256-byte-aligned block) into shared memory with two bulk copies that complete on one
// mbarrier. In-flight bytes then cost no registers, which is what keeps enough of the matrix
// stream in flight per SM to approach the HBM roofline (the register-staged loads topped out
// near a third of it, profiles/).
#pragma once

#include <stdint.h>

namespace bar {

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

// Order this thread's earlier generic-proxy shared-memory accesses before later async-proxy
// (bulk copy) writes to the same buffer (buffer reuse).
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ bool mbar_try_wait(uint64_t *bar, uint32_t phase) {
    uint32_t done;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(phase)
        : "memory");
    return done != 0;
}

__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t phase) {
    while (!mbar_try_wait(bar, phase)) {
    }
}

// 1-D bulk copy global -> shared (size and both addresses 16-byte aligned), completing
// `bytes` of transaction count on `bar`.
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}

// Shared-memory loads by 32-bit shared-window address (hoisted base + offsets: no generic-to-shared
// conversion per access inside branchy per-entry code).
__device__ __forceinline__ double lds_f64(uint32_t a) {
    double v;
    asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ void sts_f64(uint32_t a, double v) {
    asm volatile("st.shared.f64 [%0], %1;" ::"r"(a), "d"(v) : "memory");
}

__device__ __forceinline__ int32_t lds_s32(uint32_t a) {
    int32_t v;
    asm volatile("ld.shared.b32 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ uint32_t lds_u8(uint32_t a) {
    uint16_t v;
    asm volatile("ld.shared.u8 %0, [%1];" : "=h"(v) : "r"(a));
    return v;
}

// L2 eviction policies for the streaming kernels (createpolicy; used as .L2::cache_hint operands).
// The matrix slab and b are read once per global iteration and never again within it: evict them
// first, so that L2 keeps the iterate x between the reads of one subdomain's values as its own
// x_J and as its neighbours' ghosts.
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}

// bulk_g2s with an L2 cache-policy hint.
__device__ __forceinline__ void bulk_g2s_hint(void *dst, const void *src, uint32_t bytes, uint64_t *bar,
                                              uint64_t pol) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], "
        "%4;" ::"r"(smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
        : "memory");
}

__device__ __forceinline__ void bulk_prefetch_l2_hint(const void *src, uint32_t bytes, uint64_t pol) {
    asm volatile("cp.async.bulk.prefetch.L2.global.L2::cache_hint [%0], %1, %2;" ::"l"(src), "r"(bytes), "l"(pol)
                 : "memory");
}

// Bulk L2 prefetch (no shared-memory destination, no completion): a hint that brings
// [src, src + bytes) into L2 ahead of the loads that will read it. 16-byte aligned and sized.
__device__ __forceinline__ void bulk_prefetch_l2(const void *src, uint32_t bytes) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(src), "r"(bytes) : "memory");
}

// Prefetch the x ranges of one subdomain's ghost table entry (Layout::gr, kGhostRanges pairs of
// (first column, count) already in shared memory) into L2.
__device__ __forceinline__ void prefetch_ghost_x(const double *x, const int32_t *g, int nranges) {
    for (int r = 0; r < nranges; ++r) {
        const int32_t cnt = g[2 * r + 1];
        if (cnt <= 0) continue;
        const uintptr_t a0 = reinterpret_cast<uintptr_t>(x + g[2 * r]) & ~(uintptr_t)15;
        const uintptr_t a1 = (reinterpret_cast<uintptr_t>(x + g[2 * r] + cnt) + 15) & ~(uintptr_t)15;
        bulk_prefetch_l2(reinterpret_cast<const void *>(a0), (uint32_t)(a1 - a0));
    }
}

}  // namespace bar
