// devutil.cuh -- device helpers shared by the relax kernels (internal).
#pragma once

#include <stdint.h>

#include "internal.cuh"

namespace tigr {

// Read-only streaming loads (edge / weight chunks): not allocated in L1, and marked
// evict-first in L2 so that the 1+ GB edge stream does not push the value / accumulator
// arrays out of the 126 MB L2.  Not volatile: the compiler may hoist them.
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}

__device__ __forceinline__ uint64_t policy_evict_last() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}

__device__ __forceinline__ uint4 ldg_chunk(const uint4* p) {
    uint4 r;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
        : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p), "l"(policy_evict_first()));
    return r;
}

// 32 bytes at a 32-byte-aligned address as ONE 256-bit load (LDG.E.256 on sm_100): a lane's
// whole span is one L1 sector access instead of two 16-byte requests
__device__ __forceinline__ void ldg_span(const uint4* p, uint4& a, uint4& b) {
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
        : "=r"(a.x), "=r"(a.y), "=r"(a.z), "=r"(a.w), "=r"(b.x), "=r"(b.y), "=r"(b.z), "=r"(b.w)
        : "l"(p), "l"(policy_evict_first()));
}

// ---- the edge units of one virtual node ----------------------------------------
// A node's segment starts at 16-byte chunk cb (span-aligned, padded with kPad); its arcs are
// grouped into units of U: U = 8 (one 32-byte span, 8 | K), U = 4 (one 16-byte chunk, 4 | K).
// Virtual node jj of the family owns units k, k + step, ... < kend: strided (Fig. 12 / Alg. 3)
// k = jj, step = m_v; consecutive (Fig. 10 / Alg. 2) the K / U units from jj * K / U.
template <int U, int LAYOUT>
__device__ __forceinline__ void unit_range(uint32_t d, uint32_t jj, uint32_t mv, uint32_t K, uint32_t& k,
                                           uint32_t& step, uint32_t& kend) {
    const uint32_t q = (d + U - 1) / U;
    if (LAYOUT == TIGR_LAYOUT_STRIDED) {
        k = jj; step = mv; kend = q;
    } else {
        const uint32_t per = (K == 0xFFFFFFFFu) ? 0xFFFFFFFFu : K / U;
        k = jj * per; step = 1;
        kend = (per >= q - k) ? q : k + per;
    }
}

// one batch of 8 slots starting at unit k: U = 8 the span k; U = 4 the chunks k and k + step
// (absent units read as `pad`); returns the first unit of the next batch
template <int U>
__device__ __forceinline__ uint32_t load8(const uint4* __restrict__ p, uint32_t cb, uint32_t k, uint32_t step,
                                          uint32_t kend, uint4& a, uint4& b, uint4 pad) {
    if (U == 8) {
        if (k < kend) ldg_span(p + cb + 2 * k, a, b);
        else a = b = pad;
        return k + step;
    }
    a = k < kend ? ldg_chunk(p + cb + k) : pad;
    b = k + step < kend ? ldg_chunk(p + cb + k + step) : pad;
    return k + 2 * step;
}

__device__ __forceinline__ uint32_t ldg_u32(const uint32_t* p) {
    uint32_t r;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(policy_evict_first()));
    return r;
}

// fire-and-forget float64 add into the accumulator, kept resident in L2 (evict-last)
__device__ __forceinline__ void red_add_f64(double* p, double v, uint64_t pol) {
    asm volatile("red.global.add.L2::cache_hint.f64 [%0], %1, %2;" :: "l"(p), "d"(v), "l"(pol) : "memory");
}

// relax semantics per algorithm (Alg. 2/3 line 5-6): candidate value and the improvement test
template <int A>
__device__ __forceinline__ bool better(uint32_t alt, uint32_t cur) {
    return A == TIGR_SSWP ? alt > cur : alt < cur;
}

template <int A>
__device__ __forceinline__ uint32_t combine(uint32_t x, uint32_t w) {
    if (A == TIGR_BFS) return x + 1;
    if (A == TIGR_SSSP) {  // saturating: x + w >= 2^32 - 1 (infinity) gives 2^32 - 2
        const uint32_t s = x + w;
        return (s < x || s == kInf) ? kInf - 1 : s;
    }
    if (A == TIGR_CC) return x;
    return x < w ? x : w;  // SSWP
}

}  // namespace tigr
