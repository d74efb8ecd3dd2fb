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
    if (A == TIGR_SSSP) {
        const uint64_t s = (uint64_t)x + w;
        return s >= kInf ? kInf - 1 : (uint32_t)s;
    }
    if (A == TIGR_CC) return x;
    return x < w ? x : w;  // SSWP
}

}  // namespace tigr
