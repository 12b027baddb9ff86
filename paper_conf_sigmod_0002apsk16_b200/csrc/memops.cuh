// Cache-policy-tagged global memory operations for sm_100a.
//
// Topology pages and the read-only attribute vector are streamed once per
// sweep: they are loaded with an L2 evict_first policy (and no L1 allocation)
// so they do not push the randomly-updated write attribute vector (acc /
// labels / bitmaps) out of the 126 MB L2.
#pragma once

#include <cstdint>

namespace gts {

__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}

__device__ __forceinline__ uint4 ld_stream_v4(const void* p, uint64_t pol) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "l"(p), "l"(pol));
    return r;
}

__device__ __forceinline__ uint32_t ld_stream_u32(const void* p, uint64_t pol) {
    uint32_t r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol));
    return r;
}

// L1-allocating variant: for small strided loads that re-touch the same sectors
__device__ __forceinline__ uint32_t ld_stream_l1_u32(const void* p, uint64_t pol) {
    uint32_t r;
    asm volatile("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol));
    return r;
}

// L1-allocating 8-byte variant (weighted (neighbour, weight) pairs of a gathered record)
__device__ __forceinline__ uint2 ld_stream_l1_v2(const void* p, uint64_t pol) {
    uint2 r;
    asm volatile("ld.global.nc.L2::cache_hint.v2.u32 {%0,%1}, [%2], %3;" : "=r"(r.x), "=r"(r.y) : "l"(p), "l"(pol));
    return r;
}

__device__ __forceinline__ uint2 ld_stream_v2(const void* p, uint64_t pol) {
    uint2 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.u32 {%0,%1}, [%2], %3;"
                 : "=r"(r.x), "=r"(r.y)
                 : "l"(p), "l"(pol));
    return r;
}

__device__ __forceinline__ float ld_stream_f32(const float* p, uint64_t pol) {
    return __uint_as_float(ld_stream_u32(p, pol));
}

__device__ __forceinline__ uint32_t word_of(const uint4& v, int k) {
    return k == 0 ? v.x : k == 1 ? v.y : k == 2 ? v.z : v.w;
}

// out[v] = f(idx[v]) for v < n, where f is a random read (the caller-order
// gathers of the results of degree-ordered graphs).  Four consecutive outputs
// per thread per step: one 16-byte streaming load of idx, four independent
// random reads in flight, one 16-byte streaming store.  A one-element-per-step
// loop kept a single random read in flight per thread and ran at ~55% of the
// L2 gather rate (tools/bfs_timeline.py).  Falls back to the scalar loop when
// out or idx is not 16-byte aligned.
template <class F>
__device__ __forceinline__ void gather_x4(uint32_t* out, const uint32_t* __restrict__ idx, uint64_t n, F f) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    const uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if ((((uintptr_t)out | (uintptr_t)idx) & 15u) != 0) {
        for (uint64_t v = t; v < n; v += stride) out[v] = f(idx[v]);
        return;
    }
    const uint64_t n4 = n >> 2;
    const uint4* idx4 = reinterpret_cast<const uint4*>(idx);
    uint4* out4 = reinterpret_cast<uint4*>(out);
    // two 16-byte index loads, then eight random reads, in flight per thread
    uint64_t q = t;
    for (; q + stride < n4; q += 2 * stride) {
        const uint4 i = __ldcs(idx4 + q), j = __ldcs(idx4 + q + stride);
        uint4 o, p;
        o.x = f(i.x);
        o.y = f(i.y);
        o.z = f(i.z);
        o.w = f(i.w);
        p.x = f(j.x);
        p.y = f(j.y);
        p.z = f(j.z);
        p.w = f(j.w);
        __stcs(out4 + q, o);
        __stcs(out4 + q + stride, p);
    }
    if (q < n4) {
        const uint4 i = __ldcs(idx4 + q);
        uint4 o;
        o.x = f(i.x);
        o.y = f(i.y);
        o.z = f(i.z);
        o.w = f(i.w);
        __stcs(out4 + q, o);
    }
    if (t < (n & 3u)) out[4 * n4 + t] = f(idx[4 * n4 + t]);
}

}  // namespace gts
