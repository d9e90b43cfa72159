// device.cuh -- device helpers shared by libphast's kernels (sweep.cu, top.cu, next.cu).
// Internal to libphast.so.
#pragma once
#include <cstdint>

#include "kernels.h"

namespace phast {

// min(a + l, INF) without wrap: min(a, INF - l) + l  (reading R1: labels
// saturate at PHAST_INF, so every label is exactly min(dist, INF))
__device__ __forceinline__ uint32_t sat_add(uint32_t a, uint32_t l) { return min(a, INF - l) + l; }

// k trees are moved as W-wide vectors: one 16-byte lane holds four trees (k >= 4), the
// B200 analogue of "four trees per SSE register" (§IV-B)
template <int K> struct RowT { using T = uint4; static constexpr int W = 4; };
template <> struct RowT<1> { using T = uint32_t; static constexpr int W = 1; };
template <> struct RowT<2> { using T = uint2; static constexpr int W = 2; };

// relax(acc, x, l) = min(acc, sat(x + l)) per tree (§III "if d(v) >
// d(u)+l(u,v), we set d(v) = d(u)+l(u,v)")
__device__ __forceinline__ uint32_t relax(uint32_t acc, uint32_t x, uint32_t l) { return min(acc, sat_add(x, l)); }
__device__ __forceinline__ uint2 relax(uint2 acc, uint2 x, uint32_t l) {
    const uint32_t c = INF - l;
    return make_uint2(min(acc.x, min(x.x, c) + l), min(acc.y, min(x.y, c) + l));
}
__device__ __forceinline__ uint4 relax(uint4 acc, uint4 x, uint32_t l) {
    const uint32_t c = INF - l;
    return make_uint4(min(acc.x, min(x.x, c) + l), min(acc.y, min(x.y, c) + l), min(acc.z, min(x.z, c) + l),
                      min(acc.w, min(x.w, c) + l));
}
// the largest finite label of a vector (0 if none): the diameter's per-thread max (a5)
__device__ __forceinline__ uint32_t fmax_of(uint32_t a) { return a == INF ? 0u : a; }
__device__ __forceinline__ uint32_t fmax_of(uint2 a) { return max(fmax_of(a.x), fmax_of(a.y)); }
__device__ __forceinline__ uint32_t fmax_of(uint4 a) {
    return max(max(fmax_of(a.x), fmax_of(a.y)), max(fmax_of(a.z), fmax_of(a.w)));
}
template <class T> __device__ __forceinline__ T inf_row();
template <> __device__ __forceinline__ uint32_t inf_row<uint32_t>() { return INF; }
template <> __device__ __forceinline__ uint2 inf_row<uint2>() { return make_uint2(INF, INF); }
template <> __device__ __forceinline__ uint4 inf_row<uint4>() { return make_uint4(INF, INF, INF, INF); }
// two adjacent 16-byte lanes (eight trees) handled by one thread (band kernel variant)
struct alignas(16) U8 {
    uint4 a, b;
};
template <> __device__ __forceinline__ U8 inf_row<U8>() { return U8{inf_row<uint4>(), inf_row<uint4>()}; }
__device__ __forceinline__ U8 relax(U8 acc, U8 x, uint32_t l) { return U8{relax(acc.a, x.a, l), relax(acc.b, x.b, l)}; }
__device__ __forceinline__ uint32_t fmax_of(U8 x) { return max(fmax_of(x.a), fmax_of(x.b)); }
// a row whose every tree holds x (the no-gather probe A34)
template <class T> __device__ __forceinline__ T splat(uint32_t x);
template <> __device__ __forceinline__ uint32_t splat<uint32_t>(uint32_t x) { return x; }
template <> __device__ __forceinline__ uint2 splat<uint2>(uint32_t x) { return make_uint2(x, x); }
template <> __device__ __forceinline__ uint4 splat<uint4>(uint32_t x) { return make_uint4(x, x, x, x); }

__device__ __forceinline__ uint32_t warp_min(uint32_t a) { return __reduce_min_sync(0xFFFFFFFFu, a); }
__device__ __forceinline__ uint2 warp_min(uint2 a) { return make_uint2(warp_min(a.x), warp_min(a.y)); }
__device__ __forceinline__ uint4 warp_min(uint4 a) {
    return make_uint4(warp_min(a.x), warp_min(a.y), warp_min(a.z), warp_min(a.w));
}

// visited bit of v in a slot's bitmap (§IV-C "we mark vertices visited
// during the CH search with a single bit")
__device__ __forceinline__ bool visited(const uint32_t* __restrict__ flags, uint32_t v) {
    return (__ldg(&flags[v >> 5]) >> (v & 31)) & 1u;
}

// per-CTA max, then one atomicMax into *diam (a5, §VII-B "making each core
// keep track of the maximum label it encounters"); every thread of the CTA must call it
template <int THREADS>
__device__ __forceinline__ void cta_max_to(uint32_t mx, uint32_t* diam) {
    __shared__ uint32_t wmax[THREADS / 32];
    mx = __reduce_max_sync(0xFFFFFFFFu, mx);
    if ((threadIdx.x & 31) == 0) wmax[threadIdx.x >> 5] = mx;
    __syncthreads();
    if (threadIdx.x < 32) {
        uint32_t w = threadIdx.x < THREADS / 32 ? wmax[threadIdx.x] : 0u;
        w = __reduce_max_sync(0xFFFFFFFFu, w);
        if (threadIdx.x == 0 && w) atomicMax(diam, w);
    }
}

// shared memory / async copy / mbarrier primitives (sm_90+ PTX, valid on sm_100a)
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }
__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(smem)), "l"(gmem) : "memory");
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t phase) {
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
        "@!P1 bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(bar)),
        "r"(phase)
        : "memory");
}

// dispatch a runtime k in {1, 2, 4, ..., 64} to a template instance
#define PHAST_K_SWITCH(k, CALL)                \
    switch (k) {                               \
        case 1: return CALL(1);                \
        case 2: return CALL(2);                \
        case 4: return CALL(4);                \
        case 8: return CALL(8);                \
        case 16: return CALL(16);              \
        case 32: return CALL(32);              \
        case 64: return CALL(64);              \
        default: return cudaErrorInvalidValue; \
    }

}  // namespace phast
