// common.cuh -- shared device helpers of the Betty B200 library (sm_100a).
// Nothing here is shared with oracle/ (the CPU oracle has its own code).
#pragma once
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>

#define BETTY_WARP 32
#define BETTY_NUM_SMS 148

namespace betty {

// ---------------------------------------------------------------- numerics
__device__ __forceinline__ float ld_act(const float* p) { return *p; }
__device__ __forceinline__ float ld_act(const __nv_bfloat16* p) { return __bfloat162float(*p); }
__device__ __forceinline__ void st_act(float* p, float v) { *p = v; }
__device__ __forceinline__ void st_act(__nv_bfloat16* p, float v) { *p = __float2bfloat16_rn(v); }
// 4 consecutive activations in one vector store (p aligned to 4 elements)
__device__ __forceinline__ void st_act4(float* p, const float* v) { *(float4*)p = make_float4(v[0], v[1], v[2], v[3]); }
__device__ __forceinline__ void st_act4(__nv_bfloat16* p, const float* v) {
    __nv_bfloat162 a = __floats2bfloat162_rn(v[0], v[1]), b = __floats2bfloat162_rn(v[2], v[3]);
    *(uint2*)p = make_uint2(*(uint32_t*)&a, *(uint32_t*)&b);
}

// 16-byte vector of activations: 4 fp32 or 8 bf16
template <typename T> struct Vec;
template <> struct Vec<float> {
    static constexpr int N = 4;
    float v[4];
    __device__ __forceinline__ void load(const float* p) {
        float4 t = __ldg(reinterpret_cast<const float4*>(p));
        v[0] = t.x; v[1] = t.y; v[2] = t.z; v[3] = t.w;
    }
    __device__ __forceinline__ void load_cg(const float* p) {   // coherent (buffers written by earlier kernels)
        float4 t = *reinterpret_cast<const float4*>(p);
        v[0] = t.x; v[1] = t.y; v[2] = t.z; v[3] = t.w;
    }
    __device__ __forceinline__ void store(float* p) const {
        *reinterpret_cast<float4*>(p) = make_float4(v[0], v[1], v[2], v[3]);
    }
    // raw 16-byte loads kept packed while in flight (registers), unpacked when summed
    typedef float4 Raw;
    __device__ __forceinline__ static Raw ld_raw(const float* p) { return __ldg(reinterpret_cast<const float4*>(p)); }
    __device__ __forceinline__ static Raw zero_raw() { return make_float4(0.f, 0.f, 0.f, 0.f); }
    __device__ __forceinline__ static void add_raw(float* acc, Raw t) { acc[0] += t.x; acc[1] += t.y; acc[2] += t.z; acc[3] += t.w; }
};
template <> struct Vec<__nv_bfloat16> {
    static constexpr int N = 8;
    float v[8];
    __device__ __forceinline__ void unpack(uint4 t) {
        const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&t);
#pragma unroll
        for (int i = 0; i < 4; ++i) { float2 f = __bfloat1622float2(h[i]); v[2 * i] = f.x; v[2 * i + 1] = f.y; }
    }
    __device__ __forceinline__ void load(const __nv_bfloat16* p) { unpack(__ldg(reinterpret_cast<const uint4*>(p))); }
    __device__ __forceinline__ void load_cg(const __nv_bfloat16* p) { unpack(*reinterpret_cast<const uint4*>(p)); }
    __device__ __forceinline__ void store(__nv_bfloat16* p) const {
        uint4 t;
        __nv_bfloat162* h = reinterpret_cast<__nv_bfloat162*>(&t);
#pragma unroll
        for (int i = 0; i < 4; ++i) h[i] = __floats2bfloat162_rn(v[2 * i], v[2 * i + 1]);
        *reinterpret_cast<uint4*>(p) = t;
    }
    typedef uint4 Raw;
    __device__ __forceinline__ static Raw ld_raw(const __nv_bfloat16* p) { return __ldg(reinterpret_cast<const uint4*>(p)); }
    __device__ __forceinline__ static Raw zero_raw() { return make_uint4(0u, 0u, 0u, 0u); }
    // bf16x2 word -> (lo << 16, hi & 0xffff0000) is the exact fp32 pair; summed with one FADD2
    __device__ __forceinline__ static void add_raw(float* acc, Raw t) {
        const uint32_t w[4] = {t.x, t.y, t.z, t.w};
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            const unsigned long long x = (unsigned long long)(w[i] << 16) | ((unsigned long long)(w[i] & 0xffff0000u) << 32);
            unsigned long long a = (unsigned long long)__float_as_uint(acc[2 * i]) |
                                   ((unsigned long long)__float_as_uint(acc[2 * i + 1]) << 32);
            asm("add.rn.f32x2 %0, %0, %1;" : "+l"(a) : "l"(x));
            acc[2 * i] = __uint_as_float((uint32_t)a);
            acc[2 * i + 1] = __uint_as_float((uint32_t)(a >> 32));
        }
    }
};

__host__ __device__ __forceinline__ int64_t mn64(int64_t a, int64_t b) { return a < b ? a : b; }

// ------------------------------------------------------------ warp / block
__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }
// GPU-scope acquire-release fence for the "last CTA reduces" and flag patterns.  __threadfence() is
// fence.sc.gpu (MEMBAR.SC.GPU), a sequentially-consistent fence that cost the small scans ~10 us each
// (ncu r06: a 7-CTA scan of 28 K elements ran 15 us with 1 K active cycles per SM)
__device__ __forceinline__ void fence_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
__device__ __forceinline__ int warp_id() { return threadIdx.x >> 5; }

// ascending bitonic sort of one int32 per lane across the warp
__device__ __forceinline__ int32_t warp_bitonic32(int32_t x) {
    const int lane = lane_id();
#pragma unroll
    for (int k = 2; k <= 32; k <<= 1) {
#pragma unroll
        for (int j = k >> 1; j > 0; j >>= 1) {
            const int32_t y = __shfl_xor_sync(0xffffffffu, x, j);
            const bool up = ((lane & k) == 0);
            const bool lower = ((lane & j) == 0);
            // lower element keeps min when ascending
            x = (lower == up) ? min(x, y) : max(x, y);
        }
    }
    return x;
}

template <typename T> __device__ __forceinline__ T warp_incl_scan(T v) {
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T n = __shfl_up_sync(0xffffffffu, v, o);
        if (lane_id() >= o) v += n;
    }
    return v;
}
template <typename T> __device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}

// exclusive block scan; smem must hold blockDim.x/32 + 1 elements; returns
// the exclusive prefix, block total in *total.  All threads must call.
template <typename T> __device__ __forceinline__ T block_excl_scan(T v, T* smem, T* total) {
    const int nw = blockDim.x >> 5;
    T inc = warp_incl_scan(v);
    if (lane_id() == 31) smem[warp_id()] = inc;
    __syncthreads();
    if (warp_id() == 0) {
        T w = lane_id() < nw ? smem[lane_id()] : T(0);
        T wi = warp_incl_scan(w);
        if (lane_id() < nw) smem[lane_id()] = wi - w;
        if (lane_id() == nw - 1) smem[nw] = wi;
    }
    __syncthreads();
    T res = inc - v + smem[warp_id()];
    *total = smem[nw];
    __syncthreads();
    return res;
}

// number of CTAs for a persistent grid-stride kernel
inline int persistent_grid(int per_sm = 4) { return BETTY_NUM_SMS * per_sm; }

}  // namespace betty
