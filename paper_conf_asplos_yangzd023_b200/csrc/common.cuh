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
};

__host__ __device__ __forceinline__ int64_t mn64(int64_t a, int64_t b) { return a < b ? a : b; }

// ------------------------------------------------------------ warp / block
__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ int warp_id() { return threadIdx.x >> 5; }

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
