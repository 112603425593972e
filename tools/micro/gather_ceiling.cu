// Practical HBM ceiling for random feature-row gathers on this GPU (evidence for DESIGN.md §7):
// every warp reads rows whose ids come from a random index array; lanes < row_bytes/16 load one
// 16-byte vector each (cp-free plain LDG.128, 4 rows in flight per warp), sum them and keep a
// checksum.  Table >> L2 and indices uniform, so every row comes from DRAM.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/gc tools/micro/gather_ceiling.cu && /tmp/gc
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void k_gather(const uint4* __restrict__ X, int64_t ld16, const int32_t* __restrict__ idx, int64_t n,
                         int nv, unsigned* out) {
    const int lane = threadIdx.x & 31;
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    unsigned acc = 0;
    for (int64_t r = gw * 4; r < n; r += nw * 4) {
        uint4 v[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            v[k] = make_uint4(0, 0, 0, 0);
            if (r + k < n && lane < nv) v[k] = __ldcs(X + (int64_t)idx[r + k] * ld16 + lane);
        }
#pragma unroll
        for (int k = 0; k < 4; ++k) acc ^= v[k].x ^ v[k].y ^ v[k].z ^ v[k].w;
    }
    if (acc == 0x12345678u) out[0] = acc;
}

int main() {
    const int64_t N = 20000000;            // rows in the table
    const int64_t n = 30000000;            // gathers
    int32_t* idx;
    cudaMalloc(&idx, n * 4);
    int32_t* h = (int32_t*)malloc(n * 4);
    uint64_t s = 88172645463325252ull;
    for (int64_t i = 0; i < n; ++i) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; h[i] = (int32_t)(s % N); }
    cudaMemcpy(idx, h, n * 4, cudaMemcpyHostToDevice);
    unsigned* out;
    cudaMalloc(&out, 4);
    int dev_sms = 0;
    cudaDeviceGetAttribute(&dev_sms, cudaDevAttrMultiProcessorCount, 0);
    for (int row_bytes : {208, 224, 256, 416}) {
        const int64_t ld16 = row_bytes / 16;
        uint4* X;
        if (cudaMalloc(&X, N * ld16 * 16) != cudaSuccess) { printf("alloc failed\n"); return 1; }
        cudaMemset(X, 1, N * ld16 * 16);
        const int nv = (int)ld16;
        for (int blocksPerSm : {8}) {
            const int grid = dev_sms * blocksPerSm;
            k_gather<<<grid, 256>>>(X, ld16, idx, n, nv, out);
            cudaEvent_t a, b;
            cudaEventCreate(&a); cudaEventCreate(&b);
            cudaEventRecord(a);
            const int reps = 5;
            for (int r = 0; r < reps; ++r) k_gather<<<grid, 256>>>(X, ld16, idx, n, nv, out);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms = 0;
            cudaEventElapsedTime(&ms, a, b);
            ms /= reps;
            const double bytes = (double)n * row_bytes + (double)n * 4;
            printf("random %d-byte rows (16-B aligned, %d vectors): %.3f ms  %.0f GB/s (row bytes + index)\n",
                   row_bytes, nv, ms, bytes / ms / 1e6);
        }
        cudaFree(X);
    }
    return 0;
}
