// Gather rate of 208-byte feature rows (C3's bf16 rows) by plain LDG.128 into registers, table
// L2-resident (12.5 MB) or not (0.52 GB, argv[1] = big), random row ids from an index array; one
// warp instruction covers two rows (13 lanes each), 4 row pairs in flight per warp.  Evidence for
// from L2 this reaches ~75 rows/ns chip-wide, ~3x the layer-0 aggregation's rate,
// whose time nevertheless scales with 1 / (SMs used) (profiles/r03_agg_bound.txt); on the real mixed
// workload (45 % of row fetches from DRAM) a register-gather aggregation measured 1.98 ms against
// the TMA pipeline's 1.07 ms, so the pipeline stays.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/gl2 tools/micro/gather_l2.cu && /tmp/gl2 [big]
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

constexpr int ROWB = 208;                 // bytes per row (104 bf16)
constexpr int LD16 = ROWB / 16;           // 13 vectors

__global__ void k_ldg(const uint4* __restrict__ X, const int32_t* __restrict__ idx, int64_t n, unsigned* out) {
    const int lane = threadIdx.x & 31, half = lane >> 4, sub = lane & 15;
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    unsigned acc = 0;
    constexpr int U = 4;                 // row pairs in flight per warp
    for (int64_t r = gw * 2 * U; r < n; r += nw * 2 * U) {
        uint4 v[U];
#pragma unroll
        for (int k = 0; k < U; ++k) {
            const int64_t row = r + 2 * k + half;
            v[k] = make_uint4(0, 0, 0, 0);
            if (row < n && sub < LD16) v[k] = __ldcg(X + (int64_t)idx[row] * LD16 + sub);
        }
#pragma unroll
        for (int k = 0; k < U; ++k) acc ^= v[k].x ^ v[k].y ^ v[k].z ^ v[k].w;
    }
    if (acc == 0x12345678u) out[0] = acc;
}

int main(int argc, char** argv) {
    const int64_t T = argc > 1 ? 2500000 : 60000;     // table rows: 12.5 MB (L2-resident) or 0.52 GB
    const int64_t n = 40000000;                        // gathers
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    void* X;
    cudaMalloc(&X, T * ROWB);
    cudaMemset(X, 1, T * ROWB);
    int32_t* idx;
    cudaMalloc(&idx, n * 4);
    int32_t* h = (int32_t*)malloc(n * 4);
    uint64_t s = 88172645463325252ull;
    for (int64_t i = 0; i < n; ++i) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; h[i] = (int32_t)(s % T); }
    cudaMemcpy(idx, h, n * 4, cudaMemcpyHostToDevice);
    unsigned* out;
    cudaMalloc(&out, 4);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float ms = 0.f;
    for (int per_sm : {4, 8, 16}) {
        for (int rep = 0; rep < 2; ++rep) {
            cudaEventRecord(a);
            k_ldg<<<sms * per_sm, 128>>>((const uint4*)X, idx, n, out);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
        }
        cudaEventElapsedTime(&ms, a, b);
        printf("table %.2f GB  CTAs/SM %2d (128 thr): %.3f ms  %.1f rows/ns  (%.2f TB/s of rows)\n",
               T * ROWB / 1e9, per_sm, ms, n / (ms * 1e6), n * (double)ROWB / (ms * 1e9));
    }
    return 0;
}
