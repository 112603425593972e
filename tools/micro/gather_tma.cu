// Rate of TMA tile::gather4 for 208-byte rows (C3's bf16 feature rows): evidence for DESIGN.md §7 /
// profiles/r03_agg_bound.txt.  k_tma: warp 0's lanes each issue one gather4 per stage (4 rows, ids
// from a hash, no index loads; per-lane coordinates make the compiler loop R2UR -> UTMALDG over the
// lanes), warp 1 waits for each stage and releases it.  k_tma_mw: PW producer warps each issue ONE
// gather4 per stage with warp-uniform coordinates.  No arithmetic, no stores.  Table L2-resident
// (13.6 MB) or not (0.87 GB, argv[1] = big); argv[2] = row bytes.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/gt tools/micro/gather_tma.cu && /tmp/gt [big]
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda.h>
#include <cuda_runtime.h>

int ROWB_H = 208;                          // row bytes (argv[2], default 208)
constexpr int STAGES = 16, G4_PER_STAGE = 8;          // 32 rows per stage, 512 rows in flight per CTA

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, int c) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(b)), "r"(c) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t ph) {
    asm volatile("{\n.reg .pred p;\nW: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W;\n}\n"
                 ::"r"(su32(b)), "r"(ph) : "memory");
}
__device__ __forceinline__ void gather4(uint32_t dst, const CUtensorMap* tm, int r0, int r1, int r2, int r3,
                                        uint64_t* bar) {
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
                 " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                 ::"r"(dst), "l"((uint64_t)tm), "r"(0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(su32(bar))
                 : "memory");
}
__device__ __forceinline__ int rid(uint32_t r, uint32_t mask) {
    uint32_t x = r * 0x9E3779B1u;                // murmur-style finaliser: scattered ids
    x ^= x >> 16; x *= 0x85EBCA6Bu; x ^= x >> 13;
    return (int)(x & mask);
}

__global__ void __launch_bounds__(64, 1) k_tma(const __grid_constant__ CUtensorMap tm, uint32_t mask, int64_t n,
                                               uint32_t rowb) {
    extern __shared__ __align__(1024) uint8_t sm[];
    uint64_t* full = (uint64_t*)sm;
    uint64_t* empty = full + STAGES;
    uint8_t* data = sm + 1024;
    constexpr uint32_t stage_bytes = G4_PER_STAGE * 1024;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const int64_t rows_per_stage = G4_PER_STAGE * 4;
    const int64_t nst = n / rows_per_stage;
    int s = 0;
    uint32_t ph = 0;
    if (warp == 0) {
        for (int64_t st = blockIdx.x; st < nst; st += gridDim.x) {
            mbar_wait(&empty[s], ph ^ 1);
            if (lane == 0) mbar_expect_tx(&full[s], G4_PER_STAGE * 4 * rowb);
            __syncwarp();
            if (lane < G4_PER_STAGE) {               // one gather4 per lane
                const uint32_t r = (uint32_t)(st * rows_per_stage + 4 * lane);
                gather4(su32(data + s * stage_bytes + lane * 1024), &tm, rid(r, mask), rid(r + 1, mask),
                        rid(r + 2, mask), rid(r + 3, mask), &full[s]);
            }
            if (++s == STAGES) { s = 0; ph ^= 1; }
        }
    } else {
        for (int64_t st = blockIdx.x; st < nst; st += gridDim.x) {
            mbar_wait(&full[s], ph);
            if (lane == 0) mbar_arrive(&empty[s]);
            __syncwarp();
            if (++s == STAGES) { s = 0; ph ^= 1; }
        }
    }
}

// PW producer warps, each issuing ONE gather4 per stage with warp-uniform coordinates (no per-lane
// R2UR loop), one consumer warp; full barrier expects the stage's bytes, empty barrier 1 arrival
template <int PW, int STAGES>
__global__ void __launch_bounds__(32 * (PW + 1), 1) k_tma_mw(const __grid_constant__ CUtensorMap tm, uint32_t mask,
                                                               int64_t n, uint32_t rowb) {
    extern __shared__ __align__(1024) uint8_t sm[];
    uint64_t* full = (uint64_t*)sm;
    uint64_t* empty = full + STAGES;
    uint8_t* data = sm + 1024;
    constexpr uint32_t stage_bytes = PW * 1024;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s) { mbar_init(&full[s], PW); mbar_init(&empty[s], 1); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const int64_t rows_per_stage = PW * 4;
    const int64_t nst = n / rows_per_stage;
    int s = 0;
    uint32_t ph = 0;
    if (warp < PW) {
        for (int64_t st = blockIdx.x; st < nst; st += gridDim.x) {
            mbar_wait(&empty[s], ph ^ 1);
            if (lane == 0) {
                mbar_expect_tx(&full[s], 4 * rowb);
                const uint32_t r = (uint32_t)(st * rows_per_stage + 4 * warp);
                gather4(su32(data + s * stage_bytes + warp * 1024), &tm, rid(r, mask), rid(r + 1, mask),
                        rid(r + 2, mask), rid(r + 3, mask), &full[s]);
            }
            __syncwarp();
            if (++s == STAGES) { s = 0; ph ^= 1; }
        }
    } else {
        for (int64_t st = blockIdx.x; st < nst; st += gridDim.x) {
            mbar_wait(&full[s], ph);
            if (lane == 0) mbar_arrive(&empty[s]);
            __syncwarp();
            if (++s == STAGES) { s = 0; ph ^= 1; }
        }
    }
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                             const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                             CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main(int argc, char** argv) {
    const int64_t T = argc > 1 && argv[1][0] == 'b' ? (1 << 22) : (1 << 16);
    const int ROWB = argc > 2 ? atoi(argv[2]) : ROWB_H;        // <= 256 (a 4-row group fits a 1024-B slot)
    const int64_t n = 40000000;
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    void* X;
    cudaMalloc(&X, T * ROWB);
    cudaMemset(X, 1, T * ROWB);
    EncodeFn enc = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q);
    CUtensorMap tm;
    cuuint64_t dims[2] = {(cuuint64_t)(ROWB / 2), (cuuint64_t)T};
    cuuint64_t strides[1] = {(cuuint64_t)ROWB};
    cuuint32_t box[2] = {(cuuint32_t)(ROWB / 2), 1};
    cuuint32_t estr[2] = {1, 1};
    if (enc(&tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, X, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
            CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
        printf("encode failed\n");
        return 1;
    }
    const int smem = 1024 + STAGES * G4_PER_STAGE * 1024;
    cudaFuncSetAttribute(k_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float ms = 0.f;
    {
        const int sm8 = 1024 + 16 * 8 * 1024, sm16 = 1024 + 8 * 16 * 1024, sm4 = 1024 + 16 * 4 * 1024;
        cudaFuncSetAttribute(k_tma_mw<8, 16>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm8);
        cudaFuncSetAttribute(k_tma_mw<16, 8>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm16);
        cudaFuncSetAttribute(k_tma_mw<4, 16>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm4);
        for (int pw : {4, 8, 16}) {
            for (int rep = 0; rep < 2; ++rep) {
                cudaEventRecord(a);
                if (pw == 4) k_tma_mw<4, 16><<<sms, 32 * 5, sm4>>>(tm, (uint32_t)(T - 1), n, (uint32_t)ROWB);
                else if (pw == 8) k_tma_mw<8, 16><<<sms, 32 * 9, sm8>>>(tm, (uint32_t)(T - 1), n, (uint32_t)ROWB);
                else k_tma_mw<16, 8><<<sms, 32 * 17, sm16>>>(tm, (uint32_t)(T - 1), n, (uint32_t)ROWB);
                cudaEventRecord(b);
                cudaEventSynchronize(b);
            }
            cudaError_t e = cudaGetLastError();
            cudaEventElapsedTime(&ms, a, b);
            printf("row %d B  table %.2f GB  %2d producer warps x 1 gather4: %.3f ms  %.1f rows/ns  %s\n", ROWB,
                   T * ROWB / 1e9, pw, ms, n / (ms * 1e6), e ? cudaGetErrorString(e) : "");
        }
    }
    for (int ctas : {1, 2, 4}) {
        for (int used : {sms, sms / 2}) {
            for (int rep = 0; rep < 2; ++rep) {
                cudaEventRecord(a);
                k_tma<<<used * ctas, 64, smem>>>(tm, (uint32_t)(T - 1), n, (uint32_t)ROWB);
                cudaEventRecord(b);
                cudaEventSynchronize(b);
            }
            cudaError_t e = cudaGetLastError();
            cudaEventElapsedTime(&ms, a, b);
            printf("row %d B  table %.2f GB  grid %3d x %d CTAs: %.3f ms  %.1f rows/ns  %.3f rows/ns per grid/%d  %s\n",
                   ROWB, T * ROWB / 1e9, used, ctas, ms, n / (ms * 1e6), n / (ms * 1e6) / used, ctas,
                   e ? cudaGetErrorString(e) : "");
        }
    }
    return 0;
}
