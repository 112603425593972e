// gemm_tc.cu -- the dense SAGE layers on the 5th-generation tensor cores
// (tcgen05.mma kind::f16, bf16 operands, fp32 accumulation in TMEM), BF16
// mode.  Hand-written PTX: TMA (cp.async.bulk.tensor, 128B swizzle) fills a
// multi-stage shared-memory ring, one elected thread issues tcgen05.mma into
// TMEM, four epilogue warps drain TMEM with tcgen05.ld and apply the fused
// epilogue.  Warp roles (192 threads, 1 CTA / SM, persistent):
//   warp 0: TMA producer   warp 1: TMEM allocator + MMA issuer   warps 2-5: epilogue
//
//   k_tc_row : C[M x N] = A[M x K] B[K x N]   (A, B K-major; M on the device)
//              epilogues: store / ReLU + ones column / ReLU' mask / residual + mask
//              two TMEM accumulators so the epilogue of tile i overlaps the MMAs of tile i+1
//   k_tc_red : P[K1 x N] = A^T B over the node dimension (dW), A and B MN-major
//              (node rows contiguous in features), a fixed row range per CTA
//              accumulated in TMEM, partials reduced deterministically by
//              k_red_final (gemm.cu) into the flat gradient.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>
#include "common.cuh"
#include "internal.h"
#include "sage.h"

namespace betty {
namespace tc {

constexpr int BM = 128;            // UMMA M (cta_group::1)
constexpr int BK = 64;             // 64 bf16 = 128 B = one SW128 atom row
constexpr int UK = 16;             // UMMA K for kind::f16
constexpr int THREADS = 192;

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t n) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(b)), "r"(n) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(b)) : "memory");
}
__device__ __forceinline__ bool mbar_try(uint64_t* b, uint32_t parity) {
    uint32_t ok;
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(ok) : "r"(su32(b)), "r"(parity) : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
    while (!mbar_try(b, parity)) {}
}
__device__ __forceinline__ void tma_2d(void* dst, const CUtensorMap* tm, int c0, int c1, uint64_t* bar) {
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                 ::"r"(su32(dst)), "l"((uint64_t)tm), "r"(c0), "r"(c1), "r"(su32(bar)) : "memory");
}
__device__ __forceinline__ void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void umma_commit(uint64_t* b) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(b)) : "memory");
}
__device__ __forceinline__ void umma_f16(uint32_t tmem_d, uint64_t ad, uint64_t bd, uint32_t idesc, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}"
                 ::"r"(tmem_d), "l"(ad), "l"(bd), "r"(idesc), "r"(acc));
}
// shared-memory matrix descriptor, SWIZZLE_128B, sm_100 version 1
__device__ __forceinline__ uint64_t sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    uint64_t d = (uint64_t)((saddr >> 4) & 0x3FFF);
    d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
    d |= (uint64_t)1 << 46;
    d |= (uint64_t)2 << 61;
    return d;
}
// instruction descriptor: bf16 x bf16 -> f32, M x N, operand majors (0 = K, 1 = MN)
__host__ __device__ constexpr uint32_t idesc_bf16(int M, int N, int a_mn, int b_mn) {
    return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)a_mn << 15) | ((uint32_t)b_mn << 16) |
           ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, float* v) {
    uint32_t r[32];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
                 "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                   "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]),
                   "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]),
                   "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]),
                   "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
                 : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
}
__device__ __forceinline__ uint32_t tmem_alloc_warp(uint32_t* slot, uint32_t ncols) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(su32(slot)), "r"(ncols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    return 0;
}
__device__ __forceinline__ void tmem_free_warp(uint32_t taddr, uint32_t ncols) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
}
__device__ __forceinline__ bool elect_lane0() { return (threadIdx.x & 31) == 0; }

// --------------------------------------------------------------- row GEMM
// B (the weights, <= 256 x K) stays resident in shared memory for the whole
// persistent CTA; only A tiles stream through the TMA ring.  Eight epilogue
// warps: warp w drains TMEM lanes 32*(w%4).. (tile rows) for one half of the
// columns; each thread owns one output row and writes 16-byte vectors, with
// the next chunk's TMEM load (and mask load) issued before the current chunk
// is processed.
constexpr int ROW_THREADS = 64 + 256;
struct RowArgs {
    const int64_t* M_dev;
    int K, N, BN, nk, stages;
    void* C; int64_t ldc; int c_bf16;
    int epi;
    const void* mask; int64_t ldm; int m_bf16;
    const float* res; int64_t ldr; const int64_t* nres_dev;
    uint32_t tmem_cols;
    int half_cols;           // columns per epilogue half (multiple of 32)
};

__device__ __forceinline__ uint32_t pack_bf16x2(float a, float b) {
    __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
    return *(uint32_t*)&h;
}

// one 32-column chunk of one row: epilogue math + vector stores
__device__ __forceinline__ void row_chunk_out(const RowArgs& p, float* v, int64_t m, int c0, const uint4* mk,
                                              int64_t nres) {
    const int nval = min(32, p.N - c0);            // valid output columns in this chunk
    if (nval <= 0) return;
#pragma unroll
    for (int j = 0; j < 32; ++j) {
        float x = v[j];
        if (p.epi == EPI_RELU_ONES) x = fmaxf(x, 0.f);
        if (p.epi == EPI_RES_MASK && m < nres && j < nval) x += p.res[m * p.ldr + c0 + j];
        if (p.epi == EPI_MASK || p.epi == EPI_RES_MASK) {
            float mv;
            if (p.m_bf16) {
                const __nv_bfloat16* hb = (const __nv_bfloat16*)&mk[j / 8];
                mv = __bfloat162float(hb[j % 8]);
            } else {
                mv = ((const float*)&mk[j / 4])[j % 4];
            }
            if (!(mv > 0.f)) x = 0.f;
        }
        v[j] = x;
    }
    if (p.c_bf16) {
        __nv_bfloat16* cp = (__nv_bfloat16*)p.C + m * p.ldc + c0;
        if (nval == 32 && (p.ldc & 7) == 0) {
#pragma unroll
            for (int q = 0; q < 4; ++q)
                ((uint4*)cp)[q] = make_uint4(pack_bf16x2(v[8 * q], v[8 * q + 1]), pack_bf16x2(v[8 * q + 2], v[8 * q + 3]),
                                             pack_bf16x2(v[8 * q + 4], v[8 * q + 5]),
                                             pack_bf16x2(v[8 * q + 6], v[8 * q + 7]));
        } else {
#pragma unroll
            for (int j = 0; j < 32; ++j)
                if (j < nval) cp[j] = __float2bfloat16_rn(v[j]);
        }
    } else {
        float* cp = (float*)p.C + m * p.ldc + c0;
        if (nval == 32 && (p.ldc & 3) == 0) {
#pragma unroll
            for (int q = 0; q < 8; ++q) ((float4*)cp)[q] = make_float4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
        } else {
#pragma unroll
            for (int j = 0; j < 32; ++j)
                if (j < nval) cp[j] = v[j];
        }
    }
}

__device__ __forceinline__ void load_mask_chunk(const RowArgs& p, int64_t m, int c0, bool ok, uint4* mk) {
    const int nv = p.m_bf16 ? 4 : 8;                // 16-byte vectors per 32 columns
    if (!ok) return;
    const char* base = (const char*)p.mask + (m * p.ldm + c0) * (p.m_bf16 ? 2 : 4);
    const int64_t rowbytes = (int64_t)(p.N - c0) * (p.m_bf16 ? 2 : 4);
#pragma unroll
    for (int q = 0; q < 8; ++q)
        if (q < nv && q * 16 < rowbytes) mk[q] = __ldg((const uint4*)(base + q * 16));
}

__global__ void __launch_bounds__(ROW_THREADS, 1) k_tc_row(const __grid_constant__ CUtensorMap tmA,
                                                           const __grid_constant__ CUtensorMap tmB, RowArgs p) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    const int S = p.stages;
    const uint32_t a_bytes = BM * BK * 2;
    const uint32_t bblk = (uint32_t)p.BN * BK * 2;          // one K-block of the resident B
    uint8_t* bres = smem;                                    // nk * bblk
    uint8_t* aring = smem + p.nk * bblk;                     // S * a_bytes
    uint64_t* full = (uint64_t*)(aring + S * a_bytes);
    uint64_t* empty = full + S;
    uint64_t* tfull = empty + S;      // [2]
    uint64_t* tempty = tfull + 2;     // [2]
    uint64_t* bfull = tempty + 2;     // [1]
    uint32_t* tslot = (uint32_t*)(bfull + 1);

    const int warp = threadIdx.x >> 5;
    const int64_t M = *p.M_dev;
    const int64_t tiles = (M + BM - 1) / BM;

    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
        for (int a = 0; a < 2; ++a) { mbar_init(&tfull[a], 1); mbar_init(&tempty[a], 256); }
        mbar_init(bfull, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmA) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmB) : "memory");
    }
    if (warp == 1) tmem_alloc_warp(tslot, p.tmem_cols);
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tmem = *tslot;

    if (warp == 0) {
        if (elect_lane0() && blockIdx.x < tiles) {
            mbar_expect_tx(bfull, p.nk * bblk);
            for (int kb = 0; kb < p.nk; ++kb) tma_2d(bres + kb * bblk, &tmB, kb * BK, 0, bfull);
            int s = 0;
            uint32_t ph = 0;
            for (int64_t t = blockIdx.x; t < tiles; t += gridDim.x) {
                for (int kb = 0; kb < p.nk; ++kb) {
                    mbar_wait(&empty[s], ph ^ 1);
                    mbar_expect_tx(&full[s], a_bytes);
                    tma_2d(aring + s * a_bytes, &tmA, kb * BK, (int)(t * BM), &full[s]);
                    if (++s == S) { s = 0; ph ^= 1; }
                }
            }
        }
    } else if (warp == 1) {
        const uint32_t idesc = idesc_bf16(BM, p.BN, 0, 0);
        int s = 0;
        uint32_t ph = 0;
        int it = 0;
        if (blockIdx.x < tiles) mbar_wait(bfull, 0);
        for (int64_t t = blockIdx.x; t < tiles; t += gridDim.x, ++it) {
            const int acc = it & 1;
            const uint32_t aph = (it >> 1) & 1;
            mbar_wait(&tempty[acc], aph ^ 1);
            fence_after();
            const uint32_t d = tmem + acc * p.BN;
            for (int kb = 0; kb < p.nk; ++kb) {
                mbar_wait(&full[s], ph);
                fence_after();
                if (elect_lane0()) {
                    const uint32_t a0 = su32(aring + s * a_bytes), b0 = su32(bres + kb * bblk);
#pragma unroll
                    for (int k = 0; k < BK / UK; ++k) {
                        const uint64_t ad = sdesc(a0 + k * UK * 2, 0, 1024);
                        const uint64_t bd = sdesc(b0 + k * UK * 2, 0, 1024);
                        umma_f16(d, ad, bd, idesc, (kb | k) != 0);
                    }
                    umma_commit(&empty[s]);
                    if (kb == p.nk - 1) umma_commit(&tfull[acc]);
                }
                __syncwarp();
                if (++s == S) { s = 0; ph ^= 1; }
            }
        }
    } else {
        const int ew = warp - 2;                 // 0..7
        const int q = warp & 3;                  // TMEM lane quadrant (hardware: warp id % 4)
        const int h = ew >> 2;                   // column half
        const int lane = threadIdx.x & 31;
        const int cbeg = h * p.half_cols;
        const int cend = min(p.BN, cbeg + p.half_cols);
        const bool has_mask = p.epi == EPI_MASK || p.epi == EPI_RES_MASK;
        const int64_t nres = (p.epi == EPI_RES_MASK) ? *p.nres_dev : 0;
        int it = 0;
        for (int64_t t = blockIdx.x; t < tiles; t += gridDim.x, ++it) {
            const int acc = it & 1;
            const uint32_t aph = (it >> 1) & 1;
            const int64_t m = t * BM + q * 32 + lane;
            const bool ok = m < M;
            uint4 mk[8], mk_next[8];
            if (has_mask && cbeg < cend) load_mask_chunk(p, m, cbeg, ok, mk);
            mbar_wait(&tfull[acc], aph);
            fence_after();
            const uint32_t tbase = tmem + ((uint32_t)(q * 32) << 16) + acc * p.BN;
            float v[32];
            if (cbeg < cend) tmem_ld32(tbase + cbeg, v);
            for (int c0 = cbeg; c0 < cend; c0 += 32) {
                const bool more = c0 + 32 < cend;
                float nx[32];
                if (more) {
                    // next chunk's TMEM load in flight while this chunk is stored
                    uint32_t r[32];
                    asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,"
                                 "%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
                                   "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]),
                                   "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]),
                                   "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]),
                                   "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]),
                                   "=r"(r[31])
                                 : "r"(tbase + c0 + 32));
#pragma unroll
                    for (int j = 0; j < 32; ++j) nx[j] = __uint_as_float(r[j]);
                    if (has_mask) load_mask_chunk(p, m, c0 + 32, ok, mk_next);
                }
                if (ok) row_chunk_out(p, v, m, c0, mk, nres);
                if (more) {
                    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
                    for (int j = 0; j < 32; ++j) v[j] = nx[j];
#pragma unroll
                    for (int q2 = 0; q2 < 8; ++q2) mk[q2] = mk_next[q2];
                }
            }
            fence_before();
            mbar_arrive(&tempty[acc]);
            // trailing columns [N, ldc): the ones column after a ReLU layer, zeros elsewhere
            if (h == 1 && ok && p.ldc > p.N) {
                for (int col = p.N; col < p.ldc; ++col) {
                    const float x = (p.epi == EPI_RELU_ONES && col == p.N) ? 1.f : 0.f;
                    if (p.c_bf16) ((__nv_bfloat16*)p.C)[m * p.ldc + col] = __float2bfloat16_rn(x);
                    else ((float*)p.C)[m * p.ldc + col] = x;
                }
            }
        }
    }
    __syncthreads();
    if (warp == 1) {
        fence_after();
        tmem_free_warp(tmem, p.tmem_cols);
    }
}

// ---------------------------------------------------------- reduction GEMM
struct RedArgs {
    const int64_t* M_dev;      // rows (the reduction dimension)
    int K1, N, BN, nbA, nbB, stages, S, mtiles;
    float* partials;           // [S][K1][N]
    uint32_t tmem_cols;
};

__global__ void __launch_bounds__(THREADS, 1) k_tc_red(const __grid_constant__ CUtensorMap tmA,
                                                       const __grid_constant__ CUtensorMap tmB, RedArgs p) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    const int S = p.stages;
    const uint32_t box = BK * 128;                    // 64 rows x 128 B
    const uint32_t a_bytes = p.nbA * box, b_bytes = p.nbB * box;
    const uint32_t stage_bytes = a_bytes + b_bytes;
    uint64_t* full = (uint64_t*)(smem + S * stage_bytes);
    uint64_t* empty = full + S;
    uint64_t* tfull = empty + S;
    uint32_t* tslot = (uint32_t*)(tfull + 1);

    const int warp = threadIdx.x >> 5;
    const int mt = blockIdx.x % p.mtiles, split = blockIdx.x / p.mtiles;
    const int64_t M = *p.M_dev;
    const int64_t nkb = (M + BK - 1) / BK;
    const int64_t kb0 = nkb * split / p.S, kb1 = nkb * (split + 1) / p.S;

    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
        mbar_init(&tfull[0], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 1) tmem_alloc_warp(tslot, p.tmem_cols);
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tmem = *tslot;

    if (warp == 0) {
        if (elect_lane0()) {
            int s = 0;
            uint32_t ph = 0;
            for (int64_t kb = kb0; kb < kb1; ++kb) {
                mbar_wait(&empty[s], ph ^ 1);
                uint8_t* sa = smem + s * stage_bytes;
                mbar_expect_tx(&full[s], stage_bytes);
                for (int i = 0; i < p.nbA; ++i) tma_2d(sa + i * box, &tmA, mt * BM + i * 64, (int)(kb * BK), &full[s]);
                for (int i = 0; i < p.nbB; ++i) tma_2d(sa + a_bytes + i * box, &tmB, i * 64, (int)(kb * BK), &full[s]);
                if (++s == S) { s = 0; ph ^= 1; }
            }
        }
    } else if (warp == 1) {
        const uint32_t idesc = idesc_bf16(BM, p.BN, 1, 1);
        int s = 0;
        uint32_t ph = 0;
        for (int64_t kb = kb0; kb < kb1; ++kb) {
            mbar_wait(&full[s], ph);
            uint8_t* sa = smem + s * stage_bytes;
            const int64_t valid = M - kb * BK;       // rows of this k-block inside [0, M)
            if (valid < BK) {                        // zero the tail rows of every box (generic proxy)
                const int nboxes = p.nbA + p.nbB;
                for (int idx = threadIdx.x & 31; idx < nboxes * (BK - (int)valid) * 8; idx += 32) {
                    const int b = idx / ((BK - (int)valid) * 8);
                    const int rr = (idx / 8) % (BK - (int)valid) + (int)valid;
                    const int ch = idx & 7;
                    *(uint4*)(sa + b * box + rr * 128 + ch * 16) = make_uint4(0, 0, 0, 0);
                }
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                __syncwarp();
            }
            fence_after();
            if (elect_lane0()) {
                const uint32_t a0 = su32(sa), b0 = a0 + a_bytes;
#pragma unroll
                for (int k = 0; k < BK / UK; ++k) {
                    // MN-major SW128: atoms of 64 (MN) x 8 (K) at SBO = 1024 along K, LBO = box along MN
                    const uint64_t ad = sdesc(a0 + k * UK * 128, box, 1024);
                    const uint64_t bd = sdesc(b0 + k * UK * 128, box, 1024);
                    umma_f16(tmem, ad, bd, idesc, (kb != kb0 || k != 0));
                }
                umma_commit(&empty[s]);
                if (kb == kb1 - 1) umma_commit(&tfull[0]);
            }
            __syncwarp();
            if (++s == S) { s = 0; ph ^= 1; }
        }
    } else {
        const int q = warp & 3;
        const int r_in = q * 32 + (threadIdx.x & 31);
        const int feat = mt * BM + r_in;
        float* out = p.partials + ((int64_t)split * p.K1 + feat) * p.N;
        if (kb1 > kb0) {
            mbar_wait(&tfull[0], 0);
            fence_after();
        }
        for (int c0 = 0; c0 < p.BN; c0 += 32) {
            float v[32];
            if (kb1 > kb0) tmem_ld32(tmem + ((uint32_t)(q * 32) << 16) + c0, v);
            else {
#pragma unroll
                for (int j = 0; j < 32; ++j) v[j] = 0.f;
            }
            if (feat < p.K1)
                for (int j = 0; j < 32 && c0 + j < p.N; ++j) out[c0 + j] = v[j];
        }
        fence_before();
    }
    __syncthreads();
    if (warp == 1) {
        fence_after();
        tmem_free_warp(tmem, p.tmem_cols);
    }
}

// ------------------------------------------------------------------ host
typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                             const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                             CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeFn encode_fn() {
    static EncodeFn fn = nullptr;
    if (!fn) {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (EncodeFn)p;
    }
    return fn;
}

// 2-D bf16 tensor [rows x cols] with row stride ld (elements); box {64 cols, box_rows}
static bool make_map(CUtensorMap* m, const void* base, int64_t cols, int64_t rows, int64_t ld, int box_rows) {
    EncodeFn f = encode_fn();
    if (!f) return false;
    cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
    cuuint64_t strides[1] = {(cuuint64_t)ld * 2};
    cuuint32_t box[2] = {64, (cuuint32_t)box_rows};
    cuuint32_t es[2] = {1, 1};
    return f(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, es,
             CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

static uint32_t tmem_cols_for(int n) {
    uint32_t c = 32;
    while ((int)c < n) c <<= 1;
    return c;
}

}  // namespace tc

bool tc_available() { return tc::encode_fn() != nullptr; }

// C = A B on the tensor cores; B given K-major as Bk[N x K] (ld ldbk).  Returns false if the shape is unsupported.
bool gemm_row_tc(betty_ctx* c, const GemmRow& g, const void* Bk, int64_t ldbk, cudaStream_t s) {
    using namespace tc;
    if (!g.a_bf16 || !g.b_bf16 || g.N > 256 || g.N < 1 || (g.lda & 7) || (ldbk & 7)) return false;
    if ((g.epi == EPI_MASK || g.epi == EPI_RES_MASK) && (g.ldm & 7)) return false;
    const int BN = (g.N + 15) / 16 * 16;
    const int nk = (g.K + BK - 1) / BK;
    const size_t b_bytes = (size_t)nk * BN * BK * 2;
    const size_t a_bytes = BM * BK * 2;
    const size_t budget = 220 * 1024;
    if (b_bytes + 2 * a_bytes + 2048 > budget) return false;       // B must fit resident
    CUtensorMap ma, mb;
    if (!make_map(&ma, g.A, g.K, g.M_cap, g.lda, BM) || !make_map(&mb, Bk, g.K, g.N, ldbk, BN)) return false;
    RowArgs p{};
    p.M_dev = g.M_dev; p.K = g.K; p.N = g.N; p.BN = BN; p.nk = nk;
    p.stages = (int)std::max<size_t>(2, std::min<size_t>(8, (budget - b_bytes - 2048) / a_bytes));
    p.C = g.C; p.ldc = g.ldc; p.c_bf16 = g.c_bf16; p.epi = g.epi;
    p.mask = g.mask; p.ldm = g.ldm; p.m_bf16 = g.m_bf16; p.res = g.res; p.ldr = g.ldr; p.nres_dev = g.nres_dev;
    p.tmem_cols = tmem_cols_for(2 * BN);
    p.half_cols = ((BN + 63) / 64) * 32;
    if (p.tmem_cols > 512) return false;
    const size_t smem = b_bytes + (size_t)p.stages * a_bytes + 1024 + 256;
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(k_tc_row, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
        attr = true;
    }
    const int64_t tiles = (g.M_cap + BM - 1) / BM;
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(tiles, c->num_sms));
    k_tc_row<<<grid, ROW_THREADS, smem, s>>>(ma, mb, p);
    return true;
}

bool gemm_red_tc(betty_ctx* c, const GemmRed& g, cudaStream_t s) {
    using namespace tc;
    if (!g.a_bf16 || !g.b_bf16 || g.N > 256 || (g.lda & 7) || (g.ldb & 7)) return false;
    const int BN = (g.N + 15) / 16 * 16;
    CUtensorMap ma, mb;
    if (!make_map(&ma, g.A, g.K1, g.M_cap, g.lda, BK) || !make_map(&mb, g.B, g.N, g.M_cap, g.ldb, BK)) return false;
    RedArgs p{};
    p.M_dev = g.M_dev; p.K1 = g.K1; p.N = g.N; p.BN = BN;
    p.nbA = BM / 64; p.nbB = (BN + 63) / 64;
    const int stage_bytes = (p.nbA + p.nbB) * BK * 128;
    p.stages = std::max(2, std::min(8, (200 * 1024) / stage_bytes));
    p.mtiles = (g.K1 + BM - 1) / BM;
    p.S = g.S;
    p.partials = g.partials;
    p.tmem_cols = tmem_cols_for(BN);
    const size_t smem = (size_t)p.stages * stage_bytes + 1024 + 256;
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(k_tc_red, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
        attr = true;
    }
    k_tc_red<<<p.mtiles * p.S, THREADS, smem, s>>>(ma, mb, p);
    return true;
}

}  // namespace betty
