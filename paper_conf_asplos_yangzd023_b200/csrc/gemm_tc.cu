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
// columns, one output row per thread.  Each 32-column chunk goes TMEM ->
// registers (epilogue math) -> a swizzled shared-memory staging slot -> TMA
// bulk-tensor store, so the global writes are full-line, asynchronous and off
// the epilogue's critical path.  The ReLU' mask of a backward layer comes as
// one bit per element (written by the forward epilogue), 32 B per 256-wide row
// instead of re-reading the bf16 activations.  The kernel is templated on the
// epilogue so each 32-column chunk is straight-line code (~150 instructions).
constexpr int EPI_WARPS = 8;
constexpr int ESLOTS = 2;                       // staging slots per epilogue warp
constexpr int ROW_THREADS = 64 + 32 * EPI_WARPS;
constexpr int MAXCH = 4;                        // 32-column chunks per epilogue half (N <= 256)
struct RowArgs {
    const int64_t* M_dev;
    int K, N, BN, nk, stages;
    void* C; int64_t ldc;
    const void* mask; int64_t ldm; int m_bf16;  // EPI_MASK / EPI_RES_MASK from activations (MBITS = false)
    const uint32_t* mbits; int64_t ldmb;        // ... or from ReLU bits (MBITS = true)
    uint32_t* obits; int64_t ldob;              // EPI_RELU_ONES: ReLU bits out (words per row), or null
    const float* res; int64_t ldr; const int64_t* nres_dev;
    uint32_t tmem_cols;
    int acc_stride;          // TMEM columns between the two accumulators (>= BN, multiple of 32)
    int half_cols;           // columns per epilogue half (multiple of 32, <= 32 * MAXCH)
    uint32_t slot_bytes;     // one staging slot: 32 rows x 32 columns
    int bstream;             // 1: B is streamed with A through the ring (B too large to stay resident)
    int64_t cend;            // trailing columns [N, cend) of a row are written (ones column / zeros)
};

__device__ __forceinline__ uint32_t pack_bf16x2(float a, float b) {
    __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
    return *(uint32_t*)&h;
}
__device__ __forceinline__ void tma_store_2d(const CUtensorMap* tm, const void* src, int c0, int c1) {
    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];"
                 ::"l"((uint64_t)tm), "r"(c0), "r"(c1), "r"(su32(src)) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N> __device__ __forceinline__ void bulk_wait_read() {
    asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

__device__ __forceinline__ void tmem_ld32_nowait(uint32_t taddr, uint32_t* r) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
                 "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                   "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]),
                   "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]),
                   "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]),
                   "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
                 : "r"(taddr));
}
// tcgen05.wait::ld that the compiler cannot move reads of r across
__device__ __forceinline__ void tmem_wait_regs(uint32_t* r) {
    asm volatile("tcgen05.wait::ld.sync.aligned;"
                 : "+r"(r[0]), "+r"(r[1]), "+r"(r[2]), "+r"(r[3]), "+r"(r[4]), "+r"(r[5]), "+r"(r[6]), "+r"(r[7]),
                   "+r"(r[8]), "+r"(r[9]), "+r"(r[10]), "+r"(r[11]), "+r"(r[12]), "+r"(r[13]), "+r"(r[14]),
                   "+r"(r[15]), "+r"(r[16]), "+r"(r[17]), "+r"(r[18]), "+r"(r[19]), "+r"(r[20]), "+r"(r[21]),
                   "+r"(r[22]), "+r"(r[23]), "+r"(r[24]), "+r"(r[25]), "+r"(r[26]), "+r"(r[27]), "+r"(r[28]),
                   "+r"(r[29]), "+r"(r[30]), "+r"(r[31])
                 :
                 : "memory");
}

// [activation > 0] of a stored 32-column chunk (mask from activations, MBITS = false)
__device__ __forceinline__ uint32_t mask_word_from_act(const RowArgs& p, int64_t m, int c0, bool ok) {
    if (!ok) return 0u;
    uint32_t w = 0;
    const int nval = min(32, p.N - c0);
    if (p.m_bf16) {
        const uint4* src = (const uint4*)((const __nv_bfloat16*)p.mask + m * p.ldm + c0);
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            if (q * 8 >= nval) break;
            const uint4 t = src[q];
            const uint32_t u[4] = {t.x, t.y, t.z, t.w};
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const __nv_bfloat162 h = *(const __nv_bfloat162*)&u[k];
                w |= (uint32_t)(__low2float(h) > 0.f) << (8 * q + 2 * k);
                w |= (uint32_t)(__high2float(h) > 0.f) << (8 * q + 2 * k + 1);
            }
        }
    } else {
        const float4* src = (const float4*)((const float*)p.mask + m * p.ldm + c0);
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            if (q * 4 >= nval) break;
            const float4 t = src[q];
            w |= (uint32_t)(t.x > 0.f) << (4 * q) | (uint32_t)(t.y > 0.f) << (4 * q + 1) |
                 (uint32_t)(t.z > 0.f) << (4 * q + 2) | (uint32_t)(t.w > 0.f) << (4 * q + 3);
        }
    }
    if (nval < 32) w &= (1u << nval) - 1u;
    return w;
}

// one 32-column chunk: epilogue math on v (fp32 bits in r), staged for the TMA store.
// Returns the ReLU bits (EPI_RELU_ONES).
template <int EPI, bool CBF>
__device__ __forceinline__ uint32_t chunk_epilogue(const RowArgs& p, const uint32_t* r, int64_t m, int c0, bool ok,
                                                   uint32_t mword, int64_t nres, uint8_t* slot, int lane) {
    float v[32];
#pragma unroll
    for (int j = 0; j < 32; ++j) v[j] = __uint_as_float(r[j]);
    if (EPI == EPI_RES_MASK && ok && m < nres) {
        const float* rp = p.res + m * p.ldr + c0;
        const int nval = min(32, p.N - c0);
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            if (q * 4 < nval) {
                const float4 t = *(const float4*)(rp + 4 * q);
                v[4 * q] += t.x; v[4 * q + 1] += t.y; v[4 * q + 2] += t.z; v[4 * q + 3] += t.w;
            }
        }
    }
    if (EPI == EPI_MASK || EPI == EPI_RES_MASK) {
#pragma unroll
        for (int j = 0; j < 32; ++j) v[j] = ((mword >> j) & 1u) ? v[j] : 0.f;
    }
    if (EPI == EPI_RELU_ONES) {
#pragma unroll
        for (int j = 0; j < 32; ++j) v[j] = fmaxf(v[j], 0.f);
    }
    if (!ok) {
#pragma unroll
        for (int j = 0; j < 32; ++j) v[j] = 0.f;
    }
    uint32_t bits = 0;
    if (CBF) {
        uint32_t w[16];
#pragma unroll
        for (int k = 0; k < 16; ++k) w[k] = pack_bf16x2(v[2 * k], v[2 * k + 1]);
        if (EPI == EPI_RELU_ONES) {     // bit = [stored bf16 value > 0] (ReLU output: non-negative)
#pragma unroll
            for (int k = 0; k < 16; ++k)
                bits |= (uint32_t)((w[k] & 0x7fffu) != 0u) << (2 * k) | (uint32_t)((w[k] & 0x7fff0000u) != 0u) << (2 * k + 1);
        }
        // 64 B rows, SWIZZLE_64B: 16-B chunk c of row r at c ^ ((r >> 1) & 3)
        uint8_t* row = slot + lane * 64;
#pragma unroll
        for (int c = 0; c < 4; ++c)
            *(uint4*)(row + ((c ^ ((lane >> 1) & 3)) << 4)) = make_uint4(w[4 * c], w[4 * c + 1], w[4 * c + 2], w[4 * c + 3]);
    } else {
        if (EPI == EPI_RELU_ONES) {
#pragma unroll
            for (int j = 0; j < 32; ++j) bits |= (uint32_t)(v[j] > 0.f) << j;
        }
        // 128 B rows, SWIZZLE_128B: 16-B chunk c of row r at c ^ (r & 7)
        uint8_t* row = slot + lane * 128;
#pragma unroll
        for (int c = 0; c < 8; ++c)
            *(float4*)(row + ((c ^ (lane & 7)) << 4)) = make_float4(v[4 * c], v[4 * c + 1], v[4 * c + 2], v[4 * c + 3]);
    }
    return bits;
}

template <int EPI, bool CBF, bool MBITS>
__global__ void __launch_bounds__(ROW_THREADS, 1) k_tc_row(const __grid_constant__ CUtensorMap tmA,
                                                           const __grid_constant__ CUtensorMap tmB,
                                                           const __grid_constant__ CUtensorMap tmC, RowArgs p) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    const int S = p.stages;
    const uint32_t a_bytes = BM * BK * 2;
    const uint32_t bblk = (uint32_t)p.BN * BK * 2;          // one K-block of B
    const uint32_t ring_bytes = a_bytes + (p.bstream ? bblk : 0u);   // one ring stage: A (+ B when streamed)
    uint8_t* bres = smem;                                    // nk * bblk (resident B) or nothing
    uint8_t* aring = smem + (p.bstream ? 0 : p.nk * bblk);   // S * ring_bytes
    uint8_t* stage = aring + S * ring_bytes;                 // EPI_WARPS * ESLOTS * slot_bytes
    uint64_t* full = (uint64_t*)(stage + EPI_WARPS * ESLOTS * p.slot_bytes);
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
        for (int a = 0; a < 2; ++a) { mbar_init(&tfull[a], 1); mbar_init(&tempty[a], 32 * EPI_WARPS); }
        mbar_init(bfull, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmA) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmB) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmC) : "memory");
    }
    if (warp == 1) tmem_alloc_warp(tslot, p.tmem_cols);
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tmem = *tslot;

    if (warp == 0) {
        if (elect_lane0() && blockIdx.x < tiles) {
            if (!p.bstream) {
                mbar_expect_tx(bfull, p.nk * bblk);
                for (int kb = 0; kb < p.nk; ++kb) tma_2d(bres + kb * bblk, &tmB, kb * BK, 0, bfull);
            }
            int s = 0;
            uint32_t ph = 0;
            for (int64_t t = blockIdx.x; t < tiles; t += gridDim.x) {
                for (int kb = 0; kb < p.nk; ++kb) {
                    mbar_wait(&empty[s], ph ^ 1);
                    mbar_expect_tx(&full[s], ring_bytes);
                    tma_2d(aring + s * ring_bytes, &tmA, kb * BK, (int)(t * BM), &full[s]);
                    if (p.bstream) tma_2d(aring + s * ring_bytes + a_bytes, &tmB, kb * BK, 0, &full[s]);
                    if (++s == S) { s = 0; ph ^= 1; }
                }
            }
        }
    } else if (warp == 1) {
        const uint32_t idesc = idesc_bf16(BM, p.BN, 0, 0);
        int s = 0;
        uint32_t ph = 0;
        int it = 0;
        if (blockIdx.x < tiles && !p.bstream) mbar_wait(bfull, 0);
        for (int64_t t = blockIdx.x; t < tiles; t += gridDim.x, ++it) {
            const int acc = it & 1;
            const uint32_t aph = (it >> 1) & 1;
            mbar_wait(&tempty[acc], aph ^ 1);
            fence_after();
            const uint32_t d = tmem + acc * p.acc_stride;
            for (int kb = 0; kb < p.nk; ++kb) {
                mbar_wait(&full[s], ph);
                fence_after();
                if (elect_lane0()) {
                    const uint32_t a0 = su32(aring + s * ring_bytes);
                    const uint32_t b0 = p.bstream ? a0 + a_bytes : su32(bres + kb * bblk);
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
        constexpr bool HAS_MASK = EPI == EPI_MASK || EPI == EPI_RES_MASK;
        const int ew = warp - 2;                 // 0..7
        const int q = warp & 3;                  // TMEM lane quadrant (hardware: warp id % 4)
        const int h = ew >> 2;                   // column half
        const int lane = threadIdx.x & 31;
        const int cbeg = h * p.half_cols;
        const int cstore = min(min(p.BN, cbeg + p.half_cols), p.N);   // chunks at or past N are not stored
        const int nch = cstore > cbeg ? (cstore - cbeg + 31) / 32 : 0;
        const int64_t nres = EPI == EPI_RES_MASK ? *p.nres_dev : 0;
        uint8_t* my_stage = stage + ew * ESLOTS * p.slot_bytes;
        int slot = 0;
        int it = 0;
        // ReLU' bit words of this thread's row, one tile ahead (short-K layers finish the MMA long
        // before a load round trip, so loading them at the top of the tile left them exposed)
        uint32_t mw_next[MAXCH];
#pragma unroll
        for (int ci = 0; ci < MAXCH; ++ci) mw_next[ci] = 0u;
        auto load_bits = [&](int64_t tt, uint32_t (&dst)[MAXCH]) {
            const int64_t mm = tt * BM + q * 32 + lane;
            if (tt < tiles && mm < M) {
                const uint32_t* wb = p.mbits + mm * p.ldmb + cbeg / 32;
#pragma unroll
                for (int ci = 0; ci < MAXCH; ++ci) if (ci < nch) dst[ci] = wb[ci];
            }
        };
        if (HAS_MASK && MBITS) load_bits(blockIdx.x, mw_next);
        for (int64_t t = blockIdx.x; t < tiles; t += gridDim.x, ++it) {
            const int acc = it & 1;
            const uint32_t aph = (it >> 1) & 1;
            const int64_t row0 = t * BM + q * 32;
            const int64_t m = row0 + lane;
            const bool ok = m < M;
            // mask words of this thread's chunks, loaded before the accumulator wait (latency hidden)
            uint32_t mw[MAXCH];
#pragma unroll
            for (int ci = 0; ci < MAXCH; ++ci) mw[ci] = 0u;
            if (HAS_MASK) {
                if (MBITS) {
#pragma unroll
                    for (int ci = 0; ci < MAXCH; ++ci) { mw[ci] = ok ? mw_next[ci] : 0u; mw_next[ci] = 0u; }
                    load_bits(t + gridDim.x, mw_next);
                } else {
#pragma unroll
                    for (int ci = 0; ci < MAXCH; ++ci) if (ci < nch) mw[ci] = mask_word_from_act(p, m, cbeg + 32 * ci, ok);
                }
            }
            mbar_wait(&tfull[acc], aph);
            fence_after();
            const uint32_t tbase = tmem + ((uint32_t)(q * 32) << 16) + acc * p.acc_stride;
            uint32_t ra[32], rb[32];
            uint32_t obits[MAXCH];
            if (nch > 0) { tmem_ld32_nowait(tbase + cbeg, ra); tmem_wait_regs(ra); }
#pragma unroll
            for (int ci = 0; ci < MAXCH; ++ci) {
                obits[ci] = 0u;
                if (ci < nch) {
                    uint32_t* cur = (ci & 1) ? rb : ra;
                    uint32_t* nxt = (ci & 1) ? ra : rb;
                    const int c0 = cbeg + 32 * ci;
                    if (ci + 1 < nch) tmem_ld32_nowait(tbase + c0 + 32, nxt);   // next chunk in flight
                    uint8_t* sl = my_stage + slot * p.slot_bytes;
                    if (lane == 0) bulk_wait_read<ESLOTS - 1>();    // the store that used this slot has read it
                    __syncwarp();
                    obits[ci] = chunk_epilogue<EPI, CBF>(p, cur, m, c0, ok, mw[ci], nres, sl, lane);
                    fence_proxy_async();
                    __syncwarp();
                    if (lane == 0) {
                        tma_store_2d(&tmC, sl, c0, (int)row0);
                        bulk_commit();
                    }
                    if (++slot == ESLOTS) slot = 0;
                    if (ci + 1 < nch) tmem_wait_regs(nxt);
                }
            }
            fence_before();
            mbar_arrive(&tempty[acc]);
            if (EPI == EPI_RELU_ONES && p.obits && ok && nch > 0) {
                uint32_t* ob = p.obits + m * p.ldob + cbeg / 32;
                if (nch == 4 && ((uintptr_t)ob & 15) == 0)
                    *(uint4*)ob = make_uint4(obits[0], obits[1], obits[2], obits[3]);
                else
#pragma unroll
                    for (int ci = 0; ci < MAXCH; ++ci) if (ci < nch) ob[ci] = obits[ci];
            }
            // trailing columns [N, ldc): the ones column after a ReLU layer, zeros elsewhere
            if (h == 1 && ok && p.cend > p.N) {
                const int w = (int)(p.cend - p.N);
                if (CBF && w == 8 && ((m * p.ldc + p.N) & 7) == 0) {
                    const uint32_t one = EPI == EPI_RELU_ONES ? 0x3F80u : 0u;
                    *(uint4*)((__nv_bfloat16*)p.C + m * p.ldc + p.N) = make_uint4(one, 0u, 0u, 0u);
                } else {
                    for (int col = p.N; col < p.cend; ++col) {
                        const float x = (EPI == EPI_RELU_ONES && col == p.N) ? 1.f : 0.f;
                        if (CBF) ((__nv_bfloat16*)p.C)[m * p.ldc + col] = __float2bfloat16_rn(x);
                        else ((float*)p.C)[m * p.ldc + col] = x;
                    }
                }
            }
        }
        if (lane == 0) bulk_wait_all();
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
    int mt_cta;                // feature tiles per CTA: 1 (grid = mtiles x S) or mtiles (grid = S; A, B read once)
    int acc_stride;            // TMEM columns per feature tile accumulator
    float* partials;           // [S][K1][N]
    uint32_t tmem_cols;
};

__global__ void __launch_bounds__(THREADS, 1) k_tc_red(const __grid_constant__ CUtensorMap tmA,
                                                       const __grid_constant__ CUtensorMap tmB, RedArgs p) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    const int S = p.stages;
    const uint32_t box = BK * 128;                    // 64 rows x 128 B
    const int nbA_cta = p.nbA * p.mt_cta;             // A boxes per stage (64 features each)
    const uint32_t a_bytes = nbA_cta * box, b_bytes = p.nbB * box;
    const uint32_t stage_bytes = a_bytes + b_bytes;
    uint64_t* full = (uint64_t*)(smem + S * stage_bytes);
    uint64_t* empty = full + S;
    uint64_t* tfull = empty + S;
    uint32_t* tslot = (uint32_t*)(tfull + 1);

    const int warp = threadIdx.x >> 5;
    const int nsplit = p.mt_cta == 1 ? p.mtiles : 1;
    const int mt0 = p.mt_cta == 1 ? blockIdx.x % p.mtiles : 0;
    const int split = blockIdx.x / nsplit;
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
                for (int i = 0; i < nbA_cta; ++i) tma_2d(sa + i * box, &tmA, mt0 * BM + i * 64, (int)(kb * BK), &full[s]);
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
                const int nboxes = nbA_cta + p.nbB;
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
                const uint32_t b0 = su32(sa) + a_bytes;
                for (int mt = 0; mt < p.mt_cta; ++mt) {
                    const uint32_t a0 = su32(sa) + mt * p.nbA * box;
#pragma unroll
                    for (int k = 0; k < BK / UK; ++k) {
                        // MN-major SW128: atoms of 64 (MN) x 8 (K) at SBO = 1024 along K, LBO = box along MN
                        const uint64_t ad = sdesc(a0 + k * UK * 128, box, 1024);
                        const uint64_t bd = sdesc(b0 + k * UK * 128, box, 1024);
                        umma_f16(tmem + mt * p.acc_stride, ad, bd, idesc, (kb != kb0 || k != 0));
                    }
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
        if (kb1 > kb0) {
            mbar_wait(&tfull[0], 0);
            fence_after();
        }
        for (int mt = 0; mt < p.mt_cta; ++mt) {
            const int feat = (mt0 + mt) * BM + r_in;
            float* out = p.partials + ((int64_t)split * p.K1 + feat) * p.N;
            for (int c0 = 0; c0 < p.BN; c0 += 32) {
                float v[32];
                if (kb1 > kb0) tmem_ld32(tmem + ((uint32_t)(q * 32) << 16) + mt * p.acc_stride + c0, v);
                else {
#pragma unroll
                    for (int j = 0; j < 32; ++j) v[j] = 0.f;
                }
                if (feat < p.K1) {
                    if (c0 + 32 <= p.N && (p.N & 3) == 0) {
#pragma unroll
                        for (int j = 0; j < 32; j += 4) *(float4*)(out + c0 + j) = make_float4(v[j], v[j + 1], v[j + 2], v[j + 3]);
                    } else {
                        for (int j = 0; j < 32 && c0 + j < p.N; ++j) out[c0 + j] = v[j];
                    }
                }
            }
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

// 2-D tensor [rows x cols] with row stride ld (elements); box {box_cols, box_rows}
static bool make_map_t(CUtensorMap* m, const void* base, bool f32, int64_t cols, int64_t rows, int64_t ld,
                       int box_cols, int box_rows, CUtensorMapSwizzle sw,
                       CUtensorMapL2promotion promo = CU_TENSOR_MAP_L2_PROMOTION_L2_256B) {
    EncodeFn f = encode_fn();
    if (!f) return false;
    const int es = f32 ? 4 : 2;
    if (((uintptr_t)base & 15) || (ld * es) % 16) return false;
    cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
    cuuint64_t strides[1] = {(cuuint64_t)ld * es};
    cuuint32_t box[2] = {(cuuint32_t)box_cols, (cuuint32_t)box_rows};
    cuuint32_t estr[2] = {1, 1};
    return f(m, f32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base),
             dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, sw, promo,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}
// bf16 operand maps: box {64 cols (128 B), box_rows}, 128-byte swizzle
static bool make_map(CUtensorMap* m, const void* base, int64_t cols, int64_t rows, int64_t ld, int box_rows) {
    return make_map_t(m, base, false, cols, rows, ld, 64, box_rows, CU_TENSOR_MAP_SWIZZLE_128B);
}

static uint32_t tmem_cols_for(int n) {
    uint32_t c = 32;
    while ((int)c < n) c <<= 1;
    return c;
}

}  // namespace tc

bool tc_available() { return tc::encode_fn() != nullptr; }

// Row-gather map for tile::gather4 (agg.cu): a [rows x cols] table with row stride ld, box
// {box_cols, 1}; columns >= cols and out-of-range rows (e.g. -1) read as zeros.
bool make_gather_map(CUtensorMap* m, const void* base, bool f32, int64_t cols, int64_t rows, int64_t ld,
                     int box_cols) {
    // no L2 promotion: a gathered row is fetched at sector granularity, not as 256-byte blocks
    return tc::make_map_t(m, base, f32, cols, rows, ld, box_cols, 1, CU_TENSOR_MAP_SWIZZLE_NONE,
                          CU_TENSOR_MAP_L2_PROMOTION_NONE);
}

// C = A B on the tensor cores; B given K-major as Bk[N x K] (ld ldbk).  Returns false if the shape is unsupported.
bool gemm_row_tc(betty_ctx* c, const GemmRow& g, const void* Bk, int64_t ldbk, cudaStream_t s) {
    using namespace tc;
    if (!g.a_bf16 || !g.b_bf16 || g.N > 256 || g.N < 1 || (g.lda & 7) || (ldbk & 7)) return false;
    if ((g.epi == EPI_MASK || g.epi == EPI_RES_MASK) && !g.mbits && (g.ldm & 7)) return false;
    const int BN = (g.N + 15) / 16 * 16;
    const int nk = (g.K + BK - 1) / BK;
    const size_t b_bytes = (size_t)nk * BN * BK * 2;
    const size_t a_bytes = BM * BK * 2;
    const uint32_t slot_bytes = 32 * 32 * (g.c_bf16 ? 2 : 4);
    const size_t stage_bytes = (size_t)EPI_WARPS * ESLOTS * slot_bytes;
    const size_t budget = 227 * 1024;           // the sm_100 opt-in maximum of dynamic shared memory per CTA
    const size_t bblk = (size_t)BN * BK * 2;
    // B resident when it fits next to a 2-stage A ring, else streamed with A
    const bool bstream = b_bytes + stage_bytes + 2 * a_bytes + 1024 + 256 > budget;
    const size_t ring = a_bytes + (bstream ? bblk : 0);
    const size_t fixed = (bstream ? 0 : b_bytes) + stage_bytes + 1024 + 256;
    if (fixed + 2 * ring > budget) return false;
    CUtensorMap ma, mb, mc;
    if (!make_map(&ma, g.A, g.K, g.M_cap, g.lda, BM) || !make_map(&mb, Bk, g.K, g.N, ldbk, BN)) return false;
    if (!make_map_t(&mc, g.C, !g.c_bf16, g.N, g.M_cap, g.ldc, 32, 32,
                    g.c_bf16 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_128B))
        return false;
    RowArgs p{};
    p.M_dev = g.M_dev; p.K = g.K; p.N = g.N; p.BN = BN; p.nk = nk;
    p.stages = (int)std::max<size_t>(2, std::min<size_t>(8, (budget - fixed) / ring));
    p.bstream = bstream ? 1 : 0;
    p.C = g.C; p.ldc = g.ldc; p.cend = g.cend > 0 ? g.cend : g.ldc;
    p.mask = g.mask; p.ldm = g.ldm; p.m_bf16 = g.m_bf16; p.res = g.res; p.ldr = g.ldr; p.nres_dev = g.nres_dev;
    p.mbits = g.mbits; p.ldmb = g.ldmb;
    p.obits = g.epi == EPI_RELU_ONES ? g.obits : nullptr; p.ldob = g.ldob;
    p.acc_stride = (BN + 31) / 32 * 32;
    p.tmem_cols = tmem_cols_for(2 * p.acc_stride);
    p.half_cols = ((BN + 63) / 64) * 32;
    p.slot_bytes = slot_bytes;
    if (p.tmem_cols > 512 || p.half_cols > 32 * MAXCH) return false;
    const size_t smem = fixed + (size_t)p.stages * ring;
    const int64_t tiles = (g.M_cap + BM - 1) / BM;
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(tiles, c->num_sms));
    const bool usebits = g.mbits != nullptr;
#define ROW_LAUNCH(E, CB, MB)                                                                      \
    do {                                                                                           \
        static bool attr = false;                                                                  \
        if (!attr) {                                                                               \
            cudaFuncSetAttribute(k_tc_row<E, CB, MB>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024); \
            attr = true;                                                                           \
        }                                                                                          \
        k_tc_row<E, CB, MB><<<grid, ROW_THREADS, smem, s>>>(ma, mb, mc, p);                       \
    } while (0)
    switch (g.epi) {
    case EPI_STORE:
        if (g.c_bf16) ROW_LAUNCH(EPI_STORE, true, false); else ROW_LAUNCH(EPI_STORE, false, false);
        break;
    case EPI_RELU_ONES:
        if (g.c_bf16) ROW_LAUNCH(EPI_RELU_ONES, true, false); else ROW_LAUNCH(EPI_RELU_ONES, false, false);
        break;
    case EPI_MASK:
        if (g.c_bf16) { if (usebits) ROW_LAUNCH(EPI_MASK, true, true); else ROW_LAUNCH(EPI_MASK, true, false); }
        else { if (usebits) ROW_LAUNCH(EPI_MASK, false, true); else ROW_LAUNCH(EPI_MASK, false, false); }
        break;
    default:
        if (g.c_bf16) { if (usebits) ROW_LAUNCH(EPI_RES_MASK, true, true); else ROW_LAUNCH(EPI_RES_MASK, true, false); }
        else { if (usebits) ROW_LAUNCH(EPI_RES_MASK, false, true); else ROW_LAUNCH(EPI_RES_MASK, false, false); }
        break;
    }
#undef ROW_LAUNCH
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
    p.mtiles = (g.K1 + BM - 1) / BM;
    p.acc_stride = (BN + 31) / 32 * 32;
    // all feature tiles in one CTA when their accumulators fit TMEM and a stage fits 3x in smem:
    // A and B are then read exactly once
    const int stage_all = (p.nbA * p.mtiles + p.nbB) * BK * 128;
    p.mt_cta = (p.mtiles * p.acc_stride <= 512 && 3 * stage_all <= 200 * 1024) ? p.mtiles : 1;
    const int stage_bytes = (p.nbA * p.mt_cta + p.nbB) * BK * 128;
    p.stages = std::max(2, std::min(8, (200 * 1024) / stage_bytes));
    p.S = g.S;
    p.partials = g.partials;
    p.tmem_cols = tmem_cols_for(p.mt_cta * p.acc_stride);
    const size_t smem = (size_t)p.stages * stage_bytes + 1024 + 256;
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(k_tc_red, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
        attr = true;
    }
    k_tc_red<<<(p.mt_cta == 1 ? p.mtiles : 1) * p.S, THREADS, smem, s>>>(ma, mb, p);
    return true;
}

}  // namespace betty
