// gemm_tc.cu -- the dense SAGE layers on the 5th-generation tensor cores, hand-written PTX:
// TMA (cp.async.bulk.tensor, 128B swizzle) fills a multi-stage shared-memory ring, one elected
// thread issues tcgen05.mma into TMEM, epilogue warps drain TMEM with tcgen05.ld.  Persistent, one
// CTA per SM.  Two precisions:
//   BF16 mode: kind::f16 (bf16 operands), fp32 accumulation;
//   FP32 mode (TF = true): kind::tf32 as 3xTF32 -- converter warps split each landed fp32 stage into an
//     RN-tf32 hi (in place) and lo, and per k-block the MMA warp issues lo*hi, hi*lo (into a second
//     accumulator) and hi*hi; see split_tf32 and the k_tc_red drain for why (fp32-level accuracy).
//
//   k_tc_row : C[M x N] = A[M x K] B[K x N]   (A, B K-major; M on the device)
//              warps: 0 TMA producer, 1 TMEM allocator + MMA issuer, 2-9 epilogue (8 warps: warp w
//              drains TMEM lanes 32*(w%4).. for one half of the columns), + 2 converter warps in TF
//              (320 / 384 threads).  Epilogues: store / ReLU + ones column (+ ReLU' bits) / ReLU' mask
//              / residual + mask; each 32-column chunk goes TMEM -> registers -> swizzled smem slot ->
//              TMA store.  Two TMEM accumulators (BF16 always, TF when 4 * BN <= 512) so the epilogue
//              of tile i overlaps the MMAs of tile i+1.
//   k_tc_red : P[K1 x N] = A^T B over the node dimension (dW), A and B MN-major (node rows
//              contiguous in features), a fixed row range per CTA accumulated in TMEM, partials
//              reduced deterministically by k_red_final (gemm.cu) into the flat gradient.  Warps: 0
//              TMA, 1 MMA, 2-5 epilogue (+ 4 converter warps in TF: 192 / 320 threads).
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
__device__ __forceinline__ void umma_tf32(uint32_t tmem_d, uint64_t ad, uint64_t bd, uint32_t idesc, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}"
                 ::"r"(tmem_d), "l"(ad), "l"(bd), "r"(idesc), "r"(acc));
}
// shared-memory matrix descriptor, sm_100 version 1; layout type 2 = SWIZZLE_128B (16-byte swizzle
// base, 8-row atoms), 1 = SWIZZLE_128B_BASE32B (32-byte base, 4-row atoms: the only layout an MN-major
// tf32 operand may use; TMA's CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B writes it)
__device__ __forceinline__ uint64_t sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo, uint32_t layout = 2) {
    uint64_t d = (uint64_t)((saddr >> 4) & 0x3FFF);
    d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
    d |= (uint64_t)1 << 46;
    d |= (uint64_t)layout << 61;
    return d;
}
// instruction descriptor: bf16 x bf16 -> f32, M x N, operand majors (0 = K, 1 = MN)
__host__ __device__ constexpr uint32_t idesc_bf16(int M, int N, int a_mn, int b_mn) {
    return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)a_mn << 15) | ((uint32_t)b_mn << 16) |
           ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}
// tf32 x tf32 -> f32 (operands are fp32 words in shared memory; FP32 mode's 3xTF32 split)
__host__ __device__ constexpr uint32_t idesc_tf32(int M, int N, int a_mn, int b_mn) {
    return (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)a_mn << 15) | ((uint32_t)b_mn << 16) |
           ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}
// 3xTF32 split of a float4 in shared memory: hi = x rounded to the nearest tf32 (10 mantissa bits,
// so the tensor core's own fp32 -> tf32 conversion is the identity on it), lo = x - hi (exact in fp32,
// |lo| <= 2^-11 |x|) also rounded to the nearest tf32 (the dropped remainder is <= 2^-23 |x|).  With
// the lo*lo term dropped (<= 2^-22 of the product), each product is exact to ~2^-22.  hi overwrites x.
__device__ __forceinline__ float tf32_rn(float x) {
    return __uint_as_float((__float_as_uint(x) + 0x1000u) & 0xFFFFE000u);
}
// x, lo: shared-memory addresses (explicit ld/st.shared: generic accesses were the converter's cost)
__device__ __forceinline__ void split_tf32(uint32_t x, uint32_t lo) {
    float4 v;
    asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(x));
    float4 h, l;
    h.x = tf32_rn(v.x); l.x = tf32_rn(v.x - h.x);
    h.y = tf32_rn(v.y); l.y = tf32_rn(v.y - h.y);
    h.z = tf32_rn(v.z); l.z = tf32_rn(v.z - h.z);
    h.w = tf32_rn(v.w); l.w = tf32_rn(v.w - h.w);
    asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(x), "f"(h.x), "f"(h.y), "f"(h.z), "f"(h.w) : "memory");
    asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(lo), "f"(l.x), "f"(l.y), "f"(l.z), "f"(l.w) : "memory");
}
// SPLIT_NB float4 at once: every load issued before any arithmetic or store, so the shared-memory
// latency is paid once per batch instead of once per float4 (the volatile ld/st of split_tf32 kept
// the converter warps latency-bound: ncu showed the small-N fp32 GEMMs at 16 % tensor activity)
constexpr int SPLIT_NB = 4;
__device__ __forceinline__ void split_tf32_n(uint32_t x, uint32_t lo, uint32_t stride) {
    float4 v[SPLIT_NB];
#pragma unroll
    for (int b = 0; b < SPLIT_NB; ++b)
        asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                     : "=f"(v[b].x), "=f"(v[b].y), "=f"(v[b].z), "=f"(v[b].w) : "r"(x + b * stride));
#pragma unroll
    for (int b = 0; b < SPLIT_NB; ++b) {
        float4 h, l;
        h.x = tf32_rn(v[b].x); l.x = tf32_rn(v[b].x - h.x);
        h.y = tf32_rn(v[b].y); l.y = tf32_rn(v[b].y - h.y);
        h.z = tf32_rn(v[b].z); l.z = tf32_rn(v[b].z - h.z);
        h.w = tf32_rn(v[b].w); l.w = tf32_rn(v[b].w - h.w);
        asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(x + b * stride), "f"(h.x), "f"(h.y), "f"(h.z),
                     "f"(h.w) : "memory");
        asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(lo + b * stride), "f"(l.x), "f"(l.y), "f"(l.z),
                     "f"(l.w) : "memory");
    }
}
// hw_hi variant: only lo = x - trunc_tf32(x) is written; the tensor core's own fp32 -> tf32
// conversion of the untouched x must then be the truncation (BETTY_TF32_HW_HI=1, an experiment)
__device__ __forceinline__ void split_tf32_lo(uint32_t x, uint32_t lo) {
    float4 v;
    asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(x));
    float4 l;
    l.x = v.x - __uint_as_float(__float_as_uint(v.x) & 0xFFFFE000u);
    l.y = v.y - __uint_as_float(__float_as_uint(v.y) & 0xFFFFE000u);
    l.z = v.z - __uint_as_float(__float_as_uint(v.z) & 0xFFFFE000u);
    l.w = v.w - __uint_as_float(__float_as_uint(v.w) & 0xFFFFE000u);
    asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(lo), "f"(l.x), "f"(l.y), "f"(l.z), "f"(l.w) : "memory");
}
__device__ __forceinline__ void zero2_shared(uint32_t x, uint32_t lo) {
    asm volatile("st.shared.v4.u32 [%0], {%1, %1, %1, %1};" ::"r"(x), "r"(0u) : "memory");
    asm volatile("st.shared.v4.u32 [%0], {%1, %1, %1, %1};" ::"r"(lo), "r"(0u) : "memory");
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
__device__ __forceinline__ void sts128(uint32_t a, uint32_t x, uint32_t y, uint32_t z, uint32_t w) {
    asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(x), "r"(y), "r"(z), "r"(w) : "memory");
}

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
constexpr int ESLOTS = 1;                       // staging slots (4 KB) per epilogue warp (bf16 operands)
constexpr int ESLOTS_TF = 1;                    // ... FP32 mode (the 3xTF32 ring needs the room)
constexpr int ROW_THREADS = 64 + 32 * EPI_WARPS;
#ifndef BETTY_RED_CONV
#define BETTY_RED_CONV 4
#endif
#ifndef BETTY_ROW_CONV
#define BETTY_ROW_CONV 2
#endif
constexpr int CONV_WARPS = BETTY_RED_CONV;      // FP32 mode: hi/lo split of each stage (k_tc_red)
constexpr int ROW_CONV_WARPS = BETTY_ROW_CONV;  // ... of each A stage (k_tc_row; keeps the epilogue unspilled)
constexpr int ROW_THREADS_TF = ROW_THREADS + 32 * ROW_CONV_WARPS;
constexpr int MAXCH = 4;                        // 32-column chunks per epilogue half (N <= 256)
constexpr int TQ = 4;                           // tile queue entries (producer -> MMA / epilogue / converters)
struct RowArgs {
    const int64_t* M_dev;
    int K, N, BN, nk, stages;
    void* C; int64_t ldc;
    const void* mask; int64_t ldm; int m_bf16;  // EPI_MASK / EPI_RES_MASK from activations (MBITS = false)
    const uint32_t* mbits; int64_t ldmb;        // ... or from ReLU bits (MBITS = true)
    uint32_t* obits; int64_t ldob;              // EPI_RELU_ONES: ReLU bits out (words per row), or null
    const float* res; int64_t ldr; const int64_t* nres_dev;
    uint32_t tmem_cols;
    int acc_stride;          // TMEM columns of one accumulator (>= BN, multiple of 32)
    int nbuf;                // accumulator buffers (2: the epilogue of tile i overlaps the MMAs of tile i+1)
    int buf_stride;          // TMEM columns between buffers (TF: main + lo-term accumulators)
    int half_cols;           // columns per epilogue half (multiple of 32, <= 32 * MAXCH)
    uint32_t slot_bytes;     // one staging slot: 32 rows x 32 columns
    int bstream;             // 1: B is streamed with A through the ring (B too large to stay resident)
    int hw_hi;               // TF: converter writes lo only (see split_tf32_lo)
    int64_t cend;            // trailing columns [N, cend) of a row are written (ones column / zeros)
    unsigned* tctr;          // [2] dynamic tile claims (next tile, CTAs done; zero between launches), or
                             // null: static round-robin tiles
    int kbb;                 // bytes per row of one k-block: 128 (SWIZZLE_128B), or 64 (TF: SWIZZLE_64B,
                             // half the ring stage -> twice the stages when B streams or sits resident)
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

__device__ __forceinline__ void tmem_st32(uint32_t taddr, const uint32_t* r) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
                 "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};"
                 ::"r"(taddr), "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]),
                   "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]),
                   "r"(r[16]), "r"(r[17]), "r"(r[18]), "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]),
                   "r"(r[24]), "r"(r[25]), "r"(r[26]), "r"(r[27]), "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31])
                 : "memory");
}
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

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
// bf16 (CBF): `part` 1 / 2 = first / second 32 columns of a 64-column pair staged as 128-byte rows
// (SWIZZLE_128B, one TMA store per pair), 0 = a lone chunk as 64-byte rows (SWIZZLE_64B)
template <int EPI, bool CBF>
__device__ __forceinline__ uint32_t chunk_epilogue(const RowArgs& p, const uint32_t* r, int64_t m, int c0, bool ok,
                                                   uint32_t mword, int64_t nres, uint8_t* slot, int lane, int part) {
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
        // (explicit st.shared: the generic stores compiled to ST.E into the shared window)
        if (part == 0) {
            // 64 B rows, SWIZZLE_64B: 16-B chunk c of row r at c ^ ((r >> 1) & 3)
            const uint32_t row = su32(slot) + lane * 64;
#pragma unroll
            for (int c = 0; c < 4; ++c)
                sts128(row + ((c ^ ((lane >> 1) & 3)) << 4), w[4 * c], w[4 * c + 1], w[4 * c + 2], w[4 * c + 3]);
        } else {
            // 128 B rows, SWIZZLE_128B: 16-B chunk cc = 4 (part - 1) + c of row r at cc ^ (r & 7)
            const uint32_t row = su32(slot) + lane * 128;
#pragma unroll
            for (int c = 0; c < 4; ++c)
                sts128(row + (((4 * (part - 1) + c) ^ (lane & 7)) << 4), w[4 * c], w[4 * c + 1], w[4 * c + 2],
                       w[4 * c + 3]);
        }
    } else {
        if (EPI == EPI_RELU_ONES) {
#pragma unroll
            for (int j = 0; j < 32; ++j) bits |= (uint32_t)(v[j] > 0.f) << j;
        }
        // 128 B rows, SWIZZLE_128B: 16-B chunk c of row r at c ^ (r & 7)
        const uint32_t row = su32(slot) + lane * 128;
#pragma unroll
        for (int c = 0; c < 8; ++c)
            sts128(row + ((c ^ (lane & 7)) << 4), __float_as_uint(v[4 * c]), __float_as_uint(v[4 * c + 1]),
                   __float_as_uint(v[4 * c + 2]), __float_as_uint(v[4 * c + 3]));
    }
    return bits;
}

// TF (FP32 mode, 3xTF32): A, B are fp32 words; one k-block is 32 of them (the same 128-byte swizzle
// rows as 64 bf16).  Four converter warps split each landed A stage into hi (in place) and lo, B comes
// pre-split (hi, lo) from the weight prep; per k-block the MMA warp issues lo*hi, hi*lo, hi*hi into
// the same fp32 accumulator (the lo*lo term, ~2^-22 relative, is dropped).
template <int EPI, bool CBF, bool MBITS, bool TF>
__global__ void __launch_bounds__(TF ? ROW_THREADS_TF : ROW_THREADS, 1)
k_tc_row(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
         const __grid_constant__ CUtensorMap tmC, const __grid_constant__ CUtensorMap tmBlo,
         const __grid_constant__ CUtensorMap tmC2, RowArgs p) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    constexpr int ES = TF ? ESLOTS_TF : ESLOTS;
    constexpr int NSPLIT = TF ? 2 : 1;                       // hi (+ lo) copies of each operand block
    const int S = p.stages;
    const uint32_t a_bytes = BM * p.kbb;                     // one A k-block: 128 rows x kbb bytes
    const uint32_t bblk = (uint32_t)p.BN * p.kbb;            // one K-block of B
    // one ring stage: A (+ A lo) (+ B (+ B lo) when streamed)
    const uint32_t ring_bytes = NSPLIT * (a_bytes + (p.bstream ? bblk : 0u));
    uint8_t* bres = smem;                                    // NSPLIT * nk * bblk (resident B) or nothing
    uint8_t* aring = smem + (p.bstream ? 0 : NSPLIT * p.nk * bblk);   // S * ring_bytes
    uint8_t* stage = aring + S * ring_bytes;                 // EPI_WARPS * ES * slot_bytes
    uint64_t* full = (uint64_t*)(stage + EPI_WARPS * ES * p.slot_bytes);
    uint64_t* empty = full + S;
    uint64_t* tfull = empty + S;      // [2]
    uint64_t* tempty = tfull + 2;     // [2]
    uint64_t* bfull = tempty + 2;     // [1]
    uint64_t* conv = bfull + 1;       // [S] (TF) A stage split into hi / lo
    uint64_t* tqf = conv + (TF ? S : 0);   // [TQ] tile queue: entry published by the producer
    uint64_t* tqe = tqf + TQ;              // [TQ] ... read by every consumer warp
    int32_t* tq = (int32_t*)(tqe + TQ);    // [TQ] tile ids (-1: no more tiles)
    uint32_t* tslot = (uint32_t*)(tq + TQ);

    const int warp = threadIdx.x >> 5;
    const int64_t M = *p.M_dev;
    const int64_t tiles = (M + BM - 1) / BM;
    // consumers of a queue entry: the MMA warp, the epilogue warps (+ the converter warps)
    constexpr int TQ_READERS = 1 + EPI_WARPS + (TF ? ROW_CONV_WARPS : 0);
    // one warp's read of the next queue entry (every lane gets the tile id)
    int tq_i = 0;
    uint32_t tq_ph = 0;
    auto tq_pop = [&]() -> int64_t {
        mbar_wait(&tqf[tq_i], tq_ph);
        const int32_t t = tq[tq_i];
        __syncwarp();
        if ((threadIdx.x & 31) == 0) mbar_arrive(&tqe[tq_i]);
        if (++tq_i == TQ) { tq_i = 0; tq_ph ^= 1; }
        return t;
    };

    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
        for (int a = 0; a < 2; ++a) { mbar_init(&tfull[a], 1); mbar_init(&tempty[a], 32 * EPI_WARPS); }
        mbar_init(bfull, 1);
        if (TF) for (int s = 0; s < S; ++s) mbar_init(&conv[s], ROW_CONV_WARPS);
        for (int i = 0; i < TQ; ++i) { mbar_init(&tqf[i], 1); mbar_init(&tqe[i], TQ_READERS); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmA) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmB) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmC) : "memory");
        if (CBF) asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmC2) : "memory");
        if (TF) asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmBlo) : "memory");
    }
    if (warp == 1) tmem_alloc_warp(tslot, p.tmem_cols);
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tmem = *tslot;

    if (warp == 0) {
        if (elect_lane0()) {
            const int KE = TF ? p.kbb / 4 : BK;              // elements per k-block
            // TF stage: [A | A lo | B | B lo]; TMA fills A, B, B lo (the converter writes A lo)
            const uint32_t land = ring_bytes - (TF ? a_bytes : 0u);
            int s = 0;
            uint32_t ph = 0;
            int q = 0;
            uint32_t qph = 0;
            bool bload = !p.bstream;
            // Tiles are claimed one at a time from a global counter (p.tctr) and queued for the other
            // roles, so a CTA that starts late (its SM still held by a concurrent kernel, e.g. the REG
            // on the side stream) takes fewer tiles instead of delaying the whole GEMM; each output
            // row is still computed by exactly one CTA, so the result does not depend on the order.
            int64_t tn = p.tctr ? (int64_t)atomicAdd(p.tctr, 1u) : (int64_t)blockIdx.x;
            for (;;) {
                const int64_t t = tn;
                const bool end = t >= tiles;
                mbar_wait(&tqe[q], qph ^ 1);
                tq[q] = end ? -1 : (int32_t)t;
                mbar_arrive(&tqf[q]);
                if (++q == TQ) { q = 0; qph ^= 1; }
                if (end) break;
                // the next claim's round trip overlaps this tile's loads
                tn = p.tctr ? (int64_t)atomicAdd(p.tctr, 1u) : t + gridDim.x;
                if (bload) {                                 // B resident: loaded before the first tile
                    bload = false;
                    mbar_expect_tx(bfull, NSPLIT * p.nk * bblk);
                    for (int kb = 0; kb < p.nk; ++kb) {
                        tma_2d(bres + kb * bblk, &tmB, kb * KE, 0, bfull);
                        if (TF) tma_2d(bres + (p.nk + kb) * bblk, &tmBlo, kb * KE, 0, bfull);
                    }
                }
                for (int kb = 0; kb < p.nk; ++kb) {
                    mbar_wait(&empty[s], ph ^ 1);
                    mbar_expect_tx(&full[s], land);
                    uint8_t* st = aring + s * ring_bytes;
                    tma_2d(st, &tmA, kb * KE, (int)(t * BM), &full[s]);
                    if (p.bstream) {
                        tma_2d(st + NSPLIT * a_bytes, &tmB, kb * KE, 0, &full[s]);
                        if (TF) tma_2d(st + NSPLIT * a_bytes + bblk, &tmBlo, kb * KE, 0, &full[s]);
                    }
                    if (++s == S) { s = 0; ph ^= 1; }
                }
            }
        }
    } else if (warp == 1) {
        const uint32_t idesc = TF ? idesc_tf32(BM, p.BN, 0, 0) : idesc_bf16(BM, p.BN, 0, 0);
        int s = 0;
        uint32_t ph = 0;
        int it = 0;
        bool bready = p.bstream;
        for (;; ++it) {
            if (tq_pop() < 0) break;
            if (!bready) { mbar_wait(bfull, 0); bready = true; }
            const int acc = it % p.nbuf;
            const uint32_t aph = (it / p.nbuf) & 1;
            mbar_wait(&tempty[acc], aph ^ 1);
            fence_after();
            const uint32_t d = tmem + acc * p.buf_stride;
            for (int kb = 0; kb < p.nk; ++kb) {
                mbar_wait(TF ? &conv[s] : &full[s], ph);
                fence_after();
                if (elect_lane0()) {
                    const uint32_t a0 = su32(aring + s * ring_bytes);
                    const uint32_t b0 = p.bstream ? a0 + NSPLIT * a_bytes : su32(bres + kb * bblk);
                    if (TF) {
                        // 4 MMAs of K = 8 fp32 words (32 B) per 128-byte k-block, per product term.  The
                        // small terms go to their own accumulator (d + acc_stride): the tensor core's
                        // fp32 accumulation rounds toward zero (~2e-8 relative per accumulation into a
                        // growing sum), so the main sum gets only the K/8 hi*hi accumulations
                        const uint32_t alo = a0 + a_bytes;
                        const uint32_t blo = p.bstream ? b0 + bblk : su32(bres + (p.nk + kb) * bblk);
                        const uint32_t dl = d + p.acc_stride;
                        // K = 8 fp32 (32 B) per MMA; 8-row swizzle atoms of kbb bytes per row (SBO = 8 kbb)
                        const int nks = p.kbb / 32;
                        const uint32_t sbo = 8u * (uint32_t)p.kbb, lay = p.kbb == 128 ? 2u : 4u;
                        for (int k = 0; k < nks; ++k)
                            umma_tf32(dl, sdesc(alo + k * 32, 0, sbo, lay), sdesc(b0 + k * 32, 0, sbo, lay), idesc,
                                      (kb | k) != 0);
                        for (int k = 0; k < nks; ++k)
                            umma_tf32(dl, sdesc(a0 + k * 32, 0, sbo, lay), sdesc(blo + k * 32, 0, sbo, lay), idesc, 1);
                        for (int k = 0; k < nks; ++k)
                            umma_tf32(d, sdesc(a0 + k * 32, 0, sbo, lay), sdesc(b0 + k * 32, 0, sbo, lay), idesc,
                                      (kb | k) != 0);
                    } else {
#pragma unroll
                        for (int k = 0; k < BK / UK; ++k) {
                            const uint64_t ad = sdesc(a0 + k * UK * 2, 0, 1024);
                            const uint64_t bd = sdesc(b0 + k * UK * 2, 0, 1024);
                            umma_f16(d, ad, bd, idesc, (kb | k) != 0);
                        }
                    }
                    umma_commit(&empty[s]);
                    if (kb == p.nk - 1) umma_commit(&tfull[acc]);
                }
                __syncwarp();
                if (++s == S) { s = 0; ph ^= 1; }
            }
        }
    } else if (TF && warp >= 2 + EPI_WARPS) {
        // converter warps: split each landed A k-block (128 rows x 32 fp32) into hi (in place) and lo
        const int tid = (warp - 2 - EPI_WARPS) * 32 + (threadIdx.x & 31);
        int s = 0;
        uint32_t ph = 0;
        while (tq_pop() >= 0) {
            for (int kb = 0; kb < p.nk; ++kb) {
                mbar_wait(&full[s], ph);
                const uint32_t a = su32(aring + s * ring_bytes);
                if (p.hw_hi) {
#pragma unroll 4
                    for (int i = tid; i < (int)(a_bytes / 16); i += 32 * ROW_CONV_WARPS)
                        split_tf32_lo(a + 16 * i, a + a_bytes + 16 * i);
                } else {
                    constexpr int STEP = 32 * ROW_CONV_WARPS;
                    const int n16 = (int)(a_bytes / 16);
                    int i = tid;
                    for (; i + (SPLIT_NB - 1) * STEP < n16; i += SPLIT_NB * STEP)
                        split_tf32_n(a + 16 * i, a + a_bytes + 16 * i, 16 * STEP);
                    for (; i < n16; i += STEP) split_tf32(a + 16 * i, a + a_bytes + 16 * i);
                }
                fence_proxy_async();             // generic-proxy writes -> visible to the tensor core
                __syncwarp();
                if ((threadIdx.x & 31) == 0) mbar_arrive(&conv[s]);
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
        uint8_t* my_stage = stage + ew * ES * p.slot_bytes;
        int slot = 0;
        int it = 0;
        // ReLU' bit words of this thread's row, one tile ahead (short-K layers finish the MMA long
        // before a load round trip, so loading them at the top of the tile left them exposed)
        uint32_t mw_next[MAXCH];
#pragma unroll
        for (int ci = 0; ci < MAXCH; ++ci) mw_next[ci] = 0u;
        auto load_bits = [&](int64_t tt, uint32_t (&dst)[MAXCH]) {
            const int64_t mm = tt * BM + q * 32 + lane;
            if (tt >= 0 && tt < tiles && mm < M) {
                const uint32_t* wb = p.mbits + mm * p.ldmb + cbeg / 32;
#pragma unroll
                for (int ci = 0; ci < MAXCH; ++ci) if (ci < nch) dst[ci] = wb[ci];
            }
        };
        // the queue is read one entry ahead: the next tile's ReLU' bits are prefetched during this one
        int64_t t_next = tq_pop();
        if (HAS_MASK && MBITS) load_bits(t_next, mw_next);
        for (int64_t t = t_next; t >= 0; t = t_next, ++it) {
            t_next = tq_pop();
            const int acc = it % p.nbuf;
            const uint32_t aph = (it / p.nbuf) & 1;
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
                    load_bits(t_next, mw_next);
                } else {
#pragma unroll
                    for (int ci = 0; ci < MAXCH; ++ci) if (ci < nch) mw[ci] = mask_word_from_act(p, m, cbeg + 32 * ci, ok);
                }
            }
            mbar_wait(&tfull[acc], aph);
            fence_after();
            const uint32_t tbase = tmem + ((uint32_t)(q * 32) << 16) + acc * p.buf_stride;
            uint32_t ra[32], rb[32];
            uint32_t obits[MAXCH];
            if constexpr (TF) {
                // main + lo-term accumulators, summed with round-to-nearest fp32 adds
#pragma unroll
                for (int ci = 0; ci < MAXCH; ++ci) {
                    obits[ci] = 0u;
                    if (ci < nch) {
                        const int c0 = cbeg + 32 * ci;
                        tmem_ld32_nowait(tbase + c0, ra);
                        tmem_ld32_nowait(tbase + p.acc_stride + c0, rb);
                        tmem_wait_regs(ra);
                        tmem_wait_regs(rb);
#pragma unroll
                        for (int j = 0; j < 32; ++j) ra[j] = __float_as_uint(__uint_as_float(ra[j]) + __uint_as_float(rb[j]));
                        uint8_t* sl = my_stage + slot * p.slot_bytes;
                        if (lane == 0) bulk_wait_read<ES - 1>();
                        __syncwarp();
                        obits[ci] = chunk_epilogue<EPI, CBF>(p, ra, m, c0, ok, mw[ci], nres, sl, lane, 0);
                        fence_proxy_async();
                        __syncwarp();
                        if (lane == 0) {
                            tma_store_2d(&tmC, sl, c0, (int)row0);
                            bulk_commit();
                        }
                        if (++slot == ES) slot = 0;
                    }
                }
            } else {
            if (nch > 0) { tmem_ld32_nowait(tbase + cbeg, ra); tmem_wait_regs(ra); }
#pragma unroll
            for (int ci = 0; ci < MAXCH; ++ci) {
                obits[ci] = 0u;
                if (ci < nch) {
                    uint32_t* cur = (ci & 1) ? rb : ra;
                    uint32_t* nxt = (ci & 1) ? ra : rb;
                    const int c0 = cbeg + 32 * ci;
                    if (ci + 1 < nch) tmem_ld32_nowait(tbase + c0 + 32, nxt);   // next chunk in flight
                    // bf16: chunks (0,1), (2,3) of the half share a slot and one 64-column store
                    const bool second = CBF && (ci & 1) != 0;
                    const bool paired = CBF && (second || ci + 1 < nch);
                    const int part = paired ? (second ? 2 : 1) : 0;
                    uint8_t* sl = my_stage + slot * p.slot_bytes;
                    if (!second) {
                        if (lane == 0) bulk_wait_read<ES - 1>();    // the store that used this slot has read it
                        __syncwarp();
                    }
                    obits[ci] = chunk_epilogue<EPI, CBF>(p, cur, m, c0, ok, mw[ci], nres, sl, lane, part);
                    if (second || !paired) {
                        fence_proxy_async();
                        __syncwarp();
                        if (lane == 0) {
                            if (part == 2) tma_store_2d(&tmC2, sl, c0 - 32, (int)row0);
                            else tma_store_2d(&tmC, sl, c0, (int)row0);
                            bulk_commit();
                        }
                        if (++slot == ES) slot = 0;
                    }
                    if (ci + 1 < nch) tmem_wait_regs(nxt);
                }
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
    // the last CTA to finish resets the tile counter for the next launch (every claim, the one past
    // the last tile included, happened before its CTA got here)
    if (p.tctr && threadIdx.x == 0) {
        fence_gpu();
        if (atomicAdd(&p.tctr[1], 1u) == gridDim.x - 1) {
            p.tctr[0] = 0;
            p.tctr[1] = 0;
            fence_gpu();
        }
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
    uint32_t sbo;              // TF: byte stride between 4-row K atoms (512)
    int hw_hi;                 // TF: converter writes lo only (see split_tf32_lo)
};

// TF (FP32 mode, 3xTF32): fp32 operands, k-blocks of 16 nodes (boxes of 32 features x 16 nodes, the
// same 128-byte swizzle rows), four converter warps split both operands of each landed stage into hi
// (in place) and lo (a second copy of the stage) and zero the rows past M; three MMA terms per step.
// The tensor core's fp32 accumulation rounds toward zero (measured: ~2e-8 relative shrink per MMA
// accumulation into a growing sum), so a CTA's long reduction over nodes is NOT left in one
// accumulator: every RED_SB k-blocks (64 nodes, 24 accumulations) the epilogue warps add the TMEM
// accumulator into a TMEM running total with round-to-nearest fp32 adds (one feature tile per CTA,
// TMEM = accumulator + total).
constexpr int RED_THREADS_TF = THREADS + 32 * CONV_WARPS;
// TKN (fp32 mode): nodes per k-block -- 16, or 32 for narrow B (N <= 64: a k-block's MMAs are short,
// so per-k-block barrier / converter / issue overhead dominated; C3 fp32 step 10.57 -> 10.31 ms with
// 32 everywhere, while the N = 256 dW0 was faster with 16); RED_SB k-blocks = 64 nodes per drain
template <bool TF, int TKN>
__global__ void __launch_bounds__(TF ? RED_THREADS_TF : THREADS, 1)
k_tc_red(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB, RedArgs p) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    constexpr int KN = TF ? TKN : BK;                 // nodes (reduction rows) per k-block
    constexpr int RED_SB = 64 / TKN;
    const int S = p.stages;
    const uint32_t box = KN * 128;                    // KN rows x 128 B (64 bf16 / 32 fp32 features)
    const int nbA_cta = p.nbA * p.mt_cta;             // A boxes per stage
    const uint32_t a_bytes = nbA_cta * box, b_bytes = p.nbB * box;
    const uint32_t raw_bytes = a_bytes + b_bytes;
    const uint32_t stage_bytes = raw_bytes * (TF ? 2 : 1);   // TF: + the lo copy
    uint64_t* full = (uint64_t*)(smem + S * stage_bytes);
    uint64_t* empty = full + S;
    uint64_t* tfull = empty + S;
    uint64_t* tempty_r = tfull + 1;                   // [1] (TF) accumulator drained into the total
    uint64_t* conv = tempty_r + 1;                    // [S] (TF)
    uint32_t* tslot = (uint32_t*)(conv + (TF ? S : 0));

    const int warp = threadIdx.x >> 5;
    const int nsplit = p.mt_cta == 1 ? p.mtiles : 1;
    const int mt0 = p.mt_cta == 1 ? blockIdx.x % p.mtiles : 0;
    const int split = blockIdx.x / nsplit;
    const int64_t M = *p.M_dev;
    const int64_t nkb = (M + KN - 1) / KN;
    const int64_t kb0 = nkb * split / p.S, kb1 = nkb * (split + 1) / p.S;
    const int fbox = TF ? 32 : 64;                    // features per box

    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
        mbar_init(&tfull[0], 1);
        mbar_init(&tempty_r[0], 128);
        if (TF) for (int s = 0; s < S; ++s) mbar_init(&conv[s], CONV_WARPS);
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
                mbar_expect_tx(&full[s], raw_bytes);
                for (int i = 0; i < nbA_cta; ++i) tma_2d(sa + i * box, &tmA, mt0 * BM + i * fbox, (int)(kb * KN), &full[s]);
                for (int i = 0; i < p.nbB; ++i) tma_2d(sa + a_bytes + i * box, &tmB, i * fbox, (int)(kb * KN), &full[s]);
                if (++s == S) { s = 0; ph ^= 1; }
            }
        }
    } else if (warp == 1) {
        const uint32_t idesc = TF ? idesc_tf32(BM, p.BN, 1, 1) : idesc_bf16(BM, p.BN, 1, 1);
        int s = 0;
        uint32_t ph = 0;
        for (int64_t kb = kb0; kb < kb1; ++kb) {
            uint8_t* sa = smem + s * stage_bytes;
            const int64_t sb = (kb - kb0) / RED_SB;          // TF: super-block index
            const bool sb_first = TF && (kb - kb0) % RED_SB == 0;
            const bool sb_last = TF && ((kb - kb0) % RED_SB == RED_SB - 1 || kb == kb1 - 1);
            if (sb_first && sb > 0) {                        // the epilogue has drained the accumulator
                mbar_wait(&tempty_r[0], (uint32_t)((sb - 1) & 1));
                fence_after();
            }
            if (TF) {
                mbar_wait(&conv[s], ph);
            } else {
                mbar_wait(&full[s], ph);
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
            }
            fence_after();
            if (elect_lane0()) {
                const uint32_t b0 = su32(sa) + a_bytes;
                if (TF) {
                    // MN-major tf32, SWIZZLE_128B_BASE32B: atoms of 32 (MN) x 4 (K) rows of 128 B (SBO = 512
                    // between the two atoms one K = 8 MMA spans), LBO = box between 32-feature columns
                    for (int mt = 0; mt < p.mt_cta; ++mt) {
                        const uint32_t a0 = su32(sa) + mt * p.nbA * box;
#pragma unroll
                        for (int k = 0; k < KN / 8; ++k) {
                            const uint64_t ah = sdesc(a0 + k * 1024, box, p.sbo, 1), al = sdesc(a0 + raw_bytes + k * 1024, box, p.sbo, 1);
                            const uint64_t bh = sdesc(b0 + k * 1024, box, p.sbo, 1), bl = sdesc(b0 + raw_bytes + k * 1024, box, p.sbo, 1);
                            const uint32_t d = tmem + mt * p.acc_stride;
                            umma_tf32(d, al, bh, idesc, (!sb_first || k != 0));
                            umma_tf32(d, ah, bl, idesc, 1);
                            umma_tf32(d, ah, bh, idesc, 1);
                        }
                    }
                } else {
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
                }
                umma_commit(&empty[s]);
                if (TF ? sb_last : kb == kb1 - 1) umma_commit(&tfull[0]);
            }
            __syncwarp();
            if (++s == S) { s = 0; ph ^= 1; }
        }
    } else if (TF && warp >= 2 + 4) {
        // converter warps: hi in place, lo into the second half of the stage, rows >= M zeroed
        const int tid = (warp - 6) * 32 + (threadIdx.x & 31);
        int s = 0;
        uint32_t ph = 0;
        for (int64_t kb = kb0; kb < kb1; ++kb) {
            mbar_wait(&full[s], ph);
            const uint32_t sa = su32(smem + s * stage_bytes);
            const int64_t valid = M - kb * KN;
            const int n16 = (int)(raw_bytes / 16);
            if (valid >= KN && p.hw_hi) {
#pragma unroll 4
                for (int i = tid; i < n16; i += 32 * CONV_WARPS) split_tf32_lo(sa + 16 * i, sa + raw_bytes + 16 * i);
            } else if (valid >= KN) {
                constexpr int STEP = 32 * CONV_WARPS;
                int i = tid;
                for (; i + (SPLIT_NB - 1) * STEP < n16; i += SPLIT_NB * STEP)
                    split_tf32_n(sa + 16 * i, sa + raw_bytes + 16 * i, 16 * STEP);
                for (; i < n16; i += STEP) split_tf32(sa + 16 * i, sa + raw_bytes + 16 * i);
            } else {                                     // the last k-block: rows >= M are zeroed
                for (int i = tid; i < n16; i += 32 * CONV_WARPS) {
                    const int row = (i >> 3) & (KN - 1); // 8 float4 per 128-byte row, KN rows per box
                    if (row < (int)valid) split_tf32(sa + 16 * i, sa + raw_bytes + 16 * i);
                    else zero2_shared(sa + 16 * i, sa + raw_bytes + 16 * i);
                }
            }
            fence_proxy_async();
            __syncwarp();
            if ((threadIdx.x & 31) == 0) mbar_arrive(&conv[s]);
            if (++s == S) { s = 0; ph ^= 1; }
        }
    } else {
        const int q = warp & 3;
        const int r_in = q * 32 + (threadIdx.x & 31);
        if (TF) {
            // drain each super-block's accumulator (columns [0, acc_stride)) into the running total
            // (columns [acc_stride, 2 acc_stride)) with round-to-nearest fp32 adds; the total ends
            // in the accumulator columns' place for the write-out below
            const uint32_t lane_base = tmem + ((uint32_t)(q * 32) << 16);
            const int64_t nsb = (kb1 - kb0 + RED_SB - 1) / RED_SB;
            for (int64_t sb = 0; sb < nsb; ++sb) {
                mbar_wait(&tfull[0], (uint32_t)(sb & 1));
                fence_after();
                for (int c0 = 0; c0 < p.BN; c0 += 32) {
                    uint32_t a[32], t[32];
                    tmem_ld32_nowait(lane_base + c0, a);
                    if (sb > 0) tmem_ld32_nowait(lane_base + p.acc_stride + c0, t);
                    tmem_wait_regs(a);
                    if (sb > 0) {
                        tmem_wait_regs(t);
#pragma unroll
                        for (int j = 0; j < 32; ++j) t[j] = __float_as_uint(__uint_as_float(t[j]) + __uint_as_float(a[j]));
                    } else {
#pragma unroll
                        for (int j = 0; j < 32; ++j) t[j] = a[j];
                    }
                    tmem_st32(lane_base + p.acc_stride + c0, t);
                }
                tmem_wait_st();
                fence_before();
                mbar_arrive(&tempty_r[0]);
            }
        } else if (kb1 > kb0) {
            mbar_wait(&tfull[0], 0);
            fence_after();
        }
        for (int mt = 0; mt < p.mt_cta; ++mt) {
            const int feat = (mt0 + mt) * BM + r_in;
            float* out = p.partials + ((int64_t)split * p.K1 + feat) * p.N;
            for (int c0 = 0; c0 < p.BN; c0 += 32) {
                float v[32];
                if (kb1 > kb0) tmem_ld32(tmem + ((uint32_t)(q * 32) << 16) + (TF ? p.acc_stride : mt * p.acc_stride) + c0, v);
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
bool gemm_row_tc(betty_ctx* c, const GemmRow& g, const void* Bk, const void* Bk_lo, int64_t ldbk, cudaStream_t s) {
    using namespace tc;
    // TF: FP32 mode (fp32 A, B hi / lo, fp32 C) as 3xTF32; else bf16 operands
    const bool TF = !g.a_bf16;
    if (TF && (g.b_bf16 || g.c_bf16 || !Bk_lo || (g.lda & 3) || (ldbk & 3))) return false;
    if (!TF && (!g.a_bf16 || !g.b_bf16 || (g.lda & 7) || (ldbk & 7))) return false;
    if (g.N > 256 || g.N < 1) return false;
    if ((g.epi == EPI_MASK || g.epi == EPI_RES_MASK) && !g.mbits && (g.ldm & (g.m_bf16 ? 7 : 3))) return false;
    const int NS = TF ? 2 : 1;                  // hi (+ lo) copies
    const int BN = (g.N + 15) / 16 * 16;
    const uint32_t slot_bytes = 32 * 128;       // 32 rows x 128 B (bf16: a 64-column pair; fp32: 32 columns)
    const size_t stage_bytes = (size_t)EPI_WARPS * (TF ? ESLOTS_TF : ESLOTS) * slot_bytes;
    const size_t budget = 227 * 1024;           // the sm_100 opt-in maximum of dynamic shared memory per CTA
    // k-block row bytes: 128 for bf16; 64 in fp32 (TF) mode, where B hi + lo (resident or streamed) and
    // the lo copy of every A stage left room for a 2-deep ring only (the wide fp32 forward: 1.73 -> 1.57
    // ms).  C3 fp32 step, two runs each: 64 everywhere 10.14 / 10.09 ms, 64 only where B streams
    // 10.27 / 10.22, 128 everywhere 10.31 / 10.32.  BETTY_TF_KBB=128 restores the 128-byte layout.
    static const int kbb_env = getenv("BETTY_TF_KBB") ? atoi(getenv("BETTY_TF_KBB")) : 0;
    int kbb = 128;
    int KE = 0, nk = 0;
    size_t bblk = 0, b_bytes = 0, a_bytes = 0, ring = 0, fixed = 0;
    bool bstream = false;
    for (int pass = 0; pass < 2; ++pass) {
        KE = TF ? kbb / 4 : BK;                 // elements per k-block
        nk = (g.K + KE - 1) / KE;
        bblk = (size_t)BN * kbb;
        b_bytes = (size_t)nk * bblk * NS;
        a_bytes = (size_t)BM * kbb * NS;
        // B resident when it fits next to a 2-stage A ring, else streamed with A
        bstream = b_bytes + stage_bytes + 2 * a_bytes + 1024 + 512 > budget;   // 512: barriers, tile queue
        ring = a_bytes + (bstream ? bblk * NS : 0);
        fixed = (bstream ? 0 : b_bytes) + stage_bytes + 1024 + 512;
        const bool want64 = TF && kbb_env != 128;
        if (pass == 0 && want64) { kbb = 64; continue; }
        break;
    }
    if (fixed + 2 * ring > budget) return false;
    const CUtensorMapSwizzle swz = kbb == 128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B;
    CUtensorMap ma, mb, mc, mbl, mc2;
    if (!make_map_t(&ma, g.A, TF, g.K, g.M_cap, g.lda, KE, BM, swz) ||
        !make_map_t(&mb, Bk, TF, g.K, g.N, ldbk, KE, BN, swz))
        return false;
    if (TF && !make_map_t(&mbl, Bk_lo, true, g.K, g.N, ldbk, KE, BN, swz)) return false;
    if (!TF) mbl = mb;
    if (!make_map_t(&mc, g.C, !g.c_bf16, g.N, g.M_cap, g.ldc, 32, 32,
                    g.c_bf16 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_128B))
        return false;
    // bf16 C: 64-column boxes of 128-byte rows for paired chunks (half the store row segments; the
    // bf16-storing GEMMs ran at ~4.7 TB/s against 6.5 for the fp32-storing one, ncu r03)
    if (g.c_bf16) {
        if (!make_map_t(&mc2, g.C, false, g.N, g.M_cap, g.ldc, 64, 32, CU_TENSOR_MAP_SWIZZLE_128B)) return false;
    } else {
        mc2 = mc;
    }
    RowArgs p{};
    p.M_dev = g.M_dev; p.K = g.K; p.N = g.N; p.BN = BN; p.nk = nk; p.kbb = kbb;
    // dynamic tile claims (BETTY_GEMM_STATIC=1: the round-robin assignment, for A/B runs)
    static const bool gemm_static = getenv("BETTY_GEMM_STATIC") && atoi(getenv("BETTY_GEMM_STATIC")) != 0;
    p.tctr = gemm_static ? nullptr : c->L().counters + CTR_GEMM;
    p.stages = (int)std::max<size_t>(2, std::min<size_t>(8, (budget - fixed) / ring));
    p.bstream = bstream ? 1 : 0;
    static const int hw_hi_row = getenv("BETTY_TF32_HW_HI") ? atoi(getenv("BETTY_TF32_HW_HI")) : 0;
    p.hw_hi = hw_hi_row;
    p.C = g.C; p.ldc = g.ldc; p.cend = g.cend > 0 ? g.cend : g.ldc;
    p.mask = g.mask; p.ldm = g.ldm; p.m_bf16 = g.m_bf16; p.res = g.res; p.ldr = g.ldr; p.nres_dev = g.nres_dev;
    p.mbits = g.mbits; p.ldmb = g.ldmb;
    p.obits = g.epi == EPI_RELU_ONES ? g.obits : nullptr; p.ldob = g.ldob;
    p.acc_stride = (BN + 31) / 32 * 32;
    p.buf_stride = (TF ? 2 : 1) * p.acc_stride;
    p.nbuf = 2 * p.buf_stride <= 512 ? 2 : 1;
    p.tmem_cols = tmem_cols_for(p.nbuf * p.buf_stride);
    p.half_cols = ((BN + 63) / 64) * 32;
    p.slot_bytes = slot_bytes;
    if (p.tmem_cols > 512 || p.half_cols > 32 * MAXCH) return false;
    const size_t smem = fixed + (size_t)p.stages * ring;
    const int64_t tiles = (g.M_cap + BM - 1) / BM;
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(tiles, c->num_sms));
    const bool usebits = g.mbits != nullptr;
#define ROW_LAUNCH(E, CB, MB, T)                                                                   \
    do {                                                                                           \
        static bool attr = false;                                                                  \
        if (!attr) {                                                                               \
            cudaFuncSetAttribute(k_tc_row<E, CB, MB, T>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024); \
            attr = true;                                                                           \
        }                                                                                          \
        k_tc_row<E, CB, MB, T><<<grid, T ? ROW_THREADS_TF : ROW_THREADS, smem, s>>>(ma, mb, mc, mbl, mc2, p); \
    } while (0)
    if (TF) {
        switch (g.epi) {
        case EPI_STORE: ROW_LAUNCH(EPI_STORE, false, false, true); break;
        case EPI_RELU_ONES: ROW_LAUNCH(EPI_RELU_ONES, false, false, true); break;
        case EPI_MASK:
            if (usebits) ROW_LAUNCH(EPI_MASK, false, true, true); else ROW_LAUNCH(EPI_MASK, false, false, true);
            break;
        default:
            if (usebits) ROW_LAUNCH(EPI_RES_MASK, false, true, true); else ROW_LAUNCH(EPI_RES_MASK, false, false, true);
            break;
        }
        return true;
    }
    switch (g.epi) {
    case EPI_STORE:
        if (g.c_bf16) ROW_LAUNCH(EPI_STORE, true, false, false); else ROW_LAUNCH(EPI_STORE, false, false, false);
        break;
    case EPI_RELU_ONES:
        if (g.c_bf16) ROW_LAUNCH(EPI_RELU_ONES, true, false, false); else ROW_LAUNCH(EPI_RELU_ONES, false, false, false);
        break;
    case EPI_MASK:
        if (g.c_bf16) { if (usebits) ROW_LAUNCH(EPI_MASK, true, true, false); else ROW_LAUNCH(EPI_MASK, true, false, false); }
        else { if (usebits) ROW_LAUNCH(EPI_MASK, false, true, false); else ROW_LAUNCH(EPI_MASK, false, false, false); }
        break;
    default:
        if (g.c_bf16) { if (usebits) ROW_LAUNCH(EPI_RES_MASK, true, true, false); else ROW_LAUNCH(EPI_RES_MASK, true, false, false); }
        else { if (usebits) ROW_LAUNCH(EPI_RES_MASK, false, true, false); else ROW_LAUNCH(EPI_RES_MASK, false, false, false); }
        break;
    }
#undef ROW_LAUNCH
    return true;
}

bool gemm_red_tc(betty_ctx* c, const GemmRed& g, int* S_used, cudaStream_t s) {
    using namespace tc;
    const bool TF = !g.a_bf16;
    if (TF && (g.b_bf16 || (g.lda & 3) || (g.ldb & 3))) return false;
    if (!TF && (!g.a_bf16 || !g.b_bf16 || (g.lda & 7) || (g.ldb & 7))) return false;
    if (g.N > 256) return false;
    const int tkn = g.N <= 64 ? 32 : 16;        // fp32 mode: nodes per k-block (see k_tc_red)
    const int KN = TF ? tkn : BK, fbox = TF ? 32 : 64;
    const int BN = (g.N + 15) / 16 * 16;
    CUtensorMap ma, mb;
    const CUtensorMapSwizzle sw = TF ? CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B : CU_TENSOR_MAP_SWIZZLE_128B;
    if (!make_map_t(&ma, g.A, TF, g.K1, g.M_cap, g.lda, fbox, KN, sw) ||
        !make_map_t(&mb, g.B, TF, g.N, g.M_cap, g.ldb, fbox, KN, sw))
        return false;
    RedArgs p{};
    p.M_dev = g.M_dev; p.K1 = g.K1; p.N = g.N; p.BN = BN;
    p.nbA = BM / fbox; p.nbB = (BN + fbox - 1) / fbox;
    p.mtiles = (g.K1 + BM - 1) / BM;
    p.acc_stride = (BN + 31) / 32 * 32;
    // all feature tiles in one CTA when their accumulators fit TMEM and a stage fits 3x in smem:
    // A and B are then read exactly once
    const int mult = TF ? 2 : 1;
    const int stage_all = (p.nbA * p.mtiles + p.nbB) * KN * 128 * mult;
    // TF: one feature tile per CTA (TMEM holds its accumulator and the running total)
    p.mt_cta = (!TF && p.mtiles * p.acc_stride <= 512 && 3 * stage_all <= 200 * 1024) ? p.mtiles : 1;
    const int stage_bytes = (p.nbA * p.mt_cta + p.nbB) * KN * 128 * mult;
    p.stages = std::max(2, std::min(8, (200 * 1024) / stage_bytes));
    // one CTA per SM: TF runs one feature tile per CTA, so mtiles x S CTAs (fewer splits than planned)
    p.S = TF ? std::max(1, std::min(g.S, c->num_sms / std::max(1, p.mtiles))) : g.S;
    *S_used = p.S;
    p.partials = g.partials;
    p.tmem_cols = tmem_cols_for((TF ? 2 : p.mt_cta) * p.acc_stride);
    static const uint32_t sbo_env = getenv("BETTY_TF_SBO") ? (uint32_t)atoi(getenv("BETTY_TF_SBO")) : 512u;
    p.sbo = sbo_env;
    static const int hw_hi = getenv("BETTY_TF32_HW_HI") ? atoi(getenv("BETTY_TF32_HW_HI")) : 0;
    p.hw_hi = hw_hi;
    const size_t smem = (size_t)p.stages * stage_bytes + 1024 + 256;
    const int grid = (p.mt_cta == 1 ? p.mtiles : 1) * p.S;
    if (TF) {
        static bool attr = false;
        if (!attr) {
            cudaFuncSetAttribute(k_tc_red<true, 16>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
            cudaFuncSetAttribute(k_tc_red<true, 32>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
            attr = true;
        }
        if (tkn == 32) k_tc_red<true, 32><<<grid, RED_THREADS_TF, smem, s>>>(ma, mb, p);
        else k_tc_red<true, 16><<<grid, RED_THREADS_TF, smem, s>>>(ma, mb, p);
    } else {
        static bool attr = false;
        if (!attr) {
            cudaFuncSetAttribute(k_tc_red<false, 16>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
            attr = true;
        }
        k_tc_red<false, 16><<<grid, THREADS, smem, s>>>(ma, mb, p);
    }
    return true;
}

}  // namespace betty
