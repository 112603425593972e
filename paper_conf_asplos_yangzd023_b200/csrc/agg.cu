#include <cstdio>
#include <cmath>
#include <cstdlib>
// agg.cu -- a3/a5: GraphSAGE aggregation forward and backward (HBM-bound
// CSR segment reductions), Table 1, Eq. 1 PAPER.md:269.
//
// Forward kernels write the A operand of the following dense GEMM directly
// (fusing the concat and the bias "ones" column):
//   mean, aggregate-first:  XA[v] = [ h_v | (1/D_v) sum_{u in N(v)} h_u | 1 ]
//   mean, project-first:    S[v]  = Y[v, self] + (1/D_v) sum_u Y[u, neigh]
//                           (Y = [H|1] [W_n | W_s ; 0 | b] from the GEMM)
//   pool:                   XA[v] = [ h_v | max_u ReLU(Zp[u]) | 1 ], argmax
// Backward kernels gather through the CSC (deterministic, no float atomics).
// Feature rows are read with 128-bit vector loads; one warp owns a dst row
// and its lanes cover the row's 16-byte vectors; edge indices are loaded 32
// at a time and broadcast with shuffles, and up to 4 neighbour rows are in
// flight per lane.
#include "common.cuh"
#include "internal.h"
#include "sage.h"
#include "extract.h"

namespace betty {

template <typename T> __device__ __forceinline__ const T* row_ptr(const T* X, int64_t ld, const int32_t* xrow, int64_t r) {
    return X + (int64_t)(xrow ? xrow[r] : (int32_t)r) * ld;
}
// feature row g of a (possibly sharded) table: base[g / rps] + (g % rps) * ld, or X + g * ld
template <typename T> __device__ __forceinline__ const T* feat_row(const T* X, int64_t ld, const FeatShards& sh,
                                                                   int32_t g) {
    if (sh.R == 0) return X + (int64_t)g * ld;
    const int s = (int)((int64_t)g / sh.rps);
    return (const T*)sh.base[s] + ((int64_t)g - (int64_t)s * sh.rps) * ld;
}

// ------------------------------------------------ mean, aggregate-first fwd
// LPR lanes own one dst row (RPW = 32/LPR rows per warp); lane `sub` covers
// 16-byte vector `sub` (+ LPR, ...) of the feature row.  All neighbour vectors
// of a batch of up to EB edges are issued at once as cp.async copies into the
// warp's shared-memory slice (no registers held while in flight, one memory
// round trip per row instead of one per 4 edges) and summed from shared memory
// after cp.async.wait_group; each lane reads back only what it copied itself.
// Feature rows are fetched with an L2 evict_last policy and XA is written with
// streaming stores, so the output stream does not evict the rows that one
// micro-batch re-reads.  The neighbour X-row of edge e is emap ? emap[erow[e]]
// : erow[e] (layer 0 passes the edge -> global-id array written by the
// extraction); the self row of dst v is srow ? srow[v] : v.  With an order
// table (extract.h) the rows are visited micro-batch by micro-batch, and the
// grid is exactly the resident CTAs so all warps sweep the order together.
constexpr int AGG_EB = 12;       // edges per cp.async batch (layer-0 fanout 10 fits one batch)
__device__ __forceinline__ uint64_t l2_evict_last_policy() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ void cp_async16(void* sdst, const void* gsrc, uint64_t pol, int hint) {
    if (hint == 3)          // L1-allocating: rows re-read by the same SM hit L1
        asm volatile("cp.async.ca.shared.global [%0], [%1], 16;"
                     ::"r"((uint32_t)__cvta_generic_to_shared(sdst)), "l"(gsrc) : "memory");
    else if (hint)
        asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2;"
                     ::"r"((uint32_t)__cvta_generic_to_shared(sdst)), "l"(gsrc), "l"(pol) : "memory");
    else
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;"
                     ::"r"((uint32_t)__cvta_generic_to_shared(sdst)), "l"(gsrc) : "memory");
}
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init1(uint64_t* b) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_expect(uint64_t* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait_parity(uint64_t* b, uint32_t ph) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                     : "=r"(ok) : "r"(smem_u32(b)), "r"(ph) : "memory");
}
// one whole feature row global -> shared through the bulk-copy (TMA) engine, completion on `bar`
__device__ __forceinline__ void bulk_row(void* sdst, const void* gsrc, uint32_t bytes, uint64_t* bar, uint64_t pol) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
                 ::"r"(smem_u32(sdst)), "l"(gsrc), "r"(bytes), "r"(smem_u32(bar)), "l"(pol) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() {
    asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 0;" ::: "memory");
}
template <typename T> __device__ __forceinline__ void st_cs4(T* p, const float* v);
template <> __device__ __forceinline__ void st_cs4<float>(float* p, const float* v) {
    __stcs((float4*)p, make_float4(v[0], v[1], v[2], v[3]));
}
template <typename Tout, int VW> __device__ __forceinline__ void st_vec_cs(Tout* p, const float* v) {
    if constexpr (sizeof(Tout) == 2) {
        uint32_t w[VW / 2];
#pragma unroll
        for (int i = 0; i < VW / 2; ++i) {
            __nv_bfloat162 h = __floats2bfloat162_rn(v[2 * i], v[2 * i + 1]);
            w[i] = *(uint32_t*)&h;
        }
        if constexpr (VW == 8) __stcs((uint4*)p, make_uint4(w[0], w[1], w[2], w[3]));
        else __stcs((uint2*)p, make_uint2(w[0], w[1]));
    } else {
#pragma unroll
        for (int i = 0; i < VW; i += 4) __stcs((float4*)(p + i), make_float4(v[i], v[i + 1], v[i + 2], v[i + 3]));
    }
}

template <typename Tin, typename Tout, int LPR>
__global__ void __launch_bounds__(256) k_agg_mean_xa(const Tin* __restrict__ X, int64_t ldx,
                                                     const int32_t* __restrict__ srow,
                                                     const int32_t* __restrict__ erow,
                                                     const int32_t* __restrict__ emap,
                                                     const int64_t* __restrict__ indptr, const int64_t* cnt,
                                                     const int64_t* __restrict__ otab, int Fi, int Fp,
                                                     Tout* __restrict__ XA, int64_t ldxa, int hint, int vlo, int vhi,
                                                     unsigned* ctr, int sum, const __grid_constant__ FeatShards sh) {
    using VI = Vec<Tin>;
    constexpr int VW = VI::N;
    constexpr int RPW = 32 / LPR;
    static_assert(AGG_EB <= LPR || LPR == 8, "edge batch indices come from one lane each");
    constexpr int EB = AGG_EB < LPR ? AGG_EB : LPR;
    constexpr int SLOTS = EB + 1;                    // EB neighbour rows + the self row
    constexpr int CROWS = 8 * RPW;                   // rows a CTA claims per iteration
    extern __shared__ uint4 agg_sbuf[];              // [warps][RPW][SLOTS][LPR]
    __shared__ int64_t s_vs[ORDER_SMEM + 1], s_rs[ORDER_SMEM];
    __shared__ int64_t s_cta[3];
    __shared__ uint64_t s_bar[8][RPW];               // per row group: bulk-copy completion
    const int64_t nd = cnt[0];
    const int nseg = order_load(otab, s_vs, s_rs);
    const int NV = (Fi + VW - 1) / VW;
    const int lane = lane_id(), sub = lane % LPR, grp = lane / LPR;
    const int wib = threadIdx.x >> 5;
    const unsigned gmask = LPR == 32 ? 0xffffffffu : (((1u << LPR) - 1u) << (grp * LPR));
    uint4* wb = agg_sbuf + ((int64_t)wib * RPW + grp) * SLOTS * LPR;
    const uint64_t pol = l2_evict_last_policy();
    const int use_hint = hint == 3 ? 3 : (hint != 0 ? 1 : 0);
    int seg = 0;
    // Row meta (real row, edge range, first EB edge ids, self row) of the next iteration is
    // loaded while the current gather is in flight.
    // Row meta (row id, edge range, first EB edge ids, self row) of the next iteration is
    // loaded while the current rows' gathers are in flight.
    struct Meta { int64_t v, b, e; int32_t my, sr; };
    auto meta = [&](int64_t v0, Meta& m) {
        const int64_t vv = v0 + grp;
        m.v = vv; m.b = 0; m.e = 0; m.my = 0; m.sr = 0;
        if (vv < nd) {
            m.v = order_map(vv, nseg, s_vs, s_rs, seg);
            m.b = __ldcs(indptr + m.v);
            m.e = __ldcs(indptr + m.v + 1);
            m.sr = srow ? __ldcs(srow + m.v) : (int32_t)m.v;
            if (sub < m.e - m.b && sub < EB) { m.my = __ldcs(erow + m.b + sub); if (emap) m.my = emap[m.my]; }
        }
    };
    // Dynamic schedule: the CTA claims CROWS consecutive (virtual) rows per iteration, two
    // iterations ahead (the atomic's latency is off the critical path).  The rows in flight
    // chip-wide stay a narrow window of the micro-batch-major order, so the source rows one
    // micro-batch shares are re-read from L2; statically strided warps drift apart instead.
    // whole-row bulk copies (TMA engine): one instruction per neighbour row instead of one
    // 16-byte cp.async per lane; only when one pass covers the whole row
    const bool bulk = vlo == 0 && vhi == NV && hint < 2;     // hint 2: per-lane cp.async instead
    const uint32_t row_bytes = (uint32_t)NV * 16u;
    uint64_t* bar = &s_bar[wib][grp];
    uint32_t bph = 0;
    if (sub == 0) mbar_init1(bar);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    unsigned pend = 0;
    if (threadIdx.x == 0) {
        s_cta[0] = (int64_t)atomicAdd(ctr, 1u) * CROWS;
        s_cta[1] = (int64_t)atomicAdd(ctr, 1u) * CROWS;
        pend = atomicAdd(ctr, 1u);
    }
    __syncthreads();
    int64_t base = s_cta[0];
    Meta cur;
    meta(base + wib * RPW, cur);
    for (int it = 0; base < nd; ++it) {
        const int64_t v0 = base + wib * RPW;
        const bool rowok = v0 + grp < nd;
        const int vi = vlo + sub;
        const bool act = rowok && vi < vhi;
        const int n = (int)(cur.e - cur.b);
        const bool fast = vhi - vlo <= LPR && n <= EB;
        if (fast && bulk) {      // neighbours + self: one bulk row copy per lane, completion on the group's barrier
            if (rowok) {
                if (sub == 0) mbar_expect(bar, (uint32_t)(n + 1) * row_bytes);
                __syncwarp(gmask);
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                if (sub < n) bulk_row(wb + sub * LPR, feat_row(X, ldx, sh, cur.my), row_bytes, bar, pol);
                if (sub == 0) bulk_row(wb + EB * LPR, feat_row(X, ldx, sh, cur.sr), row_bytes, bar, pol);
            }
        } else if (fast) {      // the whole row (neighbours + self) in one batch of async copies
            for (int t = 0; t < n; ++t) {
                const int32_t u = __shfl_sync(gmask, cur.my, t, LPR);
                if (act) cp_async16(wb + t * LPR + sub, feat_row(X, ldx, sh, u) + vi * VW, pol, use_hint);
            }
            if (act) cp_async16(wb + EB * LPR + sub, feat_row(X, ldx, sh, cur.sr) + vi * VW, pol, use_hint);
            asm volatile("cp.async.commit_group;" ::: "memory");
        }
        if (threadIdx.x == 0) {
            s_cta[(it + 2) % 3] = (int64_t)pend * CROWS;
            pend = atomicAdd(ctr, 1u);
        }
        __syncthreads();
        const int64_t nbase = s_cta[(it + 1) % 3];
        Meta nxt;
        meta(nbase + wib * RPW, nxt);       // next rows' meta overlaps the gather
        Tout* out = XA + cur.v * ldxa;
        const float inv = n > 0 ? (sum ? 1.0f : 1.0f / (float)n) : 0.0f;     // sum aggregator: no 1/D
        if (fast) {
            if (bulk) {
                if (rowok) { mbar_wait_parity(bar, bph); bph ^= 1u; }
            } else {
                asm volatile("cp.async.wait_group 0;" ::: "memory");
            }
            if (act) {
                float acc[VW];
#pragma unroll
                for (int t = 0; t < VW; ++t) acc[t] = 0.f;
                for (int t = 0; t < n; ++t) VI::add_raw(acc, *(const typename VI::Raw*)(wb + t * LPR + sub));
                float so[VW], ao[VW];
                const typename VI::Raw sraw = *(const typename VI::Raw*)(wb + EB * LPR + sub);
#pragma unroll
                for (int t = 0; t < VW; ++t) so[t] = 0.f;
                VI::add_raw(so, sraw);
#pragma unroll
                for (int t = 0; t < VW; ++t) {
                    const bool in = vi * VW + t < Fi;
                    so[t] = in ? so[t] : 0.f;
                    ao[t] = in ? acc[t] * inv : 0.f;
                }
                if constexpr (sizeof(Tin) == sizeof(Tout)) {
                    st_vec_cs<Tout, VW>(out + vi * VW, so);
                    st_vec_cs<Tout, VW>(out + Fp + vi * VW, ao);
                } else {
#pragma unroll
                    for (int t = 0; t < VW; ++t) {
                        const int col = vi * VW + t;
                        if (col < Fi) { st_act(out + col, so[t]); st_act(out + Fp + col, ao[t]); }
                    }
                }
            }
            __syncwarp(gmask);
        } else {
            // general path: rows longer than a batch or wider than the lane group
            for (int vb = vlo; vb < vhi; vb += LPR) {
                const int vj = vb + sub;
                const bool actj = rowok && vj < vhi;
                float accj[VW];
#pragma unroll
                for (int t = 0; t < VW; ++t) accj[t] = 0.f;
                for (int64_t e0 = cur.b; e0 < cur.e; e0 += EB) {
                    const int nb = (int)mn64(EB, cur.e - e0);
                    int32_t mj = 0;
                    if (sub < nb) { mj = erow[e0 + sub]; if (emap) mj = emap[mj]; }
                    for (int t = 0; t < nb; ++t) {
                        const int32_t u = __shfl_sync(gmask, mj, t, LPR);
                        if (actj) cp_async16(wb + t * LPR + sub, feat_row(X, ldx, sh, u) + vj * VW, pol, use_hint);
                    }
                    cp_async_wait_all();
                    if (actj)
                        for (int t = 0; t < nb; ++t) VI::add_raw(accj, *(const typename VI::Raw*)(wb + t * LPR + sub));
                    __syncwarp(gmask);
                }
                if (actj) {
                    VI self;
                    self.load(feat_row(X, ldx, sh, cur.sr) + vj * VW);
#pragma unroll
                    for (int t = 0; t < VW; ++t) {
                        const int col = vj * VW + t;
                        if (col < Fi) { st_act(out + col, self.v[t]); st_act(out + Fp + col, accj[t] * inv); }
                    }
                }
            }
        }
        if (rowok && vhi == NV) {
            // (last column pass) pad columns of both halves, the ones column (bias), trailing pad
            for (int col = NV * VW + sub; col < Fp; col += LPR) { st_act(out + col, 0.f); st_act(out + Fp + col, 0.f); }
            for (int col = 2 * Fp + sub; col < ldxa; col += LPR) st_act(out + col, col == 2 * Fp ? 1.f : 0.f);
        }
        cur = nxt;
        base = nbase;
    }
}

// ------------------------------------------------ pool, vectorised (one warp per row, float4 column groups)
// Same semantics as k_agg_pool / k_route_pool (reading #14: max of ReLU(Zp) over the row, empty
// row -> 0, ties -> first in row order; the gradient goes to that argmax), but every lane owns
// T 4-column groups and a batch of 4 edges' rows is in flight at once.
template <typename Tin, typename Tout, int T, bool POS8>
__global__ void __launch_bounds__(256) k_agg_pool_v(const Tin* __restrict__ X, int64_t ldx,
                                                    const int32_t* __restrict__ xrow, const float* __restrict__ Zp,
                                                    int64_t ldz, const int64_t* __restrict__ indptr,
                                                    const int32_t* __restrict__ idx, const int64_t* cnt, int Fi, int Fp,
                                                    Tout* __restrict__ XA, int64_t ldxa, void* __restrict__ argv,
                                                    int64_t ldarg) {
    const int64_t nd = cnt[0];
    const int lane = lane_id();
    const int NG = (Fi + 3) / 4;
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t v = gw; v < nd; v += nw) {
        const int64_t b = indptr[v], e = indptr[v + 1];
        float best[T][4];
        int32_t am[T][4];
#pragma unroll
        for (int t = 0; t < T; ++t)
#pragma unroll
            for (int q = 0; q < 4; ++q) { best[t][q] = 0.f; am[t][q] = -1; }
        for (int64_t e0 = b; e0 < e; e0 += 32) {
            const int n = (int)mn64(32, e - e0);
            const int32_t my = lane < n ? idx[e0 + lane] : 0;
            for (int j0 = 0; j0 < n; j0 += 4) {
                int32_t u[4];
                float4 z[4][T];
#pragma unroll
                for (int k = 0; k < 4; ++k) u[k] = __shfl_sync(0xffffffffu, my, (j0 + k) & 31);
#pragma unroll
                for (int k = 0; k < 4; ++k)
#pragma unroll
                    for (int t = 0; t < T; ++t) {
                        const int g = lane + 32 * t;
                        z[k][t] = (j0 + k < n && g < NG) ? __ldg((const float4*)(Zp + (int64_t)u[k] * ldz) + g)
                                                         : make_float4(0.f, 0.f, 0.f, 0.f);
                    }
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    if (j0 + k >= n) break;
                    const int32_t who = POS8 ? (int32_t)(e0 - b) + j0 + k : u[k];   // position in the row / id
#pragma unroll
                    for (int t = 0; t < T; ++t) {
                        const float zz[4] = {fmaxf(z[k][t].x, 0.f), fmaxf(z[k][t].y, 0.f), fmaxf(z[k][t].z, 0.f),
                                             fmaxf(z[k][t].w, 0.f)};
#pragma unroll
                        for (int q = 0; q < 4; ++q)
                            if (am[t][q] < 0 || zz[q] > best[t][q]) { best[t][q] = zz[q]; am[t][q] = who; }
                    }
                }
            }
        }
        const Tin* xv = row_ptr(X, ldx, xrow, v);
        Tout* o = XA + v * ldxa;
#pragma unroll
        for (int t = 0; t < T; ++t) {
            const int g = lane + 32 * t;
            if (g >= NG) continue;
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const int col = 4 * g + q;
                if (col < Fi) {
                    st_act(o + col, ld_act(xv + col));
                    st_act(o + Fp + col, best[t][q]);
                    if (!POS8) ((int32_t*)argv)[v * ldarg + col] = am[t][q];
                }
            }
            if (POS8) {               // 4 byte positions per group (255: empty row)
                uint32_t w = 0;
#pragma unroll
                for (int q = 0; q < 4; ++q) w |= (uint32_t)(am[t][q] < 0 ? 255 : am[t][q]) << (8 * q);
                *(uint32_t*)((uint8_t*)argv + v * ldarg + 4 * g) = w;
            }
        }
        for (int col = Fi + lane; col < Fp; col += 32) { st_act(o + col, 0.f); st_act(o + Fp + col, 0.f); }
        for (int col = 2 * Fp + lane; col < ldxa; col += 32) st_act(o + col, col == 2 * Fp ? 1.f : 0.f);
    }
}
template <typename Tout, int T, bool POS8>
__global__ void __launch_bounds__(256) k_route_pool_v(const float* __restrict__ dXA, int64_t ldd,
                                                      const void* __restrict__ argv, int64_t ldarg,
                                                      const int64_t* __restrict__ indptr,
                                                      const int32_t* __restrict__ idx,
                                                      const int64_t* __restrict__ t_indptr,
                                                      const int32_t* __restrict__ t_idx, const int64_t* cnt, int Fi,
                                                      int Fp, const float* __restrict__ Zp, int64_t ldz,
                                                      Tout* __restrict__ out, int64_t ldo) {
    const int64_t ns = cnt[1];
    const int lane = lane_id();
    const int NG = (Fi + 3) / 4;
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t u = gw; u < ns; u += nw) {
        const int64_t b = t_indptr[u], e = t_indptr[u + 1];
        float acc[T][4];
#pragma unroll
        for (int t = 0; t < T; ++t)
#pragma unroll
            for (int q = 0; q < 4; ++q) acc[t][q] = 0.f;
        for (int64_t e0 = b; e0 < e; e0 += 32) {
            const int n = (int)mn64(32, e - e0);
            const int32_t my = lane < n ? t_idx[e0 + lane] : 0;
            // POS8: u's position in each edge's row v, one lane per edge for the whole 32-edge chunk:
            // the row's entries are loaded 8 at a time (independent loads) and compared, so the
            // search costs ~1 round trip per chunk instead of a dependent chain per 4 edges
            int32_t mykey = (int32_t)u;
            if (POS8) {
                mykey = -2;
                if (lane < n) {
                    const int64_t rb = __ldg(indptr + my), re = __ldg(indptr + my + 1);
                    for (int64_t base = rb; base < re && mykey < 0; base += 8) {
                        int32_t w[8];
#pragma unroll
                        for (int i = 0; i < 8; ++i) w[i] = base + i < re ? __ldg(idx + base + i) : -1;
#pragma unroll
                        for (int i = 0; i < 8; ++i)
                            if (mykey < 0 && w[i] == (int32_t)u) mykey = (int32_t)(base + i - rb);
                    }
                }
            }
            for (int j0 = 0; j0 < n; j0 += 4) {
                int32_t v[4];
                int4 a[4][T];
                int32_t key[4];                 // what an argmax entry must equal: u, or u's position in v's row
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    v[k] = __shfl_sync(0xffffffffu, my, (j0 + k) & 31);
                    key[k] = __shfl_sync(0xffffffffu, mykey, (j0 + k) & 31);
                }
#pragma unroll
                for (int k = 0; k < 4; ++k)
#pragma unroll
                    for (int t = 0; t < T; ++t) {
                        const int g = lane + 32 * t;
                        if (j0 + k < n && g < NG) {
                            if (POS8) {
                                const uint32_t w = __ldg((const uint32_t*)((const uint8_t*)argv + (int64_t)v[k] * ldarg) + g);
                                a[k][t] = make_int4((int)(w & 255u), (int)(w >> 8 & 255u), (int)(w >> 16 & 255u),
                                                    (int)(w >> 24));
                            } else {
                                a[k][t] = __ldg((const int4*)((const int32_t*)argv + (int64_t)v[k] * ldarg) + g);
                            }
                        } else {
                            a[k][t] = make_int4(-1, -1, -1, -1);
                        }
                    }
                float4 d[4][T];
#pragma unroll
                for (int k = 0; k < 4; ++k)
#pragma unroll
                    for (int t = 0; t < T; ++t) {
                        const int g = lane + 32 * t;
                        const bool hit = a[k][t].x == key[k] || a[k][t].y == key[k] || a[k][t].z == key[k] ||
                                         a[k][t].w == key[k];
                        d[k][t] = hit ? __ldg((const float4*)(dXA + (int64_t)v[k] * ldd + Fp) + g)
                                      : make_float4(0.f, 0.f, 0.f, 0.f);
                    }
#pragma unroll
                for (int k = 0; k < 4; ++k)
#pragma unroll
                    for (int t = 0; t < T; ++t) {
                        if (a[k][t].x == key[k]) acc[t][0] += d[k][t].x;
                        if (a[k][t].y == key[k]) acc[t][1] += d[k][t].y;
                        if (a[k][t].z == key[k]) acc[t][2] += d[k][t].z;
                        if (a[k][t].w == key[k]) acc[t][3] += d[k][t].w;
                    }
            }
        }
        const float* zu = Zp + u * ldz;
#pragma unroll
        for (int t = 0; t < T; ++t) {
            const int g = lane + 32 * t;
            if (g >= NG) continue;
            const float4 z = __ldg((const float4*)zu + g);
            const float r[4] = {z.x > 0.f ? acc[t][0] : 0.f, z.y > 0.f ? acc[t][1] : 0.f, z.z > 0.f ? acc[t][2] : 0.f,
                                z.w > 0.f ? acc[t][3] : 0.f};
#pragma unroll
            for (int q = 0; q < 4; ++q) if (4 * g + q < Fi) st_act(out + u * ldo + 4 * g + q, r[q]);
        }
        for (int col = Fi + lane; col < ldo; col += 32) st_act(out + u * ldo + col, 0.f);
    }
}

// ------------------------------------------------ mean, aggregate-first fwd: TMA gather4 pipeline
// Warp-specialised persistent kernel, one CTA per SM: G4_PROD producer warps, each owning every
// G4_PROD-th stage of a G4_STAGES ring, and G4_CONS consumer warps.
//  * A producer claims G4_CLAIM virtual rows at a time (dynamic, micro-batch-major order) ONE
//    CLAIM AHEAD: the claim's real row ids, indptr pairs and self-row ids are copied into a
//    per-warp shared buffer with cp.async while the previous claim is being issued, so no
//    global latency sits between a stage's rows and its gathers except the edge ids.
//  * A stage is a run of <= G4_MAXR consecutive real rows (one order segment, so their edges are
//    one contiguous CSR range) whose neighbour rows fit the stage's slots.  Slot s holds the
//    source row of edge E0a + s (E0a = first edge rounded down to 4): every row's neighbours are
//    consecutive slots, and 4 consecutive edges are one tile::gather4 TMA copy (four arbitrary
//    rows per instruction, completion on the stage's mbarrier; row -1 reads as zeros).  Self
//    rows are gathered the same way.
//  * Consumers map (row, 16-byte vector) pairs onto threads, sum the row's slots from shared
//    memory and stream XA out.  A row whose neighbours exceed the slots ("long" row, e.g.
//    full-neighbourhood layers) is a stage of its own that the consumers reduce straight from
//    global memory.
#ifndef BETTY_G4_STAGES          // (overridable at build time for tuning sweeps: tools/sweep_g4.sh)
#define BETTY_G4_STAGES 8
#endif
#ifndef BETTY_G4_PROD
#define BETTY_G4_PROD 4
#endif
#ifndef BETTY_G4_CPP
#define BETTY_G4_CPP 4
#endif
#ifndef BETTY_G4_MAXR
#define BETTY_G4_MAXR 16
#endif
#ifndef BETTY_G4_CLAIM
#define BETTY_G4_CLAIM 64
#endif
constexpr int G4_STAGES = BETTY_G4_STAGES, G4_PROD = BETTY_G4_PROD, G4_CPP = BETTY_G4_CPP, G4_MAXR = BETTY_G4_MAXR,
              G4_CLAIM = BETTY_G4_CLAIM;
constexpr int G4_CONS = G4_PROD * G4_CPP;             // consumer warps: G4_CPP per producer
constexpr int G4_THREADS = 32 * (G4_PROD + G4_CONS);
static_assert(G4_STAGES % G4_PROD == 0, "stages are dealt round-robin to the producers");
struct G4Hdr {
    int64_t r0;                  // first real row
    int64_t hb, he;              // long row: its edge range
    int32_t n;                   // rows (-1: end of work)
    int32_t lng;                 // 1: long row
    int32_t off[G4_MAXR + 1];    // slot offset of each row's first edge (relative to E0a)
};
struct G4Claim {                 // one claim's rows (virtual offset j)
    int64_t r[G4_CLAIM];         // real row
    int64_t lo[G4_CLAIM], hi[G4_CLAIM];   // indptr[r], indptr[r + 1]
    int32_t sid[G4_CLAIM];       // self row (srow[r] or r)
};
struct G4Args {
    const int32_t* srow; const int32_t* erow; const int32_t* emap;
    const int64_t* indptr; const int64_t* cnt; const int64_t* otab;
    void* XA; int64_t ldxa; const void* X; int64_t ldx;
    unsigned* ctr;
    int Fi, Fp, NV;
    uint32_t row_bytes, grp_bytes, slot_groups, stage_bytes;
    int hint;
    int sum;                       // sum aggregator (Table 1 "Sum"): no 1/D
};
__device__ __forceinline__ void gather4(uint32_t sdst, const CUtensorMap* tm, int32_t r0, int32_t r1, int32_t r2,
                                        int32_t r3, uint64_t* bar, uint64_t pol) {
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes.L2::cache_hint"
                 " [%0], [%1, {%2, %3, %4, %5, %6}], [%7], %8;"
                 ::"r"(sdst), "l"((uint64_t)tm), "r"(0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(smem_u32(bar)),
                   "l"(pol) : "memory");
}
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void cp_async8(void* sdst, const void* gsrc) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(sdst)), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async4(void* sdst, const void* gsrc) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(sdst)), "l"(gsrc) : "memory");
}
// the row tail of XA: pad columns of both halves and [1, 0, ...] from column 2 Fp
template <typename Tout> __device__ __forceinline__ void xa_tail(Tout* out, int c0, int Fp, int64_t ldxa) {
    for (int col = c0; col < Fp; ++col) { st_act(out + col, 0.f); st_act(out + Fp + col, 0.f); }
    Tout* t = out + 2 * Fp;
    const int w = (int)(ldxa - 2 * Fp);
    if (w * (int)sizeof(Tout) == 16 && ((uintptr_t)t & 15) == 0) {
        const uint32_t one = sizeof(Tout) == 2 ? 0x3F80u : 0x3F800000u;
        __stcs((uint4*)t, make_uint4(one, 0u, 0u, 0u));
    } else {
        for (int col = 0; col < w; ++col) st_act(t + col, col == 0 ? 1.f : 0.f);
    }
}

template <typename Tin, typename Tout>
__global__ void __launch_bounds__(G4_THREADS, 1) k_agg_mean_g4(const __grid_constant__ CUtensorMap tmX, G4Args a) {
    using VI = Vec<Tin>;
    constexpr int VW = VI::N;
    extern __shared__ __align__(128) uint8_t g4_smem[];
    __shared__ G4Hdr hdr[G4_STAGES];
    __shared__ G4Claim clm[G4_PROD][2];
    __shared__ uint64_t full[G4_STAGES], empty[G4_STAGES];
    __shared__ int64_t s_vs[ORDER_SMEM + 1], s_rs[ORDER_SMEM];
    const int64_t nd = a.cnt[0];
    const int nseg = order_load(a.otab, s_vs, s_rs);
    const int warp = threadIdx.x >> 5, lane = lane_id();
    if (threadIdx.x == 0) {
        for (int s = 0; s < G4_STAGES; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], G4_CPP); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const uint32_t sbase = smem_u32(g4_smem);
    const uint32_t self_off = a.slot_groups * a.grp_bytes;          // self rows after the edge slots
    if (warp < G4_PROD) {
        // ---------------------------------------------------------------- producer
        uint64_t pol;
        if (a.hint) pol = l2_evict_last_policy();
        else asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(pol));
        int seg = 0;
        // claim G4_CLAIM virtual rows into buffer C (async); returns the claim's first virtual row
        auto claim = [&](G4Claim& C, int64_t& vend) -> int64_t {
            int64_t v = 0;
            if (lane == 0) v = (int64_t)atomicAdd(a.ctr, 1u) * G4_CLAIM;
            v = __shfl_sync(0xffffffffu, v, 0);
            vend = v < nd ? mn64(v + G4_CLAIM, nd) : v;
            for (int j = lane; j < G4_CLAIM; j += 32) {
                if (v + j >= vend) break;
                const int64_t r = nseg > 0 ? order_map(v + j, nseg, s_vs, s_rs, seg) : v + j;
                C.r[j] = r;
                cp_async8(&C.lo[j], a.indptr + r);
                cp_async8(&C.hi[j], a.indptr + r + 1);
                if (a.srow) cp_async4(&C.sid[j], a.srow + r); else C.sid[j] = (int32_t)r;
            }
            asm volatile("cp.async.commit_group;" ::: "memory");
            return v;
        };
        int cb = 0;                                     // buffer of the current claim
        int64_t ce, ne;
        int64_t cv = claim(clm[warp][0], ce);
        int64_t nv = claim(clm[warp][1], ne);
        asm volatile("cp.async.wait_group 1;" ::: "memory");
        __syncwarp();
        int j0 = 0;                                     // next virtual row of the current claim
        const int64_t cap = (int64_t)a.slot_groups * 4;
        for (uint32_t i = 0;; ++i) {
            const int s = (warp + G4_PROD * i) % G4_STAGES;
            const uint32_t visit = i / (G4_STAGES / G4_PROD);
            G4Hdr& H = hdr[s];
            uint64_t* fb = &full[s];
            if (cv + j0 >= ce) {                        // current claim used up: rotate
                cv = nv; ce = ne; cb ^= 1; j0 = 0;
                if (cv < nd) nv = claim(clm[warp][cb ^ 1], ne);
                else asm volatile("cp.async.commit_group;" ::: "memory");
                asm volatile("cp.async.wait_group 1;" ::: "memory");
                __syncwarp();
            }
            mbar_wait_parity(&empty[s], (visit & 1u) ^ 1u);
            if (cv >= nd) {                            // no more work: tell the consumers
                if (lane == 0) { H.n = -1; mbar_arrive(fb); }
                break;
            }
            const G4Claim& C = clm[warp][cb];
            const int rem = (int)mn64(G4_MAXR, ce - cv - j0);
            const int jj = j0 + lane;
            const bool valid = lane < rem;
            const int64_t r = valid ? C.r[jj] : 0, lo = valid ? C.lo[jj] : 0, hi = valid ? C.hi[jj] : 0;
            const int32_t sidv = valid ? C.sid[jj] : -1;
            const int64_t r0 = __shfl_sync(0xffffffffu, r, 0);
            const int64_t E0 = __shfl_sync(0xffffffffu, lo, 0);
            const int64_t E0a = E0 & ~(int64_t)3;
            const bool fits = valid && r == r0 + lane && hi - E0a <= cap;
            int n = __ffs(~__ballot_sync(0xffffffffu, fits)) - 1;
            const int lng = n == 0;
            if (lng) n = 1;
            const int64_t Eend = __shfl_sync(0xffffffffu, hi, n - 1);
            if (lane == 0) { H.r0 = r0; H.n = n; H.lng = lng; H.hb = E0; H.he = Eend; }
            if (lane < n) H.off[lane] = (int32_t)(lo - E0a);
            if (lane == n - 1) H.off[n] = (int32_t)(hi - E0a);
            const int groups = lng ? 0 : (int)((Eend - E0a + 3) >> 2);
            const int sgroups = (n + 3) >> 2;
            // edge ids of this lane's groups (independent loads, all in flight together)
            int32_t id[2][4];
#pragma unroll
            for (int gg = 0; gg < 2; ++gg)
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int64_t e = E0a + 4 * (lane + 32 * gg) + q;
                    id[gg][q] = (lane + 32 * gg < groups && e >= E0 && e < Eend) ? __ldg(a.erow + e) : -1;
                }
            if (a.emap) {
#pragma unroll
                for (int gg = 0; gg < 2; ++gg)
#pragma unroll
                    for (int q = 0; q < 4; ++q) if (id[gg][q] >= 0) id[gg][q] = __ldg(a.emap + id[gg][q]);
            }
            __syncwarp();
            if (lane == 0) mbar_expect(fb, (uint32_t)(groups + sgroups) * 4u * a.row_bytes);
            const uint32_t sdat = sbase + (uint32_t)s * a.stage_bytes;
#pragma unroll
            for (int gg = 0; gg < 2; ++gg) {
                const int g = lane + 32 * gg;
                if (g < groups)
                    gather4(sdat + (uint32_t)g * a.grp_bytes, &tmX, id[gg][0], id[gg][1], id[gg][2], id[gg][3], fb, pol);
            }
            int32_t sv[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) sv[q] = __shfl_sync(0xffffffffu, sidv, (4 * lane + q) & 31);
#pragma unroll
            for (int q = 0; q < 4; ++q) if (4 * lane + q >= n) sv[q] = -1;
            if (lane < sgroups)
                gather4(sdat + self_off + (uint32_t)lane * a.grp_bytes, &tmX, sv[0], sv[1], sv[2], sv[3], fb, pol);
            j0 += n;
        }
        asm volatile("cp.async.wait_all;" ::: "memory");
    } else {
        // ---------------------------------------------------------------- consumers
        // consumer warps w*G4_CPP .. w*G4_CPP + G4_CPP-1 drain the stages of producer w
        const int w = (warp - G4_PROD) / G4_CPP, cw = (warp - G4_PROD) % G4_CPP;
        const int ct = cw * 32 + lane, NCT = G4_CPP * 32;
        const int NV = a.NV;
        for (uint32_t i = 0;; ++i) {
            const int s = (w + G4_PROD * i) % G4_STAGES;
            mbar_wait_parity(&full[s], (i / (G4_STAGES / G4_PROD)) & 1u);
            const G4Hdr& H = hdr[s];
            const int n = H.n;
            if (n < 0) break;
            const uint8_t* sdat = g4_smem + (size_t)s * a.stage_bytes;
            if (!H.lng) {
                // (row i, vector j) pairs u = ct, ct + NCT, ...: i, j advance incrementally (no division)
                int i = ct / NV, j = ct - (ct / NV) * NV;
                const int di = NCT / NV, dj = NCT - di * NV;
                for (int u = ct; u < n * NV; u += NCT, i += di, j += dj) {
                    if (j >= NV) { j -= NV; ++i; }
                    const int b = H.off[i], e = H.off[i + 1];
                    float acc[VW];
#pragma unroll
                    for (int t = 0; t < VW; ++t) acc[t] = 0.f;
                    const uint8_t* base = sdat + j * 16;
                    int sl = b;
                    for (; sl + 4 <= e; sl += 4) {          // 4 independent shared loads in flight
                        typename VI::Raw r[4];
#pragma unroll
                        for (int q = 0; q < 4; ++q)
                            r[q] = *(const typename VI::Raw*)(base + ((sl + q) >> 2) * a.grp_bytes +
                                                               ((sl + q) & 3) * a.row_bytes);
#pragma unroll
                        for (int q = 0; q < 4; ++q) VI::add_raw(acc, r[q]);
                    }
                    for (; sl < e; ++sl)
                        VI::add_raw(acc, *(const typename VI::Raw*)(base + (sl >> 2) * a.grp_bytes + (sl & 3) * a.row_bytes));
                    float so[VW];
#pragma unroll
                    for (int t = 0; t < VW; ++t) so[t] = 0.f;
                    VI::add_raw(so, *(const typename VI::Raw*)(sdat + self_off + (i >> 2) * a.grp_bytes +
                                                               (i & 3) * a.row_bytes + j * 16));
                    const float inv = e > b ? (a.sum ? 1.0f : 1.0f / (float)(e - b)) : 0.0f;
#pragma unroll
                    for (int t = 0; t < VW; ++t) {
                        const bool in = j * VW + t < a.Fi;
                        acc[t] = in ? acc[t] * inv : 0.f;
                        so[t] = in ? so[t] : 0.f;
                    }
                    Tout* out = (Tout*)a.XA + (H.r0 + i) * a.ldxa;
                    st_vec_cs<Tout, VW>(out + j * VW, so);
                    st_vec_cs<Tout, VW>(out + a.Fp + j * VW, acc);
                }
                for (int i = ct; i < n; i += NCT) xa_tail<Tout>((Tout*)a.XA + (H.r0 + i) * a.ldxa, NV * VW, a.Fp, a.ldxa);
            } else {
                // long row (first consumer warp of the pair): lanes over vectors, 4 edges in flight,
                // straight from global memory
                const int64_t hb = H.hb, he = H.he;
                for (int j = lane; cw == 0 && j < NV; j += 32) {
                    float acc[VW];
#pragma unroll
                    for (int t = 0; t < VW; ++t) acc[t] = 0.f;
                    int64_t e = hb;
                    for (; e + 4 <= he; e += 4) {
                        int32_t u[4];
                        typename VI::Raw r[4];
#pragma unroll
                        for (int q = 0; q < 4; ++q) { u[q] = __ldg(a.erow + e + q); if (a.emap) u[q] = __ldg(a.emap + u[q]); }
#pragma unroll
                        for (int q = 0; q < 4; ++q) r[q] = VI::ld_raw((const Tin*)a.X + (int64_t)u[q] * a.ldx + j * VW);
#pragma unroll
                        for (int q = 0; q < 4; ++q) VI::add_raw(acc, r[q]);
                    }
                    for (; e < he; ++e) {
                        int32_t u = __ldg(a.erow + e);
                        if (a.emap) u = __ldg(a.emap + u);
                        VI::add_raw(acc, VI::ld_raw((const Tin*)a.X + (int64_t)u * a.ldx + j * VW));
                    }
                    float so[VW];
#pragma unroll
                    for (int t = 0; t < VW; ++t) so[t] = 0.f;
                    VI::add_raw(so, *(const typename VI::Raw*)(sdat + self_off + j * 16));
                    const float inv = he > hb ? (a.sum ? 1.0f : 1.0f / (float)(he - hb)) : 0.0f;
#pragma unroll
                    for (int t = 0; t < VW; ++t) {
                        const bool in = j * VW + t < a.Fi;
                        acc[t] = in ? acc[t] * inv : 0.f;
                        so[t] = in ? so[t] : 0.f;
                    }
                    Tout* out = (Tout*)a.XA + H.r0 * a.ldxa;
                    st_vec_cs<Tout, VW>(out + j * VW, so);
                    st_vec_cs<Tout, VW>(out + a.Fp + j * VW, acc);
                }
                if (ct == 0) xa_tail<Tout>((Tout*)a.XA + H.r0 * a.ldxa, NV * VW, a.Fp, a.ldxa);
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[s]);
        }
    }
}

// ------------------------------------------------ mean, project-first fwd
// S[v,c] = Y[v, Fop + c] + (1/D_v) sum_u Y[u, c];  out = logits (fp32) or ReLU -> H (+ones col)
template <typename Tout>
__global__ void __launch_bounds__(256) k_agg_mean_pf(const float* __restrict__ Y, int64_t ldy,
                                                     const int64_t* __restrict__ indptr,
                                                     const int32_t* __restrict__ idx, const int64_t* cnt, int Fo,
                                                     int Fop, int relu, Tout* __restrict__ out, int64_t ldo, int sum) {
    const int64_t nd = cnt[0];
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t v = gw; v < nd; v += nw) {
        const int64_t b = indptr[v], e = indptr[v + 1];
        const float inv = e > b ? (sum ? 1.0f : 1.0f / (float)(e - b)) : 0.0f;
        for (int c0 = 0; c0 < Fo; c0 += 32) {
            const int c = c0 + lane;
            const bool act = c < Fo;
            float acc = 0.f;
            for (int64_t e0 = b; e0 < e; e0 += 32) {
                const int n = (int)mn64(32, e - e0);
                const int32_t my = lane < n ? idx[e0 + lane] : 0;
                for (int j = 0; j < n; ++j) {
                    const int32_t u = __shfl_sync(0xffffffffu, my, j);
                    if (act) acc += Y[(int64_t)u * ldy + c];
                }
            }
            if (act) {
                float sv = Y[v * ldy + Fop + c] + acc * inv;
                if (relu) sv = fmaxf(sv, 0.f);
                st_act(out + v * ldo + c, sv);
            }
        }
        if (relu)
            for (int col = Fo + lane; col < ldo; col += 32) st_act(out + v * ldo + col, col == Fo ? 1.f : 0.f);
    }
}

// ----------------------------------------------- A = [X[xrow] | 1 | 0] rows
template <typename Tin, typename Tout>
__global__ void k_gather_ones(const Tin* __restrict__ X, int64_t ldx, const int32_t* __restrict__ xrow,
                              const int64_t* cnt_rows, int Fi, Tout* __restrict__ out, int64_t ldo) {
    const int64_t n = cnt_rows[0];
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t r = gw; r < n; r += nw) {
        const Tin* x = row_ptr(X, ldx, xrow, r);
        for (int col = lane; col < ldo; col += 32)
            st_act(out + r * ldo + col, col < Fi ? ld_act(x + col) : (col == Fi ? 1.f : 0.f));
    }
}

// ------------------------------------ mean, aggregate-first bwd (via CSC)
// dS_prev[u,f] = ( [u < nd] dXA[u, f] + sum_{v in CSC(u)} dXA[v, Fp + f] / D_v ) * [H[u,f] > 0]
template <typename Tm, typename Tout>
__global__ void __launch_bounds__(256) k_csc_mean(const float* __restrict__ dXA, int64_t ldd,
                                                  const int64_t* __restrict__ indptr,
                                                  const int64_t* __restrict__ t_indptr,
                                                  const int32_t* __restrict__ t_idx, const int64_t* cnt, int Fi,
                                                  int Fp, const Tm* __restrict__ H, int64_t ldh,
                                                  Tout* __restrict__ out, int64_t ldo) {
    const int64_t nd = cnt[0], ns = cnt[1];
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t u = gw; u < ns; u += nw) {
        const int64_t b = t_indptr[u], e = t_indptr[u + 1];
        for (int c0 = 0; c0 < Fi; c0 += 32) {
            const int c = c0 + lane;
            const bool act = c < Fi;
            float acc = 0.f;
            for (int64_t e0 = b; e0 < e; e0 += 32) {
                const int n = (int)mn64(32, e - e0);
                int32_t my = 0;
                float myinv = 0.f;
                if (lane < n) {
                    my = t_idx[e0 + lane];
                    myinv = indptr ? 1.0f / (float)(indptr[my + 1] - indptr[my]) : 1.0f;   // null: sum
                }
                for (int j = 0; j < n; ++j) {
                    const int32_t v = __shfl_sync(0xffffffffu, my, j);
                    const float iv = __shfl_sync(0xffffffffu, myinv, j);
                    if (act) acc += dXA[(int64_t)v * ldd + Fp + c] * iv;
                }
            }
            if (act) {
                float g = acc + (u < nd ? dXA[u * ldd + c] : 0.f);
                if (!(ld_act(H + u * ldh + c) > 0.f)) g = 0.f;
                st_act(out + u * ldo + c, g);
            }
        }
        for (int col = Fi + lane; col < ldo; col += 32) st_act(out + u * ldo + col, 0.f);
    }
}

// Vectorised form of k_csc_mean for wide layers (C2 / C5 hidden layers, Fi = 256): one warp per
// source u, lane owns float4 column groups lane + 32 k (k < VPL, so a warp reads a whole 1 KB
// half-row per edge, coalesced); the CSC entries and 1/D_v of 32 edges are loaded at once and
// broadcast by shuffles, and CM_UNR edges' rows are in flight per lane before they are added.
// The additions run in CSC order per column exactly like k_csc_mean (bit-identical results).
constexpr int CM_UNR = 4;
template <typename Tm, typename Tout, int VPL>
__global__ void __launch_bounds__(256) k_csc_mean_v(const float* __restrict__ dXA, int64_t ldd,
                                                    const int64_t* __restrict__ indptr,
                                                    const int64_t* __restrict__ t_indptr,
                                                    const int32_t* __restrict__ t_idx, const int64_t* cnt, int Fi,
                                                    int Fp, const Tm* __restrict__ H, int64_t ldh,
                                                    const uint32_t* __restrict__ hbits, int64_t ldhb,
                                                    Tout* __restrict__ out, int64_t ldo) {
    const int64_t nd = cnt[0], ns = cnt[1];
    const int lane = lane_id();
    const int NG = Fi / 4;                                  // float4 groups of a row
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t u = gw; u < ns; u += nw) {
        const int64_t b = t_indptr[u], e = t_indptr[u + 1];
        float acc[VPL][4];
#pragma unroll
        for (int k = 0; k < VPL; ++k)
#pragma unroll
            for (int t = 0; t < 4; ++t) acc[k][t] = 0.f;
        for (int64_t e0 = b; e0 < e; e0 += 32) {
            const int n = (int)mn64(32, e - e0);
            int32_t my = 0;
            float myinv = 0.f;
            if (lane < n) {
                my = t_idx[e0 + lane];
                myinv = indptr ? 1.0f / (float)(indptr[my + 1] - indptr[my]) : 1.0f;       // null: sum
            }
            for (int j0 = 0; j0 < n; j0 += CM_UNR) {
                float4 x[CM_UNR][VPL];
                float iv[CM_UNR];
#pragma unroll
                for (int q = 0; q < CM_UNR; ++q) {
                    const int32_t v = __shfl_sync(0xffffffffu, my, (j0 + q) & 31);
                    iv[q] = __shfl_sync(0xffffffffu, myinv, (j0 + q) & 31);
#pragma unroll
                    for (int k = 0; k < VPL; ++k) {
                        const int g = lane + 32 * k;
                        x[q][k] = (j0 + q < n && g < NG)
                                      ? *reinterpret_cast<const float4*>(dXA + (int64_t)v * ldd + Fp + 4 * g)
                                      : make_float4(0.f, 0.f, 0.f, 0.f);
                    }
                }
#pragma unroll
                for (int q = 0; q < CM_UNR; ++q) {
                    if (j0 + q < n) {
#pragma unroll
                        for (int k = 0; k < VPL; ++k) {
                            acc[k][0] += x[q][k].x * iv[q];
                            acc[k][1] += x[q][k].y * iv[q];
                            acc[k][2] += x[q][k].z * iv[q];
                            acc[k][3] += x[q][k].w * iv[q];
                        }
                    }
                }
            }
        }
#pragma unroll
        for (int k = 0; k < VPL; ++k) {
            const int g = lane + 32 * k;
            if (g < NG) {
                const int c = 4 * g;
                float4 sf = u < nd ? *reinterpret_cast<const float4*>(dXA + u * ldd + c) : make_float4(0.f, 0.f, 0.f, 0.f);
                float gv[4] = {acc[k][0] + sf.x, acc[k][1] + sf.y, acc[k][2] + sf.z, acc[k][3] + sf.w};
                if (hbits) {            // ReLU' from the forward's bits (32 B per 256-wide row, not 512 B of H)
                    const uint32_t w = hbits[u * ldhb + (c >> 5)] >> (c & 31);
#pragma unroll
                    for (int t = 0; t < 4; ++t)
                        if (!(w >> t & 1u)) gv[t] = 0.f;
                } else {
#pragma unroll
                    for (int t = 0; t < 4; ++t)
                        if (!(ld_act(H + u * ldh + c + t) > 0.f)) gv[t] = 0.f;
                }
                st_act4(out + u * ldo + c, gv);
            }
        }
        for (int col = Fi + lane; col < ldo; col += 32) st_act(out + u * ldo + col, 0.f);
    }
}

// Lane-group form (sources of low CSC degree, e.g. C5's layer 1 with 1.2 entries per source): LPR
// lanes per source own VPL float4 groups each (LPR * VPL = Fi / 4), so a warp works on 32 / LPR
// sources at once; per source the CSC entries / 1/D_v of LPR edges are loaded together and the
// rows of two edges are in flight before they are added (same per-column CSC order: bit-identical).
template <typename Tm, typename Tout, int LPR, int VPL, int UNR>
__global__ void __launch_bounds__(256) k_csc_mean_g(const float* __restrict__ dXA, int64_t ldd,
                                                    const int64_t* __restrict__ indptr,
                                                    const int64_t* __restrict__ t_indptr,
                                                    const int32_t* __restrict__ t_idx, const int64_t* cnt, int Fi,
                                                    int Fp, const Tm* __restrict__ H, int64_t ldh,
                                                    const uint32_t* __restrict__ hbits, int64_t ldhb,
                                                    Tout* __restrict__ out, int64_t ldo) {
    constexpr int RPW = 32 / LPR;
    const int64_t nd = cnt[0], ns = cnt[1];
    const int lane = lane_id(), sub = lane % LPR, grp = lane / LPR;
    const unsigned gmask = LPR == 32 ? 0xffffffffu : (((1u << LPR) - 1u) << (grp * LPR));
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    int64_t nb = 0, ne = 0;                             // column extents one iteration ahead
    {
        const int64_t u = gw * RPW + grp;
        if (u < ns) { nb = t_indptr[u]; ne = t_indptr[u + 1]; }
    }
    for (int64_t u0 = gw * RPW; u0 < ns; u0 += nw * RPW) {
        const int64_t u = u0 + grp;
        const int64_t b = nb, e = ne;
        {
            const int64_t un = u + nw * RPW;
            nb = 0; ne = 0;
            if (un < ns) { nb = t_indptr[un]; ne = t_indptr[un + 1]; }
        }
        if (u >= ns) continue;                              // whole lane group idle
        float acc[VPL][4];
#pragma unroll
        for (int k = 0; k < VPL; ++k)
#pragma unroll
            for (int t = 0; t < 4; ++t) acc[k][t] = 0.f;
        for (int64_t e0 = b; e0 < e; e0 += LPR) {
            const int n = (int)mn64(LPR, e - e0);
            int32_t my = 0;
            float myinv = 0.f;
            if (sub < n) {
                my = t_idx[e0 + sub];
                myinv = indptr ? 1.0f / (float)(indptr[my + 1] - indptr[my]) : 1.0f;       // null: sum
            }
#pragma unroll
            for (int j0 = 0; j0 < LPR; j0 += UNR) {
                if (j0 >= n) break;
                float4 x[UNR][VPL];
                float iv[UNR];
#pragma unroll
                for (int q = 0; q < UNR; ++q) {
                    const int32_t v = __shfl_sync(gmask, my, j0 + q, LPR);
                    iv[q] = __shfl_sync(gmask, myinv, j0 + q, LPR);
#pragma unroll
                    for (int k = 0; k < VPL; ++k)
                        x[q][k] = j0 + q < n
                                      ? *reinterpret_cast<const float4*>(dXA + (int64_t)v * ldd + Fp + 4 * (sub * VPL + k))
                                      : make_float4(0.f, 0.f, 0.f, 0.f);
                }
#pragma unroll
                for (int q = 0; q < UNR; ++q) {
                    if (j0 + q < n) {
#pragma unroll
                        for (int k = 0; k < VPL; ++k) {
                            acc[k][0] += x[q][k].x * iv[q];
                            acc[k][1] += x[q][k].y * iv[q];
                            acc[k][2] += x[q][k].z * iv[q];
                            acc[k][3] += x[q][k].w * iv[q];
                        }
                    }
                }
            }
        }
#pragma unroll
        for (int k = 0; k < VPL; ++k) {
            const int c = 4 * (sub * VPL + k);
            float4 sf = u < nd ? *reinterpret_cast<const float4*>(dXA + u * ldd + c) : make_float4(0.f, 0.f, 0.f, 0.f);
            float gv[4] = {acc[k][0] + sf.x, acc[k][1] + sf.y, acc[k][2] + sf.z, acc[k][3] + sf.w};
            if (hbits) {                // ReLU' from the forward's bits
                const uint32_t w = hbits[u * ldhb + (c >> 5)] >> (c & 31);
#pragma unroll
                for (int t = 0; t < 4; ++t)
                    if (!(w >> t & 1u)) gv[t] = 0.f;
            } else {
#pragma unroll
                for (int t = 0; t < 4; ++t)
                    if (!(ld_act(H + u * ldh + c + t) > 0.f)) gv[t] = 0.f;
            }
            st_act4(out + u * ldo + c, gv);
        }
        for (int col = Fi + sub; col < ldo; col += LPR) st_act(out + u * ldo + col, 0.f);
    }
}

// --------------------------------------- mean, project-first bwd (via CSC)
// G[u] = [ sum_{v in CSC(u)} dS[v]/D_v (Fo) | 0 | [u < nd] dS[u] (Fo) | 0 ]
template <typename Tin, typename Tout>
__global__ void __launch_bounds__(256) k_csc_pf(const Tin* __restrict__ dS, int64_t ldds,
                                                const int64_t* __restrict__ indptr,
                                                const int64_t* __restrict__ t_indptr,
                                                const int32_t* __restrict__ t_idx, const int64_t* cnt, int Fo,
                                                int Fop, Tout* __restrict__ G, int64_t ldg) {
    const int64_t nd = cnt[0], ns = cnt[1];
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t u = gw; u < ns; u += nw) {
        const int64_t b = t_indptr[u], e = t_indptr[u + 1];
        for (int c0 = 0; c0 < Fop; c0 += 32) {
            const int c = c0 + lane;
            const bool act = c < Fo;
            float acc = 0.f;
            for (int64_t e0 = b; e0 < e; e0 += 32) {
                const int n = (int)mn64(32, e - e0);
                int32_t my = 0;
                float myinv = 0.f;
                if (lane < n) {
                    my = t_idx[e0 + lane];
                    myinv = indptr ? 1.0f / (float)(indptr[my + 1] - indptr[my]) : 1.0f;   // null: sum
                }
                for (int j = 0; j < n; ++j) {
                    const int32_t v = __shfl_sync(0xffffffffu, my, j);
                    const float iv = __shfl_sync(0xffffffffu, myinv, j);
                    if (act) acc += ld_act(dS + (int64_t)v * ldds + c) * iv;
                }
            }
            if (c < Fop) {
                st_act(G + u * ldg + c, act ? acc : 0.f);
                st_act(G + u * ldg + Fop + c, (act && u < nd) ? ld_act(dS + u * ldds + c) : 0.f);
            }
        }
    }
}

// ------------------------------------------------------------ pool fwd
// XA[v] = [ h_v | max_{u in N(v)} ReLU(Zp[u]) | 1 ]; arg[v,f] = first u attaining the max (-1: empty row)
template <typename Tin, typename Tout>
__global__ void __launch_bounds__(256) k_agg_pool(const Tin* __restrict__ X, int64_t ldx,
                                                  const int32_t* __restrict__ xrow, const float* __restrict__ Zp,
                                                  int64_t ldz, const int64_t* __restrict__ indptr,
                                                  const int32_t* __restrict__ idx, const int64_t* cnt, int Fi, int Fp,
                                                  Tout* __restrict__ XA, int64_t ldxa, int32_t* __restrict__ arg,
                                                  int64_t ldarg) {
    const int64_t nd = cnt[0];
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t v = gw; v < nd; v += nw) {
        const int64_t b = indptr[v], e = indptr[v + 1];
        const Tin* xv = row_ptr(X, ldx, xrow, v);
        for (int c0 = 0; c0 < Fi; c0 += 32) {
            const int c = c0 + lane;
            const bool act = c < Fi;
            float best = 0.f;
            int32_t a = -1;
            for (int64_t e0 = b; e0 < e; e0 += 32) {
                const int n = (int)mn64(32, e - e0);
                const int32_t my = lane < n ? idx[e0 + lane] : 0;
                for (int j = 0; j < n; ++j) {
                    const int32_t u = __shfl_sync(0xffffffffu, my, j);
                    if (act) {
                        const float z = fmaxf(Zp[(int64_t)u * ldz + c], 0.f);
                        if (a < 0 || z > best) { best = z; a = u; }
                    }
                }
            }
            if (act) {
                st_act(XA + v * ldxa + c, ld_act(xv + c));
                st_act(XA + v * ldxa + Fp + c, best);
                arg[v * ldarg + c] = a;
            }
        }
        for (int col = Fi + lane; col < Fp; col += 32) { st_act(XA + v * ldxa + col, 0.f); st_act(XA + v * ldxa + Fp + col, 0.f); }
        for (int col = 2 * Fp + lane; col < ldxa; col += 32) st_act(XA + v * ldxa + col, col == 2 * Fp ? 1.f : 0.f);
    }
}

// ------------------------------------------------------------ pool bwd
// dZp[u,f] = ( sum_{v in CSC(u), arg[v,f] == u} dXA[v, Fp + f] ) * [Zp[u,f] > 0]
template <typename Tout>
__global__ void __launch_bounds__(256) k_route_pool(const float* __restrict__ dXA, int64_t ldd,
                                                    const int32_t* __restrict__ arg, int64_t ldarg,
                                                    const int64_t* __restrict__ t_indptr,
                                                    const int32_t* __restrict__ t_idx, const int64_t* cnt, int Fi,
                                                    int Fp, const float* __restrict__ Zp, int64_t ldz,
                                                    Tout* __restrict__ out, int64_t ldo) {
    const int64_t ns = cnt[1];
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t u = gw; u < ns; u += nw) {
        const int64_t b = t_indptr[u], e = t_indptr[u + 1];
        for (int c0 = 0; c0 < Fi; c0 += 32) {
            const int c = c0 + lane;
            const bool act = c < Fi;
            float acc = 0.f;
            for (int64_t e0 = b; e0 < e; e0 += 32) {
                const int n = (int)mn64(32, e - e0);
                const int32_t my = lane < n ? t_idx[e0 + lane] : 0;
                for (int j = 0; j < n; ++j) {
                    const int32_t v = __shfl_sync(0xffffffffu, my, j);
                    if (act && arg[(int64_t)v * ldarg + c] == (int32_t)u) acc += dXA[(int64_t)v * ldd + Fp + c];
                }
            }
            if (act) st_act(out + u * ldo + c, Zp[u * ldz + c] > 0.f ? acc : 0.f);
        }
        for (int col = Fi + lane; col < ldo; col += 32) st_act(out + u * ldo + col, 0.f);
    }
}

// ------------------------------------ vectorised narrow-row gathers (LPR lanes / row)
// LPR lanes own a row and each lane up to PF_VPL 16-byte vectors of it, so a
// warp keeps 32/LPR rows (8 for the 48-wide layer of the products model) in
// flight; the edge loop takes LPR edge ids at a time (one per lane) and issues
// every neighbour vector of the batch before summing (predicated, unrolled).
constexpr int PF_VPL = 4;
static inline int pick_lpr_vpl(int nv) { return nv <= 4 * PF_VPL ? 4 : (nv <= 8 * PF_VPL ? 8 : (nv <= 16 * PF_VPL ? 16 : 32)); }

// mean, project-first fwd: S[v] = Y[v, Fop:] + (1/D_v) sum_u Y[u, :Fo] ; out = logits or ReLU -> H (+ ones)
template <typename Tout, int LPR>
__global__ void __launch_bounds__(256) k_agg_pf_v(const float* __restrict__ Y, const float* __restrict__ Ys, int64_t ldy,
                                                  const int64_t* __restrict__ indptr,
                                                  const int32_t* __restrict__ idx, const int64_t* cnt, int Fo, int Fop,
                                                  int relu, Tout* __restrict__ out, int64_t ldo, int sum) {
    constexpr int RPW = 32 / LPR;
    const int64_t nd = cnt[0];
    const int NV = (Fo + 3) / 4;
    const int lane = lane_id(), sub = lane % LPR, grp = lane / LPR;
    const unsigned gmask = LPR == 32 ? 0xffffffffu : (((1u << LPR) - 1u) << (grp * LPR));
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    int64_t nb = 0, ne = 0;                  // row extents one iteration ahead
    {
        const int64_t v = gw * RPW + grp;
        if (v < nd) { nb = indptr[v]; ne = indptr[v + 1]; }
    }
    for (int64_t v0 = gw * RPW; v0 < nd; v0 += nw * RPW) {
        const int64_t v = v0 + grp;
        const bool rowok = v < nd;
        const int64_t b = nb, e = ne;
        {
            const int64_t vn = v + nw * RPW;
            nb = 0; ne = 0;
            if (vn < nd) { nb = indptr[vn]; ne = indptr[vn + 1]; }
        }
        const float inv = e > b ? (sum ? 1.0f : 1.0f / (float)(e - b)) : 0.0f;
        for (int vb = 0; vb < NV; vb += LPR * PF_VPL) {
            float4 acc[PF_VPL];
#pragma unroll
            for (int k = 0; k < PF_VPL; ++k) acc[k] = make_float4(0.f, 0.f, 0.f, 0.f);
            for (int64_t e0 = b; e0 < e; e0 += LPR) {
                const int n = (int)mn64(LPR, e - e0);
                const int32_t my = sub < n ? idx[e0 + sub] : 0;
#pragma unroll
                for (int j = 0; j < LPR; ++j) {
                    const int32_t u = __shfl_sync(gmask, my, j, LPR);
                    if (j < n) {
#pragma unroll
                        for (int k = 0; k < PF_VPL; ++k) {
                            const int vi = vb + sub + LPR * k;
                            if (rowok && vi < NV) {
                                const float4 y = *(const float4*)(Y + (int64_t)u * ldy + vi * 4);
                                acc[k].x += y.x; acc[k].y += y.y; acc[k].z += y.z; acc[k].w += y.w;
                            }
                        }
                    }
                }
            }
#pragma unroll
            for (int k = 0; k < PF_VPL; ++k) {
                const int vi = vb + sub + LPR * k;
                if (rowok && vi < NV) {
                    const float4 sf = *(const float4*)(Ys + v * ldy + vi * 4);
                    float r[4] = {sf.x + acc[k].x * inv, sf.y + acc[k].y * inv, sf.z + acc[k].z * inv,
                                  sf.w + acc[k].w * inv};
#pragma unroll
                    for (int t = 0; t < 4; ++t) {
                        const int col = vi * 4 + t;
                        if (col < Fo) st_act(out + v * ldo + col, relu ? fmaxf(r[t], 0.f) : r[t]);
                    }
                }
            }
        }
        if (rowok && relu)
            for (int col = Fo + sub; col < ldo; col += LPR) st_act(out + v * ldo + col, col == Fo ? 1.f : 0.f);
    }
}

// mean, project-first bwd: G[u] = sum_{v in CSC(u)} dS[v]/D_v (the self half is dS itself)
template <typename Tin, typename Tout, int LPR>
__global__ void __launch_bounds__(256) k_csc_pf_v(const Tin* __restrict__ dS, int64_t ldds,
                                                  const int64_t* __restrict__ indptr,
                                                  const int64_t* __restrict__ t_indptr,
                                                  const int32_t* __restrict__ t_idx, const int64_t* cnt, int Fo,
                                                  int Fop, Tout* __restrict__ G, int64_t ldg) {
    using VI = Vec<Tin>;
    constexpr int VW = VI::N;
    constexpr int RPW = 32 / LPR;
    const int64_t nd = cnt[0], ns = cnt[1];
    const int NV = (Fop + VW - 1) / VW;
    const int lane = lane_id(), sub = lane % LPR, grp = lane / LPR;
    const unsigned gmask = LPR == 32 ? 0xffffffffu : (((1u << LPR) - 1u) << (grp * LPR));
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    // the next row group's column extents are loaded one iteration ahead (the CSC columns are short:
    // their extents are a dependent round trip in front of every other load)
    int64_t nb = 0, ne = 0;
    {
        const int64_t u = gw * RPW + grp;
        if (u < ns) { nb = t_indptr[u]; ne = t_indptr[u + 1]; }
    }
    for (int64_t u0 = gw * RPW; u0 < ns; u0 += nw * RPW) {
        const int64_t u = u0 + grp;
        const bool rowok = u < ns;
        const int64_t b = nb, e = ne;
        {
            const int64_t un = u + nw * RPW;
            nb = 0; ne = 0;
            if (un < ns) { nb = t_indptr[un]; ne = t_indptr[un + 1]; }
        }
        for (int vb = 0; vb < NV; vb += LPR * PF_VPL) {
            float acc[PF_VPL][VW];
#pragma unroll
            for (int k = 0; k < PF_VPL; ++k)
#pragma unroll
                for (int t = 0; t < VW; ++t) acc[k][t] = 0.f;
            for (int64_t e0 = b; e0 < e; e0 += LPR) {
                const int n = (int)mn64(LPR, e - e0);
                int32_t my = 0;
                float myinv = 0.f;
                if (sub < n) {
                    my = t_idx[e0 + sub];
                    myinv = indptr ? 1.0f / (float)(indptr[my + 1] - indptr[my]) : 1.0f;
                }
#pragma unroll
                for (int j = 0; j < LPR; ++j) {
                    const int32_t v = __shfl_sync(gmask, my, j, LPR);
                    const float iv = __shfl_sync(gmask, myinv, j, LPR);
                    if (j < n) {
#pragma unroll
                        for (int k = 0; k < PF_VPL; ++k) {
                            const int vi = vb + sub + LPR * k;
                            if (rowok && vi < NV) {
                                VI x;
                                x.load_cg(dS + (int64_t)v * ldds + vi * VW);
#pragma unroll
                                for (int t = 0; t < VW; ++t) acc[k][t] += x.v[t] * iv;
                            }
                        }
                    }
                }
            }
#pragma unroll
            for (int k = 0; k < PF_VPL; ++k) {
                const int vi = vb + sub + LPR * k;
                if (rowok && vi < NV) {
                    float ga[VW];
#pragma unroll
                    for (int t = 0; t < VW; ++t) ga[t] = vi * VW + t < Fo ? acc[k][t] : 0.f;
#pragma unroll
                    for (int t = 0; t < VW; t += 4) st_act4(G + u * ldg + vi * VW + t, ga + t);   // ldg multiple of 8
                }
            }
        }
    }
}

static inline int pick_lpr(int nv) { return nv <= 4 ? 4 : (nv <= 8 ? 8 : (nv <= 16 ? 16 : 32)); }

// ----------------------------------------------------------- launchers
static inline int warps_grid(betty_ctx* c, int64_t rows_cap) {
    return (int)std::max<int64_t>(1, std::min<int64_t>((rows_cap * 32 + 255) / 256, (int64_t)c->num_sms * 16));
}

#define DISPATCH_ACT(bf, T, ...)                              \
    if (bf) { using T = __nv_bfloat16; __VA_ARGS__; }          \
    else { using T = float; __VA_ARGS__; }

// grid = the CTAs that are resident at once (persistent sweep), at most the work
template <typename K> static int resident_grid(betty_ctx* c, K kernel, int threads, int64_t want_ctas) {
    int per_sm = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, threads, 0) != cudaSuccess || per_sm < 1)
        per_sm = 1;
    return (int)std::max<int64_t>(1, std::min<int64_t>(want_ctas, (int64_t)per_sm * c->num_sms));
}

// the gather4 pipeline (k_agg_mean_g4); false if the table cannot be described by a tensor map
static bool agg_mean_g4(betty_ctx* c, const void* X, bool x_bf16, int64_t ldx, const int32_t* srow,
                        const int32_t* erow, const int32_t* emap, const int64_t* indptr, const int64_t* cnt,
                        const int64_t* otab, int Fi, int Fp, int nv, void* XA, bool xa_bf16, int64_t ldxa, int hint,
                        unsigned* ctr, bool sum, cudaStream_t s) {
    const int vw = x_bf16 ? 8 : 4;
    CUtensorMap tm;
    if (!make_gather_map(&tm, X, !x_bf16, (int64_t)nv * vw, (int64_t)INT32_MAX, ldx, nv * vw)) return false;
    G4Args a{};
    a.srow = srow; a.erow = erow; a.emap = emap; a.indptr = indptr; a.cnt = cnt; a.otab = otab;
    a.XA = XA; a.ldxa = ldxa; a.X = X; a.ldx = ldx; a.ctr = ctr; a.Fi = Fi; a.Fp = Fp; a.NV = nv; a.hint = hint;
    a.sum = sum ? 1 : 0;
    a.row_bytes = (uint32_t)nv * 16u;
    a.grp_bytes = (4u * a.row_bytes + 127u) / 128u * 128u;
    const size_t red_bytes = 0;
    static int static_smem = -1;                                      // the kernel's static footprint
    if (static_smem < 0) {
        cudaFuncAttributes fa{};
        if (x_bf16) cudaFuncGetAttributes(&fa, xa_bf16 ? k_agg_mean_g4<__nv_bfloat16, __nv_bfloat16>
                                                       : k_agg_mean_g4<__nv_bfloat16, float>);
        else cudaFuncGetAttributes(&fa, xa_bf16 ? k_agg_mean_g4<float, __nv_bfloat16> : k_agg_mean_g4<float, float>);
        static_smem = (int)fa.sharedSizeBytes;
    }
    // dynamic smem for the stage ring: up to 196 KB, within the 227 KB opt-in minus the static part
    const size_t budget = std::min<size_t>((size_t)196 * 1024, (size_t)(227 * 1024 - static_smem - 1024)) - red_bytes;
    const int64_t groups = (int64_t)(budget / G4_STAGES) / a.grp_bytes - G4_MAXR / 4;
    if (groups < 4) return false;
    a.slot_groups = (uint32_t)std::min<int64_t>(groups, 64);     // a producer lane issues <= 2 groups
    a.stage_bytes = (a.slot_groups + G4_MAXR / 4) * a.grp_bytes;
    const size_t sm = (size_t)G4_STAGES * a.stage_bytes + red_bytes;
    DISPATCH_ACT(x_bf16, TI, DISPATCH_ACT(xa_bf16, TO, {
        static int max_dyn = -1;
        if (max_dyn < 0) {       // the opt-in maximum per CTA (227 KB) minus the kernel's static shared memory
            cudaFuncAttributes fa{};
            cudaFuncGetAttributes(&fa, k_agg_mean_g4<TI, TO>);
            max_dyn = 227 * 1024 - (int)fa.sharedSizeBytes;
            cudaFuncSetAttribute(k_agg_mean_g4<TI, TO>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_dyn);
        }
        if ((int)sm > max_dyn) return false;
        cudaMemsetAsync(ctr, 0, sizeof(unsigned), s);
        // BETTY_G4_GRID: (study) fewer CTAs than SMs -- the kernel's time scales as 1 / grid
        // (profiles/r03_agg_bound.txt: its bound is inside each SM, not L2 or HBM)
        static const int g4_grid = getenv("BETTY_G4_GRID") ? atoi(getenv("BETTY_G4_GRID")) : 0;
        k_agg_mean_g4<TI, TO><<<g4_grid > 0 ? g4_grid : c->num_sms, G4_THREADS, sm, s>>>(tm, a);
    }))
    return true;
}

void agg_mean_xa(betty_ctx* c, const void* X, bool x_bf16, int64_t ldx, const int32_t* srow, const int32_t* erow,
                 const int32_t* emap, const int64_t* indptr, const int64_t* cnt, const int64_t* otab, int64_t rows_cap,
                 int64_t src_per_mb, int Fi, int Fp, void* XA, bool xa_bf16, int64_t ldxa, bool sum,
                 const FeatShards* shards, cudaStream_t s) {
    const int vw = x_bf16 ? 8 : 4;
    FeatShards sh;
    if (shards) sh = *shards;
    const int nv = (Fi + vw - 1) / vw;
    // Column passes: one micro-batch's gathered rows must stay L2-resident between their
    // uses; when (source rows of a micro-batch) x (row bytes) exceeds the budget, the
    // feature columns are gathered in several passes over the rows, each pass touching
    // only a slice of every row (the rows' metadata is re-read, the features are not).
    static const double budget = getenv("BETTY_AGG_WS_MB") ? atof(getenv("BETTY_AGG_WS_MB")) * 1e6 : 1e12;
    unsigned* ctr = c->L().counters + CTR_AGG;
    static const int hint_env = getenv("BETTY_AGG_CA") ? 3 :
                                (getenv("BETTY_AGG_NOHINT") ? 0 : (getenv("BETTY_AGG_NOBULK") ? 2 : 1));
    // sharded tables: per-lane cp.async gathers (whole-row bulk copies are not used on peer memory)
    const int hint = sh.R > 0 ? 2 : hint_env;
    static const bool no_order = getenv("BETTY_AGG_NOORDER") != nullptr;
    const double ws = (double)src_per_mb * (double)nv * 16.0;
    int passes = (int)std::max(1.0, std::min((double)nv, std::ceil(ws / budget)));
    const int pv = (nv + passes - 1) / passes;
    passes = (nv + pv - 1) / pv;
    static const bool g4_off = getenv("BETTY_AGG_G4") && atoi(getenv("BETTY_AGG_G4")) == 0;
    if (!g4_off && sh.R == 0 && passes == 1 && nv * vw <= 256 && agg_mean_g4(c, X, x_bf16, ldx, srow, erow, emap, indptr, cnt, otab,
                                                                Fi, Fp, nv, XA, xa_bf16, ldxa, hint, ctr, sum, s))
        return;
    const int lpr = pv <= 8 ? 8 : (pv <= 16 ? 16 : 32);
    const int64_t warps = (rows_cap + (32 / lpr) - 1) / (32 / lpr);
#define AGG_L(LPR) DISPATCH_ACT(x_bf16, TI, DISPATCH_ACT(xa_bf16, TO, {                                           \
        const size_t sm = (size_t)8 * (32 / LPR) * ((AGG_EB < LPR ? AGG_EB : LPR) + 1) * LPR * 16;                    \
        static bool attr = false;                                                                              \
        if (!attr) { cudaFuncSetAttribute(k_agg_mean_xa<TI, TO, LPR>, cudaFuncAttributeMaxDynamicSharedMemorySize, \
                                          (int)sm); attr = true; }                                             \
        int per_sm = 1;                                                                                        \
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_agg_mean_xa<TI, TO, LPR>, 256, sm);           \
        const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((warps + 7) / 8, (int64_t)std::max(per_sm, 1) * c->num_sms)); \
        for (int pz = 0; pz < passes; ++pz) {                                                                   \
            cudaMemsetAsync(ctr, 0, sizeof(unsigned), s);                                                      \
            k_agg_mean_xa<TI, TO, LPR><<<grid, 256, sm, s>>>((const TI*)X, ldx, srow, erow, emap, indptr, cnt,    \
                no_order ? nullptr : otab, Fi, Fp, (TO*)XA, ldxa, hint, pz * pv, std::min(nv, (pz + 1) * pv), ctr, \
                sum ? 1 : 0, sh); } }))
    if (lpr == 8) { AGG_L(8); } else if (lpr == 16) { AGG_L(16); } else { AGG_L(32); }
#undef AGG_L
}

void agg_mean_pf(betty_ctx* c, const float* Y, const float* Ys, int64_t ldy, const int64_t* indptr, const int32_t* idx,
                 const int64_t* cnt, int64_t rows_cap, int Fo, int Fop, bool relu, void* out, bool out_bf16,
                 int64_t ldo, bool sum, cudaStream_t s) {
    const int lpr = pick_lpr_vpl((Fo + 3) / 4);
    const int grid = warps_grid(c, (rows_cap + (32 / lpr) - 1) / (32 / lpr));
#define PF_L(LPR) DISPATCH_ACT(out_bf16, TO, \
        k_agg_pf_v<TO, LPR><<<grid, 256, 0, s>>>(Y, Ys, ldy, indptr, idx, cnt, Fo, Fop, relu ? 1 : 0, (TO*)out, ldo, \
                                                 sum ? 1 : 0))
    if (lpr == 4) { PF_L(4); } else if (lpr == 8) { PF_L(8); } else if (lpr == 16) { PF_L(16); } else { PF_L(32); }
#undef PF_L
}

void gather_ones(betty_ctx* c, const void* X, bool x_bf16, int64_t ldx, const int32_t* xrow, const int64_t* cnt_rows,
                 int64_t rows_cap, int Fi, void* out, bool out_bf16, int64_t ldo, cudaStream_t s) {
    DISPATCH_ACT(x_bf16, TI, DISPATCH_ACT(out_bf16, TO,
        k_gather_ones<TI, TO><<<warps_grid(c, rows_cap), 256, 0, s>>>((const TI*)X, ldx, xrow, cnt_rows, Fi, (TO*)out,
                                                                      ldo)));
}

void csc_mean(betty_ctx* c, const float* dXA, int64_t ldd, const int64_t* indptr, const int64_t* t_indptr,
              const int32_t* t_idx, const int64_t* cnt, int64_t src_cap, int Fi, int Fp, const void* H, bool h_bf16,
              int64_t ldh, const uint32_t* hbits, int64_t ldhb, void* out, bool out_bf16, int64_t ldo,
              cudaStream_t s) {
    static const bool scalar = getenv("BETTY_CSC_MEAN_SCALAR") != nullptr;     // A/B switches
    static const bool warp_form = getenv("BETTY_CSC_MEAN_WARP") != nullptr;
    const int vpl = (Fi / 4 + 31) / 32;
    const int ng = Fi / 4;
    if (!scalar && !warp_form && Fi % 4 == 0 && Fp % 4 == 0 && ldd % 4 == 0 && ldo % 4 == 0 && ng % 4 == 0 &&
        (ng / 4) <= 32 && ((ng / 4) & (ng / 4 - 1)) == 0 && ((uintptr_t)dXA & 15) == 0 && ((uintptr_t)out & 15) == 0) {
#define CM_G(LP) do {                                                                                         \
        const int g = warps_grid(c, (src_cap + (32 / LP) - 1) / (32 / LP));                                   \
        DISPATCH_ACT(h_bf16, TM, DISPATCH_ACT(out_bf16, TO,                                                    \
        k_csc_mean_g<TM, TO, LP, 4, 2><<<g, 256, 0, s>>>(dXA, ldd, indptr, t_indptr, t_idx, cnt, Fi, Fp,        \
                                                         (const TM*)H, ldh, hbits, ldhb, (TO*)out, ldo))); } while (0)
        // 4 float4 groups per lane, 2 edges' rows in flight (C5@0.1: 22.4 ms/step vs 23.3 for 8 groups
        // per lane and 23.9 for 4 edges in flight -- measured)
        const int lpr = ng / 4;
        if (lpr == 1) { CM_G(1); } else if (lpr == 2) { CM_G(2); } else if (lpr == 4) { CM_G(4); }
        else if (lpr == 8) { CM_G(8); } else if (lpr == 16) { CM_G(16); } else { CM_G(32); }
#undef CM_G
        return;
    }
    if (!scalar && Fi % 4 == 0 && Fp % 4 == 0 && ldd % 4 == 0 && ldo % 4 == 0 && vpl <= 4 &&
        ((uintptr_t)dXA & 15) == 0 && ((uintptr_t)out & 15) == 0) {
        const int g = warps_grid(c, src_cap);
#define CM_V(V) DISPATCH_ACT(h_bf16, TM, DISPATCH_ACT(out_bf16, TO,                                              \
        k_csc_mean_v<TM, TO, V><<<g, 256, 0, s>>>(dXA, ldd, indptr, t_indptr, t_idx, cnt, Fi, Fp, (const TM*)H, ldh, \
                                                  hbits, ldhb, (TO*)out, ldo)))
        if (vpl <= 1) { CM_V(1); } else if (vpl == 2) { CM_V(2); } else { CM_V(4); }
#undef CM_V
        return;
    }
    DISPATCH_ACT(h_bf16, TM, DISPATCH_ACT(out_bf16, TO,
        k_csc_mean<TM, TO><<<warps_grid(c, src_cap), 256, 0, s>>>(dXA, ldd, indptr, t_indptr, t_idx, cnt, Fi, Fp,
                                                                  (const TM*)H, ldh, (TO*)out, ldo)));
}

void csc_pf(betty_ctx* c, const void* dS, bool ds_bf16, int64_t ldds, const int64_t* indptr, const int64_t* t_indptr,
            const int32_t* t_idx, const int64_t* cnt, int64_t src_cap, int Fo, int Fop, void* G, bool g_bf16,
            int64_t ldg, cudaStream_t s) {
    const int lpr = pick_lpr_vpl((Fop + (ds_bf16 ? 7 : 3)) / (ds_bf16 ? 8 : 4));
    const int grid = warps_grid(c, (src_cap + (32 / lpr) - 1) / (32 / lpr));
#define CSC_L(LPR) DISPATCH_ACT(ds_bf16, TI, DISPATCH_ACT(g_bf16, TO, \
        k_csc_pf_v<TI, TO, LPR><<<grid, 256, 0, s>>>((const TI*)dS, ldds, indptr, t_indptr, t_idx, cnt, Fo, Fop, \
                                                    (TO*)G, ldg)))
    if (lpr == 4) { CSC_L(4); } else if (lpr == 8) { CSC_L(8); } else if (lpr == 16) { CSC_L(16); } else { CSC_L(32); }
#undef CSC_L
}

void agg_pool(betty_ctx* c, const void* X, bool x_bf16, int64_t ldx, const int32_t* xrow, const float* Zp, int64_t ldz,
              const int64_t* indptr, const int32_t* idx, const int64_t* cnt, int64_t rows_cap, int Fi, int Fp,
              void* XA, bool xa_bf16, int64_t ldxa, void* arg, int64_t ldarg, bool pos8, cudaStream_t s) {
    const int ng = (Fi + 3) / 4;
    const bool vec = (ldz % 4) == 0 && ng <= 64 && ((uintptr_t)Zp & 15) == 0 && ((uintptr_t)arg & 15) == 0 &&
                     (pos8 ? (ldarg % 4) == 0 : (ldarg % 4) == 0);
    if (vec) {
        const int g = warps_grid(c, rows_cap);
#define POOL_V(T, P) k_agg_pool_v<TI, TO, T, P><<<g, 256, 0, s>>>((const TI*)X, ldx, xrow, Zp, ldz, indptr, idx, cnt, \
                                                                   Fi, Fp, (TO*)XA, ldxa, arg, ldarg)
        DISPATCH_ACT(x_bf16, TI, DISPATCH_ACT(xa_bf16, TO, {
            if (ng <= 32) { if (pos8) POOL_V(1, true); else POOL_V(1, false); }
            else { if (pos8) POOL_V(2, true); else POOL_V(2, false); } }))
#undef POOL_V
        return;
    }
    if (pos8) { fprintf(stderr, "betty: pool byte positions need the vectorised kernel\n"); return; }
    DISPATCH_ACT(x_bf16, TI, DISPATCH_ACT(xa_bf16, TO,
        k_agg_pool<TI, TO><<<warps_grid(c, rows_cap), 256, 0, s>>>((const TI*)X, ldx, xrow, Zp, ldz, indptr, idx, cnt,
                                                                   Fi, Fp, (TO*)XA, ldxa, (int32_t*)arg, ldarg)));
}

void route_pool(betty_ctx* c, const float* dXA, int64_t ldd, const void* arg, int64_t ldarg, bool pos8,
                const int64_t* indptr, const int32_t* idx, const int64_t* t_indptr, const int32_t* t_idx,
                const int64_t* cnt, int64_t src_cap, int Fi, int Fp, const float* Zp, int64_t ldz, void* out,
                bool out_bf16, int64_t ldo, cudaStream_t s) {
    const int ng = (Fi + 3) / 4;
    const bool vec = (ldz % 4) == 0 && (ldarg % 4) == 0 && (ldd % 4) == 0 && (Fp % 4) == 0 && ng <= 64 &&
                     ((uintptr_t)Zp & 15) == 0 && ((uintptr_t)arg & 15) == 0 && ((uintptr_t)dXA & 15) == 0;
    if (vec) {
        const int g = warps_grid(c, src_cap);
#define ROUTE_V(T, P) k_route_pool_v<TO, T, P><<<g, 256, 0, s>>>(dXA, ldd, arg, ldarg, indptr, idx, t_indptr, t_idx, \
                                                                 cnt, Fi, Fp, Zp, ldz, (TO*)out, ldo)
        DISPATCH_ACT(out_bf16, TO, {
            if (ng <= 32) { if (pos8) ROUTE_V(1, true); else ROUTE_V(1, false); }
            else { if (pos8) ROUTE_V(2, true); else ROUTE_V(2, false); } })
#undef ROUTE_V
        return;
    }
    if (pos8) { fprintf(stderr, "betty: pool byte positions need the vectorised kernel\n"); return; }
    DISPATCH_ACT(out_bf16, TO,
        k_route_pool<TO><<<warps_grid(c, src_cap), 256, 0, s>>>(dXA, ldd, (const int32_t*)arg, ldarg, t_indptr, t_idx,
                                                                cnt, Fi, Fp, Zp, ldz, (TO*)out, ldo));
}

}  // namespace betty
