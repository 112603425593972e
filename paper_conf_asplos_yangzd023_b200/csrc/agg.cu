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

// ------------------------------------------------ mean, aggregate-first fwd
// LPR lanes own one dst row (RPW = 32/LPR rows per warp in flight); each lane
// covers 16-byte vectors of the feature row and keeps AGG_BATCH neighbour
// rows in flight.  The neighbour X-row of edge e is emap ? emap[erow[e]] : erow[e]
// (layer 0 passes the edge -> global-id array written by the extraction, so no
// dependent id lookup stays on the critical path); the self row of dst v is
// srow ? srow[v] : v.  With an order table (extract.h) the rows are visited
// micro-batch by micro-batch, so the source rows one micro-batch shares stay
// in L2 between their uses; the grid is exactly the resident CTAs so all warps
// sweep the order together.
constexpr int AGG_BATCH = 4;     // neighbour rows in flight per lane (x 16 B)
template <typename Tin, typename Tout, int LPR>
__global__ void __launch_bounds__(256, 4) k_agg_mean_xa(const Tin* __restrict__ X, int64_t ldx,
                                                     const int32_t* __restrict__ srow,
                                                     const int32_t* __restrict__ erow,
                                                     const int32_t* __restrict__ emap,
                                                     const int64_t* __restrict__ indptr, const int64_t* cnt,
                                                     const int64_t* __restrict__ otab, int Fi, int Fp,
                                                     Tout* __restrict__ XA, int64_t ldxa) {
    using VI = Vec<Tin>;
    constexpr int VW = VI::N;
    constexpr int RPW = 32 / LPR;
    __shared__ int64_t s_vs[ORDER_SMEM + 1], s_rs[ORDER_SMEM];
    const int64_t nd = cnt[0];
    const int nseg = order_load(otab, s_vs, s_rs);
    const int NV = (Fi + VW - 1) / VW;
    const int lane = lane_id(), sub = lane % LPR, grp = lane / LPR;
    const unsigned gmask = LPR == 32 ? 0xffffffffu : (((1u << LPR) - 1u) << (grp * LPR));
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    int seg = 0;
    for (int64_t v0 = gw * RPW; v0 < nd; v0 += nw * RPW) {
        const int64_t vv = v0 + grp;
        const bool rowok = vv < nd;
        const int64_t v = rowok ? order_map(vv, nseg, s_vs, s_rs, seg) : vv;
        int64_t b = 0, e = 0;
        if (rowok) { b = indptr[v]; e = indptr[v + 1]; }
        const float inv = e > b ? 1.0f / (float)(e - b) : 0.0f;
        Tout* out = XA + v * ldxa;
        for (int vb = 0; vb < NV; vb += LPR) {
            const int vi = vb + sub;
            const bool act = rowok && vi < NV;
            float acc[VW];
#pragma unroll
            for (int t = 0; t < VW; ++t) acc[t] = 0.f;
            for (int64_t e0 = b; e0 < e; e0 += LPR) {
                const int n = (int)mn64(LPR, e - e0);
                int32_t my = 0;
                if (sub < n) { my = erow[e0 + sub]; if (emap) my = emap[my]; }
                for (int j = 0; j < n; j += AGG_BATCH) {
                    typename VI::Raw x[AGG_BATCH];
#pragma unroll
                    for (int t = 0; t < AGG_BATCH; ++t) {
                        const int32_t u = __shfl_sync(gmask, my, (j + t) & (LPR - 1), LPR);
                        x[t] = (act && j + t < n) ? VI::ld_raw(X + (int64_t)u * ldx + vi * VW) : VI::zero_raw();
                    }
#pragma unroll
                    for (int t = 0; t < AGG_BATCH; ++t) VI::add_raw(acc, x[t]);
                }
            }
            if (act) {
                VI self;
                self.load(X + (int64_t)(srow ? srow[v] : (int32_t)v) * ldx + vi * VW);
                if constexpr (sizeof(Tin) == sizeof(Tout)) {
                    Vec<Tout> so, ao;
#pragma unroll
                    for (int t = 0; t < VW; ++t) {
                        const bool in = vi * VW + t < Fi;
                        so.v[t] = in ? self.v[t] : 0.f;
                        ao.v[t] = in ? acc[t] * inv : 0.f;
                    }
                    so.store(out + vi * VW);
                    ao.store(out + Fp + vi * VW);
                } else {
#pragma unroll
                    for (int t = 0; t < VW; ++t) {
                        const int col = vi * VW + t;
                        if (col < Fi) { st_act(out + col, self.v[t]); st_act(out + Fp + col, acc[t] * inv); }
                    }
                }
            }
        }
        if (rowok) {
            // pad columns of both halves, the ones column (bias), trailing pad
            for (int col = NV * VW + sub; col < Fp; col += LPR) { st_act(out + col, 0.f); st_act(out + Fp + col, 0.f); }
            for (int col = 2 * Fp + sub; col < ldxa; col += LPR) st_act(out + col, col == 2 * Fp ? 1.f : 0.f);
        }
    }
}

// ------------------------------------------------ mean, project-first fwd
// S[v,c] = Y[v, Fop + c] + (1/D_v) sum_u Y[u, c];  out = logits (fp32) or ReLU -> H (+ones col)
template <typename Tout>
__global__ void __launch_bounds__(256) k_agg_mean_pf(const float* __restrict__ Y, int64_t ldy,
                                                     const int64_t* __restrict__ indptr,
                                                     const int32_t* __restrict__ idx, const int64_t* cnt, int Fo,
                                                     int Fop, int relu, Tout* __restrict__ out, int64_t ldo) {
    const int64_t nd = cnt[0];
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t v = gw; v < nd; v += nw) {
        const int64_t b = indptr[v], e = indptr[v + 1];
        const float inv = e > b ? 1.0f / (float)(e - b) : 0.0f;
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
                    myinv = 1.0f / (float)(indptr[my + 1] - indptr[my]);
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
                    myinv = 1.0f / (float)(indptr[my + 1] - indptr[my]);
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
// mean, project-first fwd: S[v] = Y[v, Fop:] + (1/D_v) sum_u Y[u, :Fo] ; out = logits or ReLU -> H (+ ones)
template <typename Tout, int LPR>
__global__ void __launch_bounds__(256) k_agg_pf_v(const float* __restrict__ Y, int64_t ldy,
                                                  const int64_t* __restrict__ indptr,
                                                  const int32_t* __restrict__ idx, const int64_t* cnt, int Fo, int Fop,
                                                  int relu, Tout* __restrict__ out, int64_t ldo) {
    constexpr int RPW = 32 / LPR;
    const int64_t nd = cnt[0];
    const int NV = (Fo + 3) / 4;
    const int lane = lane_id(), sub = lane % LPR, grp = lane / LPR;
    const unsigned gmask = LPR == 32 ? 0xffffffffu : (((1u << LPR) - 1u) << (grp * LPR));
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t v0 = gw * RPW; v0 < nd; v0 += nw * RPW) {
        const int64_t v = v0 + grp;
        const bool rowok = v < nd;
        int64_t b = 0, e = 0;
        if (rowok) { b = indptr[v]; e = indptr[v + 1]; }
        const float inv = e > b ? 1.0f / (float)(e - b) : 0.0f;
        for (int vb = 0; vb < NV; vb += LPR) {
            const int vi = vb + sub;
            const bool act = rowok && vi < NV;
            float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
            for (int64_t e0 = b; e0 < e; e0 += LPR) {
                const int n = (int)mn64(LPR, e - e0);
                const int32_t my = sub < n ? idx[e0 + sub] : 0;
                for (int j = 0; j < n; ++j) {
                    const int32_t u = __shfl_sync(gmask, my, j, LPR);
                    if (act) {
                        const float4 y = *(const float4*)(Y + (int64_t)u * ldy + vi * 4);
                        acc.x += y.x; acc.y += y.y; acc.z += y.z; acc.w += y.w;
                    }
                }
            }
            if (act) {
                const float4 sf = *(const float4*)(Y + v * ldy + Fop + vi * 4);
                float r[4] = {sf.x + acc.x * inv, sf.y + acc.y * inv, sf.z + acc.z * inv, sf.w + acc.w * inv};
#pragma unroll
                for (int t = 0; t < 4; ++t) {
                    const int col = vi * 4 + t;
                    if (col < Fo) st_act(out + v * ldo + col, relu ? fmaxf(r[t], 0.f) : r[t]);
                }
            }
        }
        if (rowok && relu)
            for (int col = Fo + sub; col < ldo; col += LPR) st_act(out + v * ldo + col, col == Fo ? 1.f : 0.f);
    }
}

// mean, project-first bwd: G[u] = [ sum_{v in CSC(u)} dS[v]/D_v | 0 | [u < nd] dS[u] | 0 ]
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
    for (int64_t u0 = gw * RPW; u0 < ns; u0 += nw * RPW) {
        const int64_t u = u0 + grp;
        const bool rowok = u < ns;
        int64_t b = 0, e = 0;
        if (rowok) { b = t_indptr[u]; e = t_indptr[u + 1]; }
        for (int vb = 0; vb < NV; vb += LPR) {
            const int vi = vb + sub;
            const bool act = rowok && vi < NV;
            float acc[VW];
#pragma unroll
            for (int t = 0; t < VW; ++t) acc[t] = 0.f;
            for (int64_t e0 = b; e0 < e; e0 += LPR) {
                const int n = (int)mn64(LPR, e - e0);
                int32_t my = 0;
                float myinv = 0.f;
                if (sub < n) {
                    my = t_idx[e0 + sub];
                    myinv = 1.0f / (float)(indptr[my + 1] - indptr[my]);
                }
                for (int j = 0; j < n; ++j) {
                    const int32_t v = __shfl_sync(gmask, my, j, LPR);
                    const float iv = __shfl_sync(gmask, myinv, j, LPR);
                    if (act) {
                        VI x;
                        x.load_cg(dS + (int64_t)v * ldds + vi * VW);
#pragma unroll
                        for (int t = 0; t < VW; ++t) acc[t] += x.v[t] * iv;
                    }
                }
            }
            if (act) {
                VI self;
                if (u < nd) self.load_cg(dS + u * ldds + vi * VW);
                float ga[VW], gs[VW];
#pragma unroll
                for (int t = 0; t < VW; ++t) {
                    const bool in = vi * VW + t < Fo;
                    ga[t] = in ? acc[t] : 0.f;
                    gs[t] = (in && u < nd) ? self.v[t] : 0.f;
                }
#pragma unroll
                for (int t = 0; t < VW; t += 4) {        // vector stores (Fop, ldg multiples of 8)
                    st_act4(G + u * ldg + vi * VW + t, ga + t);
                    st_act4(G + u * ldg + Fop + vi * VW + t, gs + t);
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

void agg_mean_xa(betty_ctx* c, const void* X, bool x_bf16, int64_t ldx, const int32_t* srow, const int32_t* erow,
                 const int32_t* emap, const int64_t* indptr, const int64_t* cnt, const int64_t* otab, int64_t rows_cap,
                 int Fi, int Fp, void* XA, bool xa_bf16, int64_t ldxa, cudaStream_t s) {
    const int vw = x_bf16 ? 8 : 4;
    const int nv = (Fi + vw - 1) / vw;
    const int lpr = nv <= 8 ? 8 : (nv <= 16 ? 16 : 32);
    const int64_t warps = (rows_cap + (32 / lpr) - 1) / (32 / lpr);
#define AGG_L(LPR) DISPATCH_ACT(x_bf16, TI, DISPATCH_ACT(xa_bf16, TO, \
        k_agg_mean_xa<TI, TO, LPR><<<resident_grid(c, k_agg_mean_xa<TI, TO, LPR>, 256, (warps + 7) / 8), 256, 0, s>>>( \
            (const TI*)X, ldx, srow, erow, emap, indptr, cnt, otab, Fi, Fp, (TO*)XA, ldxa)))
    if (lpr == 8) { AGG_L(8); } else if (lpr == 16) { AGG_L(16); } else { AGG_L(32); }
#undef AGG_L
}

void agg_mean_pf(betty_ctx* c, const float* Y, int64_t ldy, const int64_t* indptr, const int32_t* idx,
                 const int64_t* cnt, int64_t rows_cap, int Fo, int Fop, bool relu, void* out, bool out_bf16,
                 int64_t ldo, cudaStream_t s) {
    const int lpr = pick_lpr((Fo + 3) / 4);
    const int grid = warps_grid(c, (rows_cap + (32 / lpr) - 1) / (32 / lpr));
#define PF_L(LPR) DISPATCH_ACT(out_bf16, TO, \
        k_agg_pf_v<TO, LPR><<<grid, 256, 0, s>>>(Y, ldy, indptr, idx, cnt, Fo, Fop, relu ? 1 : 0, (TO*)out, ldo))
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
              int64_t ldh, void* out, bool out_bf16, int64_t ldo, cudaStream_t s) {
    DISPATCH_ACT(h_bf16, TM, DISPATCH_ACT(out_bf16, TO,
        k_csc_mean<TM, TO><<<warps_grid(c, src_cap), 256, 0, s>>>(dXA, ldd, indptr, t_indptr, t_idx, cnt, Fi, Fp,
                                                                  (const TM*)H, ldh, (TO*)out, ldo)));
}

void csc_pf(betty_ctx* c, const void* dS, bool ds_bf16, int64_t ldds, const int64_t* indptr, const int64_t* t_indptr,
            const int32_t* t_idx, const int64_t* cnt, int64_t src_cap, int Fo, int Fop, void* G, bool g_bf16,
            int64_t ldg, cudaStream_t s) {
    const int lpr = pick_lpr((Fop + (ds_bf16 ? 7 : 3)) / (ds_bf16 ? 8 : 4));
    const int grid = warps_grid(c, (src_cap + (32 / lpr) - 1) / (32 / lpr));
#define CSC_L(LPR) DISPATCH_ACT(ds_bf16, TI, DISPATCH_ACT(g_bf16, TO, \
        k_csc_pf_v<TI, TO, LPR><<<grid, 256, 0, s>>>((const TI*)dS, ldds, indptr, t_indptr, t_idx, cnt, Fo, Fop, \
                                                    (TO*)G, ldg)))
    if (lpr == 4) { CSC_L(4); } else if (lpr == 8) { CSC_L(8); } else if (lpr == 16) { CSC_L(16); } else { CSC_L(32); }
#undef CSC_L
}

void agg_pool(betty_ctx* c, const void* X, bool x_bf16, int64_t ldx, const int32_t* xrow, const float* Zp, int64_t ldz,
              const int64_t* indptr, const int32_t* idx, const int64_t* cnt, int64_t rows_cap, int Fi, int Fp,
              void* XA, bool xa_bf16, int64_t ldxa, int32_t* arg, int64_t ldarg, cudaStream_t s) {
    DISPATCH_ACT(x_bf16, TI, DISPATCH_ACT(xa_bf16, TO,
        k_agg_pool<TI, TO><<<warps_grid(c, rows_cap), 256, 0, s>>>((const TI*)X, ldx, xrow, Zp, ldz, indptr, idx, cnt,
                                                                   Fi, Fp, (TO*)XA, ldxa, arg, ldarg)));
}

void route_pool(betty_ctx* c, const float* dXA, int64_t ldd, const int32_t* arg, int64_t ldarg,
                const int64_t* t_indptr, const int32_t* t_idx, const int64_t* cnt, int64_t src_cap, int Fi, int Fp,
                const float* Zp, int64_t ldz, void* out, bool out_bf16, int64_t ldo, cudaStream_t s) {
    DISPATCH_ACT(out_bf16, TO,
        k_route_pool<TO><<<warps_grid(c, src_cap), 256, 0, s>>>(dXA, ldd, arg, ldarg, t_indptr, t_idx, cnt, Fi, Fp, Zp,
                                                                ldz, (TO*)out, ldo));
}

}  // namespace betty
