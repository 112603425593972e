// misc.cu -- a4 softmax cross-entropy (fused forward + backward), a7 Adam,
// and the per-step weight layout preparation (fp32 params -> GEMM layouts,
// cast to bf16 in BF16 mode).
#include <cmath>
#include <cstdlib>
#include "common.cuh"
#include "internal.h"
#include "sage.h"

namespace betty {

// ------------------------------------------------------------------ loss
// loss_accum += scale * sum_v [logsumexp(S_v) - S_v[y_v]] ;  dS_v = scale * (softmax(S_v) - onehot(y_v))
// (reading #15: scale = 1 / n_out of the full batch).  One warp per row, LOSS_R rows per warp at a
// time (their loads issued together and their shuffle reductions interleaved: one row's chain of
// dependent loads and shuffles left the warp stalled, ncu r02r), C <= 256.  The loss is reduced
// deterministically: per-CTA partials in a fixed order, summed by the last CTA.
constexpr int LOSS_MAXT_CAP = 8;               // C <= 256

template <typename TA, int LOSS_MAXT>        // LOSS_MAXT = ceil(C / 32) column groups per lane
__global__ void __launch_bounds__(256) k_loss(const float* __restrict__ logits, int64_t ldl,
                                              const int32_t* __restrict__ labels, const int32_t* __restrict__ gid,
                                              const int64_t* cnt, int C, float scale, float* __restrict__ dS,
                                              int64_t ldds, TA* __restrict__ dS_act, int64_t ld_act,
                                              const int64_t* __restrict__ indptr, double* partials, unsigned* ctr,
                                              float* loss_accum) {
    constexpr int R = LOSS_MAXT <= 2 ? 4 : (LOSS_MAXT <= 4 ? 2 : 1);
    __shared__ double s_w[8];
    __shared__ int s_last;
    const int64_t nd = cnt[0];
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    double wl = 0.0;
    for (int64_t v0 = gw * R; v0 < nd; v0 += nw * R) {
        int32_t gi[R], y[R];
        int64_t dg[R];
        float x[R][LOSS_MAXT];
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const int64_t v = v0 + r;
            const bool ok = v < nd;
            gi[r] = ok ? gid[v] : 0;
            dg[r] = (ok && indptr) ? indptr[v + 1] - indptr[v] : 1;
#pragma unroll
            for (int t = 0; t < LOSS_MAXT; ++t) {
                const int c = lane + 32 * t;
                x[r][t] = (ok && c < C) ? logits[v * ldl + c] : -INFINITY;
            }
        }
#pragma unroll
        for (int r = 0; r < R; ++r) y[r] = v0 + r < nd ? labels[gi[r]] : -1;
        float mx[R], se[R], lse[R], xy[R];
#pragma unroll
        for (int r = 0; r < R; ++r) {
            mx[r] = -INFINITY;
#pragma unroll
            for (int t = 0; t < LOSS_MAXT; ++t) mx[r] = fmaxf(mx[r], x[r][t]);
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1)
#pragma unroll
            for (int r = 0; r < R; ++r) mx[r] = fmaxf(mx[r], __shfl_xor_sync(0xffffffffu, mx[r], o));
#pragma unroll
        for (int r = 0; r < R; ++r) {
            se[r] = 0.f;
#pragma unroll
            for (int t = 0; t < LOSS_MAXT; ++t)
                if (lane + 32 * t < C) se[r] += expf(x[r][t] - mx[r]);
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1)
#pragma unroll
            for (int r = 0; r < R; ++r) se[r] += __shfl_xor_sync(0xffffffffu, se[r], o);
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const int64_t v = v0 + r;
            lse[r] = mx[r] + logf(se[r]);
            xy[r] = 0.f;
            if (v >= nd) continue;
            // indptr (project-first top layer): the fp32 dS is stored pre-scaled by 1/D_v for P^T D+ dS
            const float inv = indptr ? (dg[r] > 0 ? 1.f / (float)dg[r] : 0.f) : 1.f;
#pragma unroll
            for (int t = 0; t < LOSS_MAXT; ++t) {
                const int c = lane + 32 * t;
                if (c == y[r]) xy[r] = x[r][t];
                if (c < C) {
                    const float d = scale * (expf(x[r][t] - lse[r]) - (c == y[r] ? 1.f : 0.f));
                    dS[v * ldds + c] = d * inv;
                    if (dS_act) st_act(dS_act + v * ld_act + c, d);
                }
            }
            if (dS_act)
                for (int c = C + lane; c < ld_act; c += 32) st_act(dS_act + v * ld_act + c, 0.f);
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1)
#pragma unroll
            for (int r = 0; r < R; ++r) xy[r] += __shfl_xor_sync(0xffffffffu, xy[r], o);   // one lane holds y
#pragma unroll
        for (int r = 0; r < R; ++r)
            if (v0 + r < nd) wl += (double)scale * (double)(lse[r] - xy[r]);
    }
    if (lane == 0) s_w[warp_id()] = wl;
    __syncthreads();
    if (threadIdx.x == 0) {
        double b = 0.0;
        for (int i = 0; i < (int)(blockDim.x >> 5); ++i) b += s_w[i];
        partials[blockIdx.x] = b;
        fence_gpu();
        s_last = (atomicAdd(&ctr[0], 1u) == gridDim.x - 1);
    }
    __syncthreads();
    if (s_last) {                       // fixed-order reduction of the partials by the last CTA
        fence_gpu();
        double t = 0.0;
        for (unsigned i = threadIdx.x; i < gridDim.x; i += blockDim.x) t += ((volatile double*)partials)[i];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
        __syncthreads();
        if (lane == 0) s_w[warp_id()] = t;
        __syncthreads();
        if (threadIdx.x == 0) {
            double tot = 0.0;
            for (int i = 0; i < (int)(blockDim.x >> 5); ++i) tot += s_w[i];
            loss_accum[0] += (float)tot;
            ctr[0] = 0;
        }
    }
}

// C <= 64 (every C1-C5 output layer): half a warp per row, 4 consecutive classes per lane as one
// 16-byte vector, LOSS_V_R rows per half-warp per step -- a quarter of the instructions per row of
// k_loss (issue-bound there: ~290 warp-instructions per 47-class row, ncu r02r).  Same arithmetic
// and reduction structure per row (max, sum of exp, lse), dS / dS_act padding columns written as 0;
// exp / log through the SFU approximations (ex2 / lg2: ~2^-22 relative for the non-positive
// arguments here, far inside the 1e-5 gradient budget of reading #18).
constexpr int LOSS_V_R = 2;
__device__ __forceinline__ float hmax16(float v) {
#pragma unroll
    for (int o = 8; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}
__device__ __forceinline__ float hsum16(float v) {
#pragma unroll
    for (int o = 8; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}
__device__ __forceinline__ void st_act4z(float* p, const float* v) { st_act4(p, v); }
__device__ __forceinline__ void st_act4z(__nv_bfloat16* p, const float* v) { st_act4(p, v); }

template <typename TA>
__global__ void __launch_bounds__(256) k_loss_v(const float* __restrict__ logits, int64_t ldl,
                                                const int32_t* __restrict__ labels, const int32_t* __restrict__ gid,
                                                const int64_t* cnt, int C, float scale, float* __restrict__ dS,
                                                int64_t ldds, TA* __restrict__ dS_act, int64_t ld_act,
                                                const int64_t* __restrict__ indptr, double* partials, unsigned* ctr,
                                                float* loss_accum) {
    constexpr int R = LOSS_V_R;
    __shared__ double s_w[8];
    __shared__ int s_last;
    const int64_t nd = cnt[0];
    const int lane = lane_id(), hl = lane & 15, hw = lane >> 4;
    const int c0 = 4 * hl;
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    double wl = 0.0;
    for (int64_t v0 = gw * 2 * R; v0 < nd; v0 += nw * 2 * R) {
        int32_t gi[R], y[R];
        int64_t dg[R];
        float x[R][4];
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const int64_t v = v0 + 2 * r + hw;
            const bool ok = v < nd;
            gi[r] = ok ? gid[v] : 0;
            dg[r] = (ok && indptr) ? indptr[v + 1] - indptr[v] : 1;
            float4 t = make_float4(-INFINITY, -INFINITY, -INFINITY, -INFINITY);
            if (ok && c0 < C) t = *(const float4*)(logits + v * ldl + c0);
            x[r][0] = t.x; x[r][1] = c0 + 1 < C ? t.y : -INFINITY;
            x[r][2] = c0 + 2 < C ? t.z : -INFINITY; x[r][3] = c0 + 3 < C ? t.w : -INFINITY;
        }
#pragma unroll
        for (int r = 0; r < R; ++r) y[r] = v0 + 2 * r + hw < nd ? labels[gi[r]] : -1;
        float mx[R], se[R], lse[R], xy[R];
#pragma unroll
        for (int r = 0; r < R; ++r) mx[r] = hmax16(fmaxf(fmaxf(x[r][0], x[r][1]), fmaxf(x[r][2], x[r][3])));
#pragma unroll
        for (int r = 0; r < R; ++r) {
            float e = 0.f;
#pragma unroll
            for (int k = 0; k < 4; ++k)
                if (c0 + k < C) e += __expf(x[r][k] - mx[r]);
            se[r] = hsum16(e);
        }
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const int64_t v = v0 + 2 * r + hw;
            lse[r] = mx[r] + __logf(se[r]);
            xy[r] = 0.f;
            if (v < nd) {
                const float inv = indptr ? (dg[r] > 0 ? 1.f / (float)dg[r] : 0.f) : 1.f;
                float d[4];
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const int c = c0 + k;
                    if (c == y[r]) xy[r] = x[r][k];
                    d[k] = c < C ? scale * (__expf(x[r][k] - lse[r]) - (c == y[r] ? 1.f : 0.f)) : 0.f;
                }
                if (c0 < ldds)
                    *(float4*)(dS + v * ldds + c0) = make_float4(d[0] * inv, d[1] * inv, d[2] * inv, d[3] * inv);
                if (dS_act) {
                    const float z[4] = {0.f, 0.f, 0.f, 0.f};
                    for (int cc = c0; cc < ld_act; cc += 64) st_act4z(dS_act + v * ld_act + cc, cc == c0 ? d : z);
                }
            }
            xy[r] = hsum16(xy[r]);                      // one lane of the half holds y
        }
        if (hl == 0)
#pragma unroll
            for (int r = 0; r < R; ++r)
                if (v0 + 2 * r + hw < nd) wl += (double)scale * (double)(lse[r] - xy[r]);
    }
    wl += __shfl_xor_sync(0xffffffffu, wl, 16);         // the two halves' row sums (lane 0 keeps them)
    if (lane == 0) s_w[warp_id()] = wl;
    __syncthreads();
    if (threadIdx.x == 0) {
        double b = 0.0;
        for (int i = 0; i < (int)(blockDim.x >> 5); ++i) b += s_w[i];
        partials[blockIdx.x] = b;
        fence_gpu();
        s_last = (atomicAdd(&ctr[0], 1u) == gridDim.x - 1);
    }
    __syncthreads();
    if (s_last) {                       // fixed-order reduction of the partials by the last CTA
        fence_gpu();
        double t = 0.0;
        for (unsigned i = threadIdx.x; i < gridDim.x; i += blockDim.x) t += ((volatile double*)partials)[i];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
        __syncthreads();
        if (lane == 0) s_w[warp_id()] = t;
        __syncthreads();
        if (threadIdx.x == 0) {
            double tot = 0.0;
            for (int i = 0; i < (int)(blockDim.x >> 5); ++i) tot += s_w[i];
            loss_accum[0] += (float)tot;
            ctr[0] = 0;
        }
    }
}

void loss_ce(betty_ctx* c, const float* logits, int64_t ldl, const int32_t* labels, const int32_t* gid,
             const int64_t* cnt, int64_t rows_cap, int C, float scale, float* dS, int64_t ldds, void* dS_act,
             bool act_bf16, int64_t ld_act, const int64_t* prescale_indptr, float* loss_accum, cudaStream_t s) {
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((rows_cap * 8 + 255) / 256,
                                                                 std::min(2048, c->num_sms * 8)));
    double* partials = (double*)(c->L().counters + 64);   // 2048 doubles after the counters
    static const bool no_vec = getenv("BETTY_LOSS_VEC") && atoi(getenv("BETTY_LOSS_VEC")) == 0;   // A/B switch
    if (!no_vec && C <= 64 && ldl % 4 == 0 && ldds % 4 == 0 && ld_act % 4 == 0 && ((uintptr_t)logits & 15) == 0 &&
        ((uintptr_t)dS & 15) == 0 && ((uintptr_t)dS_act & 15) == 0) {
        const int gv = (int)std::max<int64_t>(1, std::min<int64_t>((rows_cap * 32 / (2 * LOSS_V_R) + 255) / 256,
                                                                   std::min(2048, c->num_sms * 8)));
        if (act_bf16)
            k_loss_v<__nv_bfloat16><<<gv, 256, 0, s>>>(logits, ldl, labels, gid, cnt, C, scale, dS, ldds,
                                                      (__nv_bfloat16*)dS_act, ld_act, prescale_indptr, partials,
                                                      c->L().counters + CTR_LOSS, loss_accum);
        else
            k_loss_v<float><<<gv, 256, 0, s>>>(logits, ldl, labels, gid, cnt, C, scale, dS, ldds, (float*)dS_act,
                                              ld_act, prescale_indptr, partials, c->L().counters + CTR_LOSS,
                                              loss_accum);
        return;
    }
    const int T = (C + 31) / 32;               // instantiated for 1, 2, 4 and 8 column groups per lane
#define LOSS_L(TT) do {                                                                                        \
        if (act_bf16)                                                                                          \
            k_loss<__nv_bfloat16, TT><<<grid, 256, 0, s>>>(logits, ldl, labels, gid, cnt, C, scale, dS, ldds,     \
                                                         (__nv_bfloat16*)dS_act, ld_act, prescale_indptr, partials, \
                                                         c->L().counters + CTR_LOSS, loss_accum);              \
        else                                                                                                   \
            k_loss<float, TT><<<grid, 256, 0, s>>>(logits, ldl, labels, gid, cnt, C, scale, dS, ldds,             \
                                                 (float*)dS_act, ld_act, prescale_indptr, partials,            \
                                                 c->L().counters + CTR_LOSS, loss_accum);                      \
    } while (0)
    if (T <= 1) LOSS_L(1); else if (T <= 2) LOSS_L(2); else if (T <= 4) LOSS_L(4); else LOSS_L(LOSS_MAXT_CAP);
#undef LOSS_L
}

// ------------------------------------------------------------------ adam
__global__ void k_adam(float* __restrict__ p, float* __restrict__ g, float* __restrict__ m, float* __restrict__ v,
                       int64_t n, float lr, float b1, float b2, float eps, float bc1, float bc2, int zero_grad) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const float gi = g[i];
        const float mi = b1 * m[i] + (1.f - b1) * gi;
        const float vi = b2 * v[i] + (1.f - b2) * gi * gi;
        m[i] = mi;
        v[i] = vi;
        const float mh = mi / bc1;
        const float vh = vi / bc2;
        p[i] -= lr * mh / (sqrtf(vh) + eps);
        if (zero_grad) g[i] = 0.f;
    }
}

void adam(betty_ctx* c, float* p, float* g, float* m, float* v, int64_t n, int t, float lr, float b1, float b2,
          float eps, bool zero_grad, cudaStream_t s) {
    const float bc1 = 1.f - powf(b1, (float)t), bc2 = 1.f - powf(b2, (float)t);
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((n + 255) / 256, (int64_t)c->num_sms * 4));
    k_adam<<<grid, 256, 0, s>>>(p, g, m, v, n, lr, b1, b2, eps, bc1, bc2, zero_grad ? 1 : 0);
}

// ----------------------------------------------------------- weight prep
constexpr int PREP_MAX_L = 16;
struct PrepArgs { PrepLayer l[PREP_MAX_L]; int L; };

// nearest tf32 (10 mantissa bits) of an fp32 value, as an fp32 word (the 3xTF32 split, gemm_tc.cu)
__device__ __forceinline__ float tf32_rn(float x) {
    return __uint_as_float((__float_as_uint(x) + 0x1000u) & 0xFFFFE000u);
}

template <typename T>
__global__ void k_prep(const float* __restrict__ params, PrepArgs a) {
    for (int li = 0; li < a.L; ++li) {
        const PrepLayer& P = a.l[li];
        // main matrix
        int64_t rows = (P.kind == 1) ? (P.Fi + 1) : (2 * P.Fp + 1);
        int64_t n = rows * P.ldb;
        T* B = (T*)P.B;
        for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
            const int i = (int)(t / P.ldb), j = (int)(t % P.ldb);
            float v = 0.f;
            if (P.kind == 1) {
                if (i < P.Fi) {
                    if (j < P.Fo) v = params[P.off_wn + (int64_t)i * P.Fo + j];
                    else if (j >= P.Fop && j < P.Fop + P.Fo) v = params[P.off_ws + (int64_t)i * P.Fo + (j - P.Fop)];
                } else if (j >= P.Fop && j < P.Fop + P.Fo) {
                    v = params[P.off_b + (j - P.Fop)];
                }
            } else if (j < P.Fo) {
                if (i < P.Fi) v = params[P.off_ws + (int64_t)i * P.Fo + j];
                else if (i >= P.Fp && i < P.Fp + P.Fi) v = params[P.off_wn + (int64_t)(i - P.Fp) * P.Fo + j];
                else if (i == 2 * P.Fp) v = params[P.off_b + j];
            }
            st_act(B + t, v);
            // FP32 mode on the tensor cores (3xTF32): hi = v rounded to the nearest tf32, lo = tf32(v - hi)
            const float hi = tf32_rn(v), lo = tf32_rn(v - hi);
            if (P.Bhi) { ((float*)P.Bhi)[t] = hi; ((float*)P.Blo)[t] = lo; }
            if (P.Bt && j < P.ldbt_rows) {                                               // K-major copy
                if (P.Btlo) {
                    ((float*)P.Bt)[(int64_t)j * P.ldbt + i] = hi;
                    ((float*)P.Btlo)[(int64_t)j * P.ldbt + i] = lo;
                } else {
                    st_act((T*)P.Bt + (int64_t)j * P.ldbt + i, v);
                }
            }
        }
        if (P.kind == 2) {
            T* Bp = (T*)P.Bp;
            const int64_t np = (int64_t)(P.Fi + 1) * P.ldbp;
            for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < np; t += (int64_t)gridDim.x * blockDim.x) {
                const int i = (int)(t / P.ldbp), j = (int)(t % P.ldbp);
                float v = 0.f;
                if (j < P.Fi) v = (i < P.Fi) ? params[P.off_wp + (int64_t)i * P.Fi + j] : params[P.off_bp + j];
                st_act(Bp + t, v);
                const float hi = tf32_rn(v), lo = tf32_rn(v - hi);
                if (P.Bphi) { ((float*)P.Bphi)[t] = hi; ((float*)P.Bplo)[t] = lo; }
                if (P.Bpt && j < P.Fi) {
                    if (P.Bptlo) {
                        ((float*)P.Bpt)[(int64_t)j * P.ldbpt + i] = hi;
                        ((float*)P.Bptlo)[(int64_t)j * P.ldbpt + i] = lo;
                    } else {
                        st_act((T*)P.Bpt + (int64_t)j * P.ldbpt + i, v);
                    }
                }
            }
        }
    }
}

__global__ void k_split_tf32(const float* __restrict__ x, float* hi, float* lo, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const float v = x[i];
        const float h = tf32_rn(v);
        hi[i] = h;
        lo[i] = tf32_rn(v - h);
    }
}

void split_tf32_dev(const float* x, float* hi, float* lo, int64_t n, cudaStream_t s) {
    k_split_tf32<<<(int)std::min<int64_t>(1024, (n + 255) / 256 + 1), 256, 0, s>>>(x, hi, lo, n);
}

void prep_weights(betty_ctx* c, const float* params, const PrepLayer* layers, int L, bool bf16, cudaStream_t s) {
    PrepArgs a;
    a.L = L;
    for (int i = 0; i < L && i < PREP_MAX_L; ++i) a.l[i] = layers[i];
    if (bf16) k_prep<__nv_bfloat16><<<c->num_sms * 2, 256, 0, s>>>(params, a);
    else k_prep<float><<<c->num_sms * 2, 256, 0, s>>>(params, a);
}

}  // namespace betty
