// misc.cu -- a4 softmax cross-entropy (fused forward + backward), a7 Adam,
// and the per-step weight layout preparation (fp32 params -> GEMM layouts,
// cast to bf16 in BF16 mode).
#include <cmath>
#include "common.cuh"
#include "internal.h"
#include "sage.h"

namespace betty {

// ------------------------------------------------------------------ loss
// loss_accum += scale * sum_v [logsumexp(S_v) - S_v[y_v]] ;  dS_v = scale * (softmax(S_v) - onehot(y_v))
// (reading #15: scale = 1 / n_out of the full batch).  One warp per row,
// C <= 256.  The loss is reduced deterministically: per-CTA partials in a
// fixed order, summed by the last CTA.
constexpr int LOSS_MAXT_CAP = 8;               // C <= 256

template <typename TA, int LOSS_MAXT>        // LOSS_MAXT = ceil(C / 32) column groups per lane
__global__ void __launch_bounds__(256) k_loss(const float* __restrict__ logits, int64_t ldl,
                                              const int32_t* __restrict__ labels, const int32_t* __restrict__ gid,
                                              const int64_t* cnt, int C, float scale, float* __restrict__ dS,
                                              int64_t ldds, TA* __restrict__ dS_act, int64_t ld_act,
                                              const int64_t* __restrict__ indptr, double* partials, unsigned* ctr,
                                              float* loss_accum) {
    __shared__ double s_w[8];
    __shared__ int s_last;
    const int64_t nd = cnt[0];
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    double wl = 0.0;
    // the next row's label, degree and logits are loaded while this row is reduced (a row's
    // arithmetic is a chain of shuffles; its loads would otherwise sit in front of it)
    int32_t ny = 0;
    int64_t ndg = 1;
    float nx[LOSS_MAXT];
    auto fetch = [&](int64_t vv) {
        if (vv < nd) {
            ny = labels[gid[vv]];
            if (indptr) ndg = indptr[vv + 1] - indptr[vv];
#pragma unroll
            for (int t = 0; t < LOSS_MAXT; ++t) {
                const int c = lane + 32 * t;
                nx[t] = c < C ? logits[vv * ldl + c] : -INFINITY;
            }
        }
    };
    fetch(gw);
    for (int64_t v = gw; v < nd; v += nw) {
        const int32_t y = ny;
        // indptr (project-first top layer): the fp32 dS is stored pre-scaled by 1/D_v for P^T D+ dS
        float inv = 1.f;
        if (indptr) inv = ndg > 0 ? 1.f / (float)ndg : 0.f;
        float x[LOSS_MAXT];
        float mx = -INFINITY;
#pragma unroll
        for (int t = 0; t < LOSS_MAXT; ++t) {
            x[t] = nx[t];
            mx = fmaxf(mx, x[t]);
        }
        fetch(v + nw);
        mx = warp_max(mx);
        float se = 0.f;
#pragma unroll
        for (int t = 0; t < LOSS_MAXT; ++t) {
            const int c = lane + 32 * t;
            if (c < C) se += expf(x[t] - mx);
        }
        se = warp_sum(se);
        const float lse = mx + logf(se);
        float xy = 0.f;
#pragma unroll
        for (int t = 0; t < LOSS_MAXT; ++t) {
            const int c = lane + 32 * t;
            if (c == y) xy = x[t];
            if (c < C) {
                const float d = scale * (expf(x[t] - lse) - (c == y ? 1.f : 0.f));
                dS[v * ldds + c] = d * inv;
                if (dS_act) st_act(dS_act + v * ld_act + c, d);
            }
        }
        xy = warp_sum(xy);   // exactly one lane holds y
        wl += (double)scale * (double)(lse - xy);
        if (dS_act)
            for (int c = C + lane; c < ld_act; c += 32) st_act(dS_act + v * ld_act + c, 0.f);
    }
    if (lane == 0) s_w[warp_id()] = wl;
    __syncthreads();
    if (threadIdx.x == 0) {
        double b = 0.0;
        for (int i = 0; i < (int)(blockDim.x >> 5); ++i) b += s_w[i];
        partials[blockIdx.x] = b;
        __threadfence();
        s_last = (atomicAdd(&ctr[0], 1u) == gridDim.x - 1);
    }
    __syncthreads();
    if (s_last) {                       // fixed-order reduction of the partials by the last CTA
        __threadfence();
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
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((rows_cap * 32 + 255) / 256,
                                                                 std::min(2048, c->num_sms * 8)));
    double* partials = (double*)(c->L().counters + 64);   // 2048 doubles after the counters
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
