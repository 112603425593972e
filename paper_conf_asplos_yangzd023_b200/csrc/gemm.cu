// gemm.cu -- dense SAGE linear layers on the CUDA cores (FP32 FFMA; no
// TF32 anywhere, reading #17), operands fp32 or bf16, fp32 accumulation.
//   gemm_row: C = A B with fused epilogues (ReLU + bias "ones" column, ReLU'
//             mask, residual + mask) -- forward layers and dX
//   gemm_red: P = A^T B reduced over the node dimension (dW), split over row
//             chunks with a fixed chunk -> split assignment, then a
//             deterministic ordered reduction that ADDS into the flat gradient
//             (fused accumulation across micro-batches, a6) with the GEMM ->
//             parameter layout mapping.
// The tcgen05 tensor-core path (gemm_tc.cu: bf16, and fp32 as 3xTF32) takes
// every shape it supports in both modes; these kernels remain for the shapes
// it rejects (and k_red_final serves both paths).
#include <algorithm>
#include "common.cuh"
#include "internal.h"
#include "sage.h"

namespace betty {

constexpr int RBM = 64, RBN = 64, RBK = 16;

template <typename TA, typename TB, typename TC, typename TM>
__global__ void __launch_bounds__(256) k_gemm_row(GemmRow g) {
    __shared__ float As[RBK][RBM + 4];
    __shared__ float Bs[RBK][RBN + 4];
    const TA* __restrict__ A = (const TA*)g.A;
    const TB* __restrict__ B = (const TB*)g.B;
    TC* __restrict__ C = (TC*)g.C;
    const int64_t M = *g.M_dev;
    const int K = g.K, N = g.N;
    const int nN = (N + RBN - 1) / RBN;
    const int64_t tiles = ((M + RBM - 1) / RBM) * nN;
    const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
    for (int64_t tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
        const int64_t m0 = (tile / nN) * RBM;
        const int n0 = (int)(tile % nN) * RBN;
        float acc[4][4];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j) acc[i][j] = 0.f;
        for (int k0 = 0; k0 < K; k0 += RBK) {
            {
                const int r = threadIdx.x >> 2, kk = (threadIdx.x & 3) * 4;
                const int64_t m = m0 + r;
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int k = k0 + kk + q;
                    As[kk + q][r] = (m < M && k < K) ? ld_act(A + m * g.lda + k) : 0.f;
                }
            }
            if (!g.transB) {
                const int kk = threadIdx.x >> 4, nn = (threadIdx.x & 15) * 4;
                const int k = k0 + kk;
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int n = n0 + nn + q;
                    Bs[kk][nn + q] = (k < K && n < N) ? ld_act(B + (int64_t)k * g.ldb + n) : 0.f;
                }
            } else {
                const int nn = threadIdx.x >> 2, kk = (threadIdx.x & 3) * 4;
                const int n = n0 + nn;
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int k = k0 + kk + q;
                    Bs[kk + q][nn] = (k < K && n < N) ? ld_act(B + (int64_t)n * g.ldb + k) : 0.f;
                }
            }
            __syncthreads();
#pragma unroll
            for (int kk = 0; kk < RBK; ++kk) {
                float a[4], b[4];
#pragma unroll
                for (int i = 0; i < 4; ++i) a[i] = As[kk][ty * 4 + i];
#pragma unroll
                for (int j = 0; j < 4; ++j) b[j] = Bs[kk][tx * 4 + j];
#pragma unroll
                for (int i = 0; i < 4; ++i)
#pragma unroll
                    for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
            }
            __syncthreads();
        }
        const int64_t nres = (g.epi == EPI_RES_MASK) ? *g.nres_dev : 0;
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            const int64_t m = m0 + ty * 4 + i;
            if (m >= M) continue;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const int n = n0 + tx * 4 + j;
                if (n >= N) continue;
                float v = acc[i][j];
                if (g.epi == EPI_RELU_ONES) v = fmaxf(v, 0.f);
                if (g.epi == EPI_RES_MASK && m < nres) v += g.res[m * g.ldr + n];
                if (g.epi == EPI_MASK || g.epi == EPI_RES_MASK)
                    if (!(ld_act((const TM*)g.mask + m * g.ldm + n) > 0.f)) v = 0.f;
                st_act(C + m * g.ldc + n, v);
            }
        }
        // trailing columns [N, ldc) of the rows of this tile: the ones column after a ReLU layer
        // (the next layer's bias input), zero elsewhere
        if (n0 == 0 && g.ldc > N) {
            const int w = (int)(g.ldc - N);
            for (int t = threadIdx.x; t < RBM * w; t += blockDim.x) {
                const int64_t m = m0 + t / w;
                const int col = N + t % w;
                if (m < M) st_act(C + m * g.ldc + col, (g.epi == EPI_RELU_ONES && col == N) ? 1.f : 0.f);
            }
        }
    }
}

template <typename TA, typename TB>
static void launch_row(betty_ctx* c, const GemmRow& g, cudaStream_t s) {
    const int64_t tiles = ((g.M_cap + RBM - 1) / RBM) * ((g.N + RBN - 1) / RBN);
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(tiles, (int64_t)c->num_sms * 6));
    if (g.c_bf16) {
        if (g.m_bf16) k_gemm_row<TA, TB, __nv_bfloat16, __nv_bfloat16><<<grid, 256, 0, s>>>(g);
        else k_gemm_row<TA, TB, __nv_bfloat16, float><<<grid, 256, 0, s>>>(g);
    } else {
        if (g.m_bf16) k_gemm_row<TA, TB, float, __nv_bfloat16><<<grid, 256, 0, s>>>(g);
        else k_gemm_row<TA, TB, float, float><<<grid, 256, 0, s>>>(g);
    }
}

bool gemm_row(betty_ctx* c, const GemmRow& g, cudaStream_t s) {
    // tensor cores: bf16 operands, or FP32 mode as 3xTF32 when the weights come split (hi / lo)
    const bool tf = !g.a_bf16 && !g.b_bf16 && !g.c_bf16 && (g.transB ? (g.Bhi && g.Blo) : (g.Bt && g.Btlo));
    if (c->use_tc && ((g.a_bf16 && g.b_bf16) || tf)) {
        const void* Bk = tf ? (g.transB ? g.Bhi : g.Bt) : (g.transB ? g.B : g.Bt);
        const void* Bl = tf ? (g.transB ? g.Blo : g.Btlo) : nullptr;
        const int64_t ldbk = g.transB ? g.ldb : g.ldbt;
        const size_t bs = tf ? 4 : 2;
        if (Bk && g.N <= 256 && gemm_row_tc(c, g, Bk, Bl, ldbk, s)) return g.epi == EPI_RELU_ONES && g.obits;
        // wider plain products (the pool layers' dXA, N = 2 Fp): 256-column blocks, left to right (each
        // block writes only its own columns; the last one the trailing columns)
        if (Bk && g.N > 256 && g.epi == EPI_STORE && (ldbk & 7) == 0) {
            const size_t cs = g.c_bf16 ? 2 : 4;
            bool ok = true;
            for (int n0 = 0; n0 < g.N && ok; n0 += 256) {
                GemmRow h = g;
                h.N = std::min(256, g.N - n0);
                h.C = (char*)g.C + (size_t)n0 * cs;
                h.cend = n0 + 256 >= g.N ? g.ldc - n0 : h.N;
                ok = gemm_row_tc(c, h, (const char*)Bk + (size_t)n0 * ldbk * bs,
                                 Bl ? (const char*)Bl + (size_t)n0 * ldbk * bs : nullptr, ldbk, s);
            }
            if (ok) return false;
        }
    }
    if (g.a_bf16) {
        if (g.b_bf16) launch_row<__nv_bfloat16, __nv_bfloat16>(c, g, s);
        else launch_row<__nv_bfloat16, float>(c, g, s);
    } else {
        if (g.b_bf16) launch_row<float, __nv_bfloat16>(c, g, s);
        else launch_row<float, float>(c, g, s);
    }
    return false;
}

// ----------------------------------------------------------- reduction GEMM
constexpr int XB = 64, XR = 16, XCHUNK = 256;

template <typename TA, typename TB>
__global__ void __launch_bounds__(256) k_gemm_red(GemmRed g) {
    __shared__ float As[XR][XB + 4];
    __shared__ float Bs[XR][XB + 4];
    const TA* __restrict__ A = (const TA*)g.A;
    const TB* __restrict__ B = (const TB*)g.B;
    const int64_t M = *g.M_dev;
    const int tI = (g.K1 + XB - 1) / XB, tJ = (g.N + XB - 1) / XB;
    const int tiles = tI * tJ;
    const int tile = blockIdx.x % tiles, split = blockIdx.x / tiles;
    const int i0 = (tile / tJ) * XB, j0 = (tile % tJ) * XB;
    const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
    float tot[4][4];
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) tot[i][j] = 0.f;
    const int64_t nchunks = (M + XCHUNK - 1) / XCHUNK;
    for (int64_t ch = split; ch < nchunks; ch += g.S) {
        float acc[4][4];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j) acc[i][j] = 0.f;
        const int64_t rend = mn64(M, (ch + 1) * XCHUNK);
        for (int64_t r0 = ch * XCHUNK; r0 < rend; r0 += XR) {
            const int rr = threadIdx.x >> 4, cc = (threadIdx.x & 15) * 4;
            const int64_t r = r0 + rr;
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const int i = i0 + cc + q, j = j0 + cc + q;
                As[rr][cc + q] = (r < rend && i < g.K1) ? ld_act(A + r * g.lda + i) : 0.f;
                Bs[rr][cc + q] = (r < rend && j < g.N) ? ld_act(B + r * g.ldb + j) : 0.f;
            }
            __syncthreads();
#pragma unroll
            for (int k = 0; k < XR; ++k) {
                float a[4], b[4];
#pragma unroll
                for (int i = 0; i < 4; ++i) a[i] = As[k][ty * 4 + i];
#pragma unroll
                for (int j = 0; j < 4; ++j) b[j] = Bs[k][tx * 4 + j];
#pragma unroll
                for (int i = 0; i < 4; ++i)
#pragma unroll
                    for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
            }
            __syncthreads();
        }
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j) tot[i][j] += acc[i][j];
    }
    float* P = g.partials + (int64_t)split * g.K1 * g.N;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        const int ii = i0 + ty * 4 + i;
        if (ii >= g.K1) continue;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const int jj = j0 + tx * 4 + j;
            if (jj < g.N) P[(int64_t)ii * g.N + jj] = tot[i][j];
        }
    }
}

// GEMM layout (i, j) -> flat parameter index, or -1 (padding / unused)
__device__ __forceinline__ int64_t map_index(const GradMap& m, int i, int j) {
    if (m.mode == MAP_AGG) {            // rows [0,Fi) W_self, [Fp,Fp+Fi) W_neigh, 2Fp bias; cols < Fo
        if (j >= m.Fo) return -1;
        if (i < m.Fi) return m.off_ws + (int64_t)i * m.Fo + j;
        if (i >= m.Fp && i < m.Fp + m.Fi) return m.off_wn + (int64_t)(i - m.Fp) * m.Fo + j;
        if (i == 2 * m.Fp) return m.off_b + j;
        return -1;
    } else if (m.mode == MAP_PF_N) {    // neighbour half alone: cols [0,Fo) W_neigh (bias row: none)
        if (j >= m.Fo || i >= m.Fi) return -1;
        return m.off_wn + (int64_t)i * m.Fo + j;
    } else if (m.mode == MAP_PF_S) {    // self half alone: cols [0,Fo) W_self; row Fi = bias
        if (j >= m.Fo) return -1;
        if (i < m.Fi) return m.off_ws + (int64_t)i * m.Fo + j;
        if (i == m.Fi) return m.off_b + j;
        return -1;
    } else if (m.mode == MAP_PF) {      // cols [0,Fo) W_neigh, [Fop,Fop+Fo) W_self; row Fi = bias (self half)
        const bool self = j >= m.Fop && j < m.Fop + m.Fo;
        const bool nb = j < m.Fo;
        if (i < m.Fi) {
            if (nb) return m.off_wn + (int64_t)i * m.Fo + j;
            if (self) return m.off_ws + (int64_t)i * m.Fo + (j - m.Fop);
            return -1;
        }
        if (i == m.Fi && self) return m.off_b + (j - m.Fop);
        return -1;
    } else {                            // pool: rows [0,Fi) W_pool, row Fi b_pool; cols < Fi
        if (j >= m.Fi) return -1;
        if (i < m.Fi) return m.off_wp + (int64_t)i * m.Fi + j;
        if (i == m.Fi) return m.off_bp + j;
        return -1;
    }
}

// grad[map(t)] += sum_s partials[s][t], t < K1*N: a CTA takes 32 consecutive outputs, its 8 warps
// sum the splits s = w, w+8, ... (coalesced 128-byte rows of partials), then the 8 warp sums are
// added in a fixed order -- deterministic, and 8x the parallelism of one thread per output
__global__ void __launch_bounds__(256) k_red_final(const float* __restrict__ partials, int S, int K1, int N,
                                                   float* grad, GradMap map) {
    __shared__ float s_part[8][33];
    const int64_t n = (int64_t)K1 * N;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (int64_t t0 = (int64_t)blockIdx.x * 32; t0 < n; t0 += (int64_t)gridDim.x * 32) {
        const int64_t t = t0 + lane;
        float sum = 0.f;
        if (t < n) {
            // 4 independent chains of loads in flight (a single chain waited one memory latency per
            // split: ~19 us per launch at 148 splits); fixed order for a given S -> deterministic
            float s0 = 0.f, s1 = 0.f, s2 = 0.f, s3 = 0.f;
            int sp = w;
            for (; sp + 24 < S; sp += 32) {
                s0 += partials[(int64_t)sp * n + t];
                s1 += partials[(int64_t)(sp + 8) * n + t];
                s2 += partials[(int64_t)(sp + 16) * n + t];
                s3 += partials[(int64_t)(sp + 24) * n + t];
            }
            for (; sp < S; sp += 8) s0 += partials[(int64_t)sp * n + t];
            sum = (s0 + s1) + (s2 + s3);
        }
        s_part[w][lane] = sum;
        __syncthreads();
        if (w == 0 && t < n) {
            float tot = 0.f;
#pragma unroll
            for (int q = 0; q < 8; ++q) tot += s_part[q][lane];
            const int i = (int)(t / N), j = (int)(t % N);
            const int64_t dst = map_index(map, i, j);
            if (dst >= 0) grad[dst] += tot;
        }
        __syncthreads();
    }
}

int gemm_red_splits(int64_t M_cap, int K1, int N) {
    // the same split count serves the SIMT path (tiles of 64 x 64) and the tensor-core path
    // (M tiles of 128 features, one CTA per SM): enough CTAs for either, never more than row chunks
    const int tiles = ((K1 + XB - 1) / XB) * ((N + XB - 1) / XB);
    const int mtiles = (K1 + 127) / 128;
    const int64_t chunks = std::max<int64_t>(1, (M_cap + XCHUNK - 1) / XCHUNK);
    (void)mtiles;
    const int want = std::max(148, (148 * 4) / tiles);
    return (int)std::max<int64_t>(1, std::min<int64_t>(chunks, want));
}

void gemm_red(betty_ctx* c, const GemmRed& g, cudaStream_t s) {
    // tensor cores: bf16 operands, or fp32 operands as 3xTF32 (FP32 mode, unless BETTY_FP32_SIMT=1)
    const bool tf = !g.a_bf16 && !g.b_bf16 && c->fp32_tc;
    int S_used = g.S;
    if (c->use_tc && ((g.a_bf16 && g.b_bf16) || tf) && gemm_red_tc(c, g, &S_used, s)) {
        const int64_t n = (int64_t)g.K1 * g.N;
        const int gf = (int)std::max<int64_t>(1, std::min<int64_t>((n + 31) / 32, (int64_t)c->num_sms * 8));
        k_red_final<<<gf, 256, 0, s>>>(g.partials, S_used, g.K1, g.N, g.grad, g.map);
        return;
    }
    const int tiles = ((g.K1 + XB - 1) / XB) * ((g.N + XB - 1) / XB);
    const int grid = tiles * g.S;
    if (g.a_bf16) {
        if (g.b_bf16) k_gemm_red<__nv_bfloat16, __nv_bfloat16><<<grid, 256, 0, s>>>(g);
        else k_gemm_red<__nv_bfloat16, float><<<grid, 256, 0, s>>>(g);
    } else {
        if (g.b_bf16) k_gemm_red<float, __nv_bfloat16><<<grid, 256, 0, s>>>(g);
        else k_gemm_red<float, float><<<grid, 256, 0, s>>>(g);
    }
    const int64_t n = (int64_t)g.K1 * g.N;
    const int gf = (int)std::max<int64_t>(1, std::min<int64_t>((n + 31) / 32, (int64_t)c->num_sms * 8));
    k_red_final<<<gf, 256, 0, s>>>(g.partials, g.S, g.K1, g.N, g.grad, g.map);
}

}  // namespace betty
