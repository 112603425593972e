// sage.h -- internal launchers of the SAGE forward/backward kernels.
#pragma once
#include <stdint.h>
#include <cuda.h>
#include <cuda_runtime.h>

struct betty_ctx;
namespace betty {

// ---- agg.cu
// A feature table sharded by rows (BASELINE configs[4]): row g lives in base[g / rps]
// at local row g % rps (row stride ld of the table); R == 0: one contiguous table (X, ldx).  The bases
// may be peer-mapped memory of other GPUs (CUDA IPC): the gathers then cross NVLink.
constexpr int MAX_SHARDS = 64;
struct FeatShards {
    int R = 0;
    int64_t rps = 0;
    const void* base[MAX_SHARDS] = {};
};
// XA[v] = [X[srow v] | mean_e X[row(e)] | 1], row(e) = emap ? emap[erow[e]] : erow[e]
// otab: optional micro-batch-major row order (extract.h), null = ascending rows
void agg_mean_xa(betty_ctx* c, const void* X, bool x_bf16, int64_t ldx, const int32_t* srow, const int32_t* erow,
                 const int32_t* emap, const int64_t* indptr, const int64_t* cnt, const int64_t* otab, int64_t rows_cap,
                 int64_t src_per_mb, int Fi, int Fp, void* XA, bool xa_bf16, int64_t ldxa, bool sum,
                 const FeatShards* shards, cudaStream_t s);
// S[v] = Ys[v] + (1/D_v) sum_u Y[u]  (Y: neighbour half over src rows, Ys: self half over dst rows, same ld)
// sum: the sum aggregator (no 1/D_v); likewise agg_mean_xa's sum and a null indptr of the CSC kernels
void agg_mean_pf(betty_ctx* c, const float* Y, const float* Ys, int64_t ldy, const int64_t* indptr, const int32_t* idx,
                 const int64_t* cnt, int64_t rows_cap, int Fo, int Fop, bool relu, void* out, bool out_bf16,
                 int64_t ldo, bool sum, cudaStream_t s);
void gather_ones(betty_ctx* c, const void* X, bool x_bf16, int64_t ldx, const int32_t* xrow, const int64_t* cnt_rows,
                 int64_t rows_cap, int Fi, void* out, bool out_bf16, int64_t ldo, cudaStream_t s);
void csc_mean(betty_ctx* c, const float* dXA, int64_t ldd, const int64_t* indptr, const int64_t* t_indptr,
              const int32_t* t_idx, const int64_t* cnt, int64_t src_cap, int Fi, int Fp, const void* H, bool h_bf16,
              int64_t ldh, const uint32_t* hbits, int64_t ldhb, void* out, bool out_bf16, int64_t ldo,
              cudaStream_t s);   // hbits (optional): [H > 0] as bits, ldhb words per row
// G = P^T D+ dS via the CSC; indptr == null: dS is already scaled by 1/D_v (the loss kernel does it)
void csc_pf(betty_ctx* c, const void* dS, bool ds_bf16, int64_t ldds, const int64_t* indptr, const int64_t* t_indptr,
            const int32_t* t_idx, const int64_t* cnt, int64_t src_cap, int Fo, int Fop, void* G, bool g_bf16,
            int64_t ldg, cudaStream_t s);
// pool: XA = [x_v | max_u ReLU(Zp[u]) | 1]; argmax per (v, column) as the source id (int32) or, with
// pos8, the byte position of the winning edge in v's row (rows of <= 254 edges)
void agg_pool(betty_ctx* c, const void* X, bool x_bf16, int64_t ldx, const int32_t* xrow, const float* Zp, int64_t ldz,
              const int64_t* indptr, const int32_t* idx, const int64_t* cnt, int64_t rows_cap, int Fi, int Fp,
              void* XA, bool xa_bf16, int64_t ldxa, void* arg, int64_t ldarg, bool pos8, cudaStream_t s);
void route_pool(betty_ctx* c, const float* dXA, int64_t ldd, const void* arg, int64_t ldarg, bool pos8,
                const int64_t* indptr, const int32_t* idx, const int64_t* t_indptr, const int32_t* t_idx,
                const int64_t* cnt, int64_t src_cap, int Fi, int Fp, const float* Zp, int64_t ldz, void* out,
                bool out_bf16, int64_t ldo, cudaStream_t s);

// ---- gemm.cu (dense layers; SIMT fp32 FFMA path, operands fp32 or bf16)
enum { EPI_STORE = 0, EPI_RELU_ONES = 1, EPI_MASK = 2, EPI_RES_MASK = 3 };
struct GemmRow {                 // C[m, n] = sum_k A[m, k] B(k, n), m < *M_dev
    const void* A; int64_t lda; bool a_bf16;
    const void* B; int64_t ldb; bool b_bf16; bool transB;   // B(k,n) = transB ? B[n*ldb+k] : B[k*ldb+n]
    const int64_t* M_dev; int64_t M_cap; int K; int N;
    void* C; int64_t ldc; bool c_bf16;
    int epi;
    const void* mask; int64_t ldm; bool m_bf16;           // EPI_MASK / EPI_RES_MASK: C *= [mask > 0]
    const float* res; int64_t ldr; const int64_t* nres_dev; // EPI_RES_MASK: C += res (rows < *nres_dev)
    const void* Bt; int64_t ldbt;                          // K-major copy of B (N x K) for the tensor-core path
    // FP32 mode on the tensor cores (3xTF32): B split into hi (tf32-exact) + lo, in B's layout (transB
    // products) and K-major (Bt holds hi, Btlo lo); null: SIMT FFMA
    const void* Bhi = nullptr; const void* Blo = nullptr; const void* Btlo = nullptr;
    const uint32_t* mbits; int64_t ldmb;   // EPI_MASK / EPI_RES_MASK: mask as ReLU bits (tensor-core path), or null
    uint32_t* obits; int64_t ldob;         // EPI_RELU_ONES: also write the ReLU bits [C > 0] (tensor-core path)
    int64_t cend = 0;                      // tensor-core path: trailing columns [N, cend) written (0: ldc)
};
// returns true iff the ReLU bits g.obits were written (EPI_RELU_ONES on the tensor-core path)
bool gemm_row(betty_ctx* c, const GemmRow& g, cudaStream_t s);
// gemm_tc.cu: tcgen05 paths (false = shape not supported, caller falls back to SIMT)
bool tc_available();
bool make_gather_map(CUtensorMap* m, const void* base, bool f32, int64_t cols, int64_t rows, int64_t ld,
                     int box_cols);
bool gemm_row_tc(betty_ctx* c, const GemmRow& g, const void* Bk, const void* Bk_lo, int64_t ldbk, cudaStream_t s);

// P[i, j] = sum_{r < *M_dev} A[r, i] B[r, j], i < K1, j < N, split over S row groups into
// partials[S][K1][N]; then grad[map(i,j)] += sum_s partials[s][i][j] (fixed order: deterministic).
enum { MAP_AGG = 0, MAP_PF = 1, MAP_POOL = 2, MAP_PF_N = 3, MAP_PF_S = 4 };
struct GradMap {
    int mode;
    int Fi, Fo, Fp, Fop;
    int64_t off_ws, off_wn, off_b, off_wp, off_bp;
};
struct GemmRed {
    const void* A; int64_t lda; bool a_bf16;
    const void* B; int64_t ldb; bool b_bf16;
    const int64_t* M_dev; int64_t M_cap; int K1; int N;
    float* partials; int S;
    float* grad; GradMap map;
};
void gemm_red(betty_ctx* c, const GemmRed& g, cudaStream_t s);
int gemm_red_splits(int64_t M_cap, int K1, int N);
// S_used: the row splits (partials) the launch wrote (<= g.S)
bool gemm_red_tc(betty_ctx* c, const GemmRed& g, int* S_used, cudaStream_t s);

// ---- misc.cu
void loss_ce(betty_ctx* c, const float* logits, int64_t ldl, const int32_t* labels, const int32_t* gid,
             const int64_t* cnt, int64_t rows_cap, int C, float scale, float* dS, int64_t ldds, void* dS_act,
             bool act_bf16, int64_t ld_act, const int64_t* prescale_indptr, float* loss_accum, cudaStream_t s);
void adam(betty_ctx* c, float* p, float* g, float* m, float* v, int64_t n, int t, float lr, float b1, float b2,
          float eps, bool zero_grad, cudaStream_t s);
// per-layer GEMM weight layouts from the flat parameter vector
struct PrepLayer {
    int kind;                    // 0 agg-first [Ws;0;Wn;0;b] ((2Fp+1) x Fo, ld ldb), 1 project-first, 2 pool
    int Fi, Fo, Fp, Fop;
    int64_t off_ws, off_wn, off_b, off_wp, off_bp;
    void* B; int64_t ldb;        // main weight in GEMM layout
    void* Bp; int64_t ldbp;      // pool: [Wp; bp] ((Fi+1) x Fi)
    void* Bt; int64_t ldbt;      // K-major (transposed) copies for the tensor-core path (may be null)
    int64_t ldbt_rows;           // rows of Bt (= columns of B that are written)
    void* Bpt; int64_t ldbpt;
    // FP32 mode, 3xTF32 (null otherwise): Bt / Bpt then hold the hi parts
    void* Bhi; void* Blo; void* Btlo; void* Bphi; void* Bplo; void* Bptlo;
};
void prep_weights(betty_ctx* c, const float* params, const PrepLayer* layers, int L, bool bf16, cudaStream_t s);
// hi = x with the low 13 mantissa bits cleared, lo = x - hi (the 3xTF32 operand split), n elements
void split_tf32_dev(const float* x, float* hi, float* lo, int64_t n, cudaStream_t s);
// ---- extract.cu: egid[e] = src_gid[nbr[e]] over a full-batch layer's E edges
void full_egid(betty_ctx* c, const int32_t* nbr, const int32_t* src_gid, int64_t E, int32_t* egid, cudaStream_t s);

}  // namespace betty
