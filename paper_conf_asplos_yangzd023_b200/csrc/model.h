// model.h -- host-side layer plan and buffer set of the SAGE path.
#pragma once
#include <stdint.h>
#include <vector>
#include <cuda_runtime.h>
#include "sage.h"

struct betty_ctx;
namespace betty {

enum { KIND_AGG = 0, KIND_PF = 1, KIND_POOL = 2 };

inline int64_t r8(int64_t x) { return (x + 7) / 8 * 8; }

struct LayerCfg {
    int kind;
    int Fi, Fo, Fp, Fop;
    bool last;
    int64_t off_wp, off_bp, off_ws, off_wn, off_b;
    int64_t ld_xa, ld_gat, ld_y, ld_g, ld_dxa, ld_zp, ld_dzp, ld_arg, ld_out, ld_ds, ld_B, ld_Bp;
};

struct ModelCfg {
    int L = 0;
    int aggr = 0;             // 0 mean, 1 pool, 2 sum (Table 1)
    bool sum = false;         // the sum aggregator: mean's kernels without 1/D_v
    bool bf16 = false;        // GEMM operands / hidden activations in bf16
    bool feat_bf16 = false;
    std::vector<int> dims;
    std::vector<LayerCfg> layers;
    int64_t n_params = 0;
    // pool layers: the argmax is stored as the byte position of the winning edge in its row (plans
    // whose pool blocks have rows of <= 254 edges), else as the source id (int32)
    std::vector<char> pos8;
    bool arg8(int l) const { return l < (int)pos8.size() && pos8[l]; }
    // does the backward of layer l need the CSC of block l?
    bool needs_csc(int l) const { return !(layers[l].kind == KIND_AGG && l == 0); }
    // layer l reads a gathered [X | 1] copy of the features (layer 0 of PF / POOL)
    bool needs_gat(int l) const { return l == 0 && layers[l].kind != KIND_AGG; }
};

bool make_model_cfg(int L, int aggr, int gemm, int feat_dtype, const int32_t* dims, ModelCfg* out);

struct BlockView {              // one layer of a (group-concatenated) micro-batch on the device
    const int64_t* indptr;
    const int32_t* indices;
    const int64_t* t_indptr;
    const int32_t* t_indices;
    const int32_t* src_gid;
    const int64_t* cnt;         // device [3]: n_dst, n_src, n_edges
    int64_t cap_dst, cap_src, cap_e;
    const int32_t* egid = nullptr;   // optional [n_edges]: global id of each edge's source (layer 0)
    const int64_t* order_tab = nullptr;   // optional micro-batch-major dst row order (extract.h)
    int64_t src_per_mb = 0;               // mean source rows per micro-batch (sizes the gather working set)
};

struct LayerBufs {
    void* XA = nullptr;   void* gat = nullptr;  float* Y = nullptr;   void* G = nullptr;
    float* Ys = nullptr;  float* R = nullptr;   // PF: self half over the dst rows; dS W_s^T residual
    float* dXA = nullptr; float* Zp = nullptr;  int32_t* arg = nullptr; void* dZp = nullptr;
    void* H = nullptr;    // input of layer l (l >= 1), written by layer l-1
    uint32_t* Hbits = nullptr;   // [H > 0] as bits (ldhb words per row), written with H by a tensor-core epilogue
    int64_t ldhb = 0;
    bool hbits_ok = false;       // Hbits holds the current H (set by the forward)
    void* dS = nullptr;   // dS of layer l as GEMM operand (l < L-1)
    void* B = nullptr;    void* Bp = nullptr;
    void* Bt = nullptr;   void* Bpt = nullptr;   // K-major weight copies (tensor-core paths; FP32 mode: hi part)
    // FP32 mode on the tensor cores (3xTF32): hi / lo parts of the weights (null: SIMT FFMA)
    void* Bhi = nullptr;  void* Blo = nullptr;  void* Btlo = nullptr;
    void* Bphi = nullptr; void* Bplo = nullptr; void* Bptlo = nullptr;
    int64_t ldbt = 0, ldbpt = 0;
    int S_main = 1, S_pool = 1, S_self = 1;   // split counts of the dW reductions
};

// CUDA-event brackets around the launches of one kernel site (bench roofline)
enum { PROBE_OFF = 0, PROBE_AGG_L0 = 1, PROBE_GEMM_FWD_L0 = 2, PROBE_GEMM_RED_L0 = 3, PROBE_EXTRACT = 4,
       PROBE_REG = 5, PROBE_AGG_L1 = 6, PROBE_GEMM_FWD_L1 = 7 };
struct Probe {
    int site = PROBE_OFF;
    std::vector<cudaEvent_t> ev;   // pairs
    int used = 0;
    void begin(int here, cudaStream_t s) {
        if (site != here) return;
        if ((int)ev.size() < 2 * (used + 1)) {
            cudaEvent_t a, b;
            cudaEventCreate(&a);
            cudaEventCreate(&b);
            ev.push_back(a);
            ev.push_back(b);
        }
        rec(ev[2 * used], s);
    }
    void end(int here, cudaStream_t s) {
        if (site != here) return;
        rec(ev[2 * used + 1], s);
        ++used;
    }
    static void rec(cudaEvent_t e, cudaStream_t s) {
        cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
        cudaStreamIsCapturing(s, &st);
        // inside a capture the record must be an external event node to be timeable
        if (st == cudaStreamCaptureStatusActive) cudaEventRecordWithFlags(e, s, cudaEventRecordExternal);
        else cudaEventRecord(e, s);
    }
    void destroy() { for (auto e : ev) cudaEventDestroy(e); ev.clear(); used = 0; }
};

struct SageBufs {
    Probe* probe = nullptr;
    const FeatShards* shards = nullptr;     // layer-0 feature table sharded by rows (or null)
    bool tf32 = false;            // FP32 mode products as 3xTF32 on tcgen05 (else SIMT FFMA)
    std::vector<LayerBufs> l;
    float* logits = nullptr;
    float* dS_last = nullptr;
    void* dS_last_act = nullptr;
    float* partials = nullptr;
    std::vector<void*> owned;
    int64_t bytes = 0;
};

// allocate buffers for per-layer capacities (cap_dst[l], cap_src[l])
bool sage_alloc(betty_ctx* c, const ModelCfg& m, const std::vector<int64_t>& cap_dst,
                const std::vector<int64_t>& cap_src, SageBufs* b, cudaStream_t s);
void sage_free(betty_ctx* c, SageBufs* b, cudaStream_t s);
void sage_prep(betty_ctx* c, const ModelCfg& m, SageBufs& b, const float* params, cudaStream_t s);
void sage_forward(betty_ctx* c, const ModelCfg& m, SageBufs& b, const BlockView* v, const void* feats,
                  int64_t ld_feats, cudaStream_t s);
void sage_loss(betty_ctx* c, const ModelCfg& m, SageBufs& b, const BlockView* v, const int32_t* labels, float scale,
               float* loss_accum, cudaStream_t s);
void sage_backward(betty_ctx* c, const ModelCfg& m, SageBufs& b, const BlockView* v, const void* feats,
                   int64_t ld_feats, float* grad, cudaStream_t s);

}  // namespace betty
