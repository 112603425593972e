/*
 * betty.h -- C ABI of the B200-native hot path of Betty's batch-level
 * partitioned GNN training step (Yang et al., ASPLOS '23; PAPER.md).
 *
 * The library (paper_conf_asplos_yangzd023_b200/libbetty.so) is hand-written
 * CUDA for sm_100a.  Every entry point takes plain pointers and sizes; no torch
 * types cross this boundary.  Unless noted, pointers are DEVICE pointers on
 * the ctx's device, calls are stream-ordered on `stream` (a cudaStream_t,
 * passed as void* so this header needs no CUDA include) and asynchronous.
 * No exceptions cross the ABI; every failure is a betty_status, with a message
 * from betty_last_error().
 *
 * Terminology (§4.2.2-4.2.3).  A batch is a multi-level
 * bipartite graph: block l (l = 0 input ... L-1 output) has dst nodes V and
 * src nodes U with dst ids == src ids [0, n_dst) (the dst list is a prefix of
 * the src list).  Betty partitions the output nodes into K micro-batches; the
 * micro-batch k of every layer is the sub-bipartite reachable from its
 * outputs.  Gradients of the K micro-batches are summed and give the
 * full-batch gradient.
 */
#ifndef BETTY_H
#define BETTY_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define BETTY_API __attribute__((visibility("default")))
#else
#define BETTY_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    BETTY_OK = 0,
    BETTY_EINVAL = 1,       /* bad argument (null pointer, k out of range, part[] out of range, duplicate edge ...) */
    BETTY_ENOMEM = 2,       /* the allocator returned null */
    BETTY_ECUDA = 3,        /* a CUDA runtime error; message in betty_last_error */
    BETTY_EOVERFLOW = 4,    /* a size exceeds int32 local ids or a plan capacity */
    BETTY_EUNSUPPORTED = 5  /* a configuration this build does not implement */
} betty_status;

typedef struct betty_ctx betty_ctx;
typedef void* betty_stream;                                          /* cudaStream_t */
typedef void* (*betty_alloc_fn)(size_t bytes, betty_stream stream, void* user);
typedef void (*betty_free_fn)(void* ptr, betty_stream stream, void* user);

/* One context per device (per rank).  alloc/free may be NULL: the library
 * then uses the CUDA stream-ordered allocator (cudaMallocAsync).  Outputs of
 * betty_extract_blocks / betty_reg_build / betty_sage_fwd and plan arenas come
 * from this allocator and are released with the matching *_free call.
 * Calls on one context must be ordered on ONE stream (or otherwise serialised):
 * the context's device scratch -- scan flags, work-claim counters (aggregation,
 * extraction, row-GEMM tile claims), loss partials -- is shared by its calls and
 * reset by each kernel for the next one.  A plan's in-step REG rebuild uses its
 * own side-stream scratch.  Concurrent work needs one context per stream. */
BETTY_API betty_status betty_ctx_create(int device, betty_alloc_fn alloc, betty_free_fn dealloc, void* user, betty_ctx** out);
BETTY_API void betty_ctx_destroy(betty_ctx* ctx);
BETTY_API const char* betty_last_error(const betty_ctx* ctx);
BETTY_API const char* betty_version(void);

/* One bipartite layer, CSR by dst.
 *   indptr    [n_dst+1] int64    row offsets
 *   indices   [n_edges] int32    src ids: local ids for a micro-batch; for the FULL batch given to
 *                                betty_extract_blocks, positions in the full-batch src list
 *   src_pos   [n_src]   int32    position of each src in the full-batch src list of this layer
 *                                (NULL for the full batch = identity)
 *   src_gid   [n_src]   int32    global node id (row of the feature / label tables)
 *   t_indptr  [n_src+1] int64    CSC (dst ids per src), may be NULL on input
 *   t_indices [n_edges] int32    dst ids, ascending per column
 * Canonical order (readings #9/#10): outputs ascending; src =
 * dst ++ (new sources ascending full-batch src position); rows keep the
 * full-batch order.  Sizes are host values. */
typedef struct {
    int64_t n_dst, n_src, n_edges;
    int64_t* indptr;
    int32_t* indices;
    int32_t* src_pos;
    int32_t* src_gid;
    int64_t* t_indptr;
    int32_t* t_indices;
} betty_block;

/* Symmetric weighted CSR (the REG): n rows, nnz entries, int64 indptr[n+1],
 * int32 col[nnz] ascending per row, int32 w[nnz] >= 1, no diagonal. */
typedef struct {
    int64_t n, nnz;
    int64_t* indptr;
    int32_t* col;
    int32_t* w;
} betty_csr;

/* aggregators of Table 1: mean h_N = (1/D_v) sum_u h_u; pool max_u ReLU(W_pool h_u +
 * b_pool); sum h_N = sum_u h_u (mean without 1/D_v, the same SAGEConv form and project-first rule) */
enum { BETTY_AGGR_MEAN = 0, BETTY_AGGR_POOL = 1, BETTY_AGGR_SUM = 2 };
enum { BETTY_GEMM_FP32 = 0, BETTY_GEMM_BF16 = 1 };
enum { BETTY_FEAT_FP32 = 0, BETTY_FEAT_BF16 = 1 };

/* GraphSAGE model (Table 1; Eq. 1; DGL SAGEConv
 * form, reading #11): L layers of widths dims[0..L] (host array).
 * Parameters are one flat fp32 vector; per layer l (Fi = dims[l], Fo = dims[l+1]):
 *   pool only: W_pool [Fi x Fi], b_pool [Fi]
 *   W_self [Fi x Fo], W_neigh [Fi x Fo], b [Fo]          (row-major, x . W)
 * gemm: FP32 = fp32 operands; the products run on tcgen05 as 3xTF32 (hi*hi +
 * lo*hi + hi*lo of an RN tf32 split, fp32 accumulation with the small terms
 * in their own accumulator and dW totals drained every 64 nodes: ~fp32
 * accuracy, never plain TF32; env BETTY_FP32_SIMT=1 selects SIMT FFMA); BF16 = GEMM operands in bf16,
 * fp32 accumulation, aggregation / loss / gradients fp32, hidden activations
 * stored bf16 (reading #17).  feat_dtype says how `feats` is stored. */
typedef struct {
    int32_t L;
    int32_t aggr;
    int32_t gemm;
    int32_t feat_dtype;
    const int32_t* dims;
} betty_model;

BETTY_API int64_t betty_num_params(const betty_model* model);

/* a1 -- REG (§4.3.2, Eq. 2-4, Alg. 1 lines 1-7 PAPER.md:934-940).
 * out_layer: the output block of the FULL batch (n_dst = n_out rows, indices =
 * full-batch src positions in [0, n_src)).  Computes c_ij = #shared sources of
 * outputs i != j as an integer SpGEMM B.B^T (B[i,u] = 1 iff u -> i); zero
 * entries dropped, diagonal removed.  Rows must not repeat a source (binary A,
 * reading #2): a repeat returns EINVAL.  Allocates reg's arrays; synchronizes
 * the stream once to learn nnz.  Result is bit-exact (integer). */
BETTY_API betty_status betty_reg_build(betty_ctx* ctx, const betty_block* out_layer, betty_csr* reg, betty_stream stream);
/* The REG rows [row0, row1) only (0 <= row0 <= row1 <= n_out), e.g. one rank's share when the
 * rows are sharded across ranks: reg->n = row1 - row0, reg->indptr rebased to
 * the slice, columns are GLOBAL output ids.  Row i of the slice equals row row0 + i of
 * betty_reg_build's result, bit-exact.  Bad ranges return EINVAL. */
BETTY_API betty_status betty_reg_build_rows(betty_ctx* ctx, const betty_block* out_layer, int64_t row0, int64_t row1,
                                            betty_csr* reg, betty_stream stream);
BETTY_API void betty_csr_free(betty_ctx* ctx, betty_csr* reg);

/* a2 -- micro-batch extraction (batch-level partition, PAPER.md:535-547;
 * block generation and the local<->global index map).
 * full[L]: full-batch blocks (indices = full-batch src positions; src_pos may
 * be NULL).  part[n_out] (device) assigns each output position to [0,K).
 * Fills mb[L] with micro-batch k (all arrays allocated, CSC included,
 * sizes written on the host after one stream synchronisation).  part values
 * out of range return EINVAL.  An empty micro-batch yields zero-sized blocks.
 * Limits of the output selection: K <= 16384, n_out < 2^23 - 1 and fewer than
 * 2^40 top-layer edges, else BETTY_EUNSUPPORTED (also for betty_mb_sizes and
 * betty_plan_create, whose launch groups hold <= 512 micro-batches). */
BETTY_API betty_status betty_extract_blocks(betty_ctx* ctx, const betty_block* full, int32_t L, const int32_t* part,
                                  int64_t n_out, int32_t K, int32_t k, betty_block* mb, betty_stream stream);
BETTY_API void betty_block_free(betty_ctx* ctx, betty_block* blocks, int32_t L);

/* a3 -- forward of one micro-batch (mean: h_N = (1/D_v) sum h_u, or pool:
 * max_u ReLU(W_pool h_u + b_pool); then h_v W_self + h_N W_neigh + b; ReLU
 * between layers).  mb[L] as returned by betty_extract_blocks (host sizes,
 * CSC present).  feats: [N x ld_feats] table indexed by src_gid of layer 0.
 * logits (optional) [n_dst(L-1) x dims[L]] fp32.  *saved receives the
 * activations the backward needs (free with betty_saved_free). */
typedef struct betty_saved betty_saved;
BETTY_API betty_status betty_sage_fwd(betty_ctx* ctx, const betty_model* model, const float* params, const betty_block* mb,
                            const void* feats, int64_t ld_feats, betty_saved** saved, float* logits,
                            betty_stream stream);
/* a4+a5+a6 -- softmax cross-entropy on the micro-batch's outputs (labels[gid],
 * int32), scaled by loss_scale (1/n_out of the full batch, so that the K
 * micro-batch losses sum to the full-batch mean loss, reading #15), and the
 * backward, ADDING the gradient into grad_accum[num_params] (fused
 * accumulation across micro-batches) and the loss into
 * loss_accum[0]. */
BETTY_API betty_status betty_sage_bwd(betty_ctx* ctx, const betty_model* model, const float* params, const betty_block* mb,
                            const betty_saved* saved, const int32_t* labels, float loss_scale, float* grad_accum,
                            float* loss_accum, betty_stream stream);
BETTY_API void betty_saved_free(betty_ctx* ctx, betty_saved* saved);

/* The fused per-step path.  A plan binds the full batch, the partition and
 * this rank's micro-batches my_k[n_my] (host array); it runs one extraction
 * pass (synchronising) to size device arenas, so that betty_step itself never
 * synchronises and can be captured in / replayed as a CUDA graph.
 * group: micro-batches executed together per launch (>= 1; <= 0 means all of
 * this rank's).  A group is the block-diagonal union of its micro-batches:
 * per-micro-batch dedupe / relabel / numerics are unchanged; memory grows
 * with the group.  flags: BETTY_PLAN_GRAPH captures the step as a CUDA graph
 * on first use; BETTY_PLAN_REG rebuilds the REG (a1) inside every step;
 * BETTY_PLAN_FRESH makes every step derive everything it needs from the
 * current contents of the bound full-batch buffers (indptr / indices /
 * src_gid and part): the full-batch CSCs the extraction filters and the
 * REG's CSC are rebuilt in the step (duplicate edges flagged) instead of
 * once at plan creation -- the mode for a batch re-copied or resampled into
 * the same buffers every step (sizes must stay within the plan's, checked on
 * the device: BETTY_EOVERFLOW at the next synchronising call). */
typedef struct betty_plan betty_plan;
enum { BETTY_PLAN_GRAPH = 1, BETTY_PLAN_REG = 2, BETTY_PLAN_FRESH = 4 };
typedef struct {
    int32_t n_groups;            /* launch groups per step */
    int32_t L;
    int64_t edges[16];           /* sum over this rank's micro-batches of E_l   (l = 0..L-1) */
    int64_t n_src[16];           /* sum of n_src,l */
    int64_t n_dst[16];           /* sum of n_dst,l */
    int64_t max_group_edges[16]; /* capacity used for layer l */
    int64_t reg_nnz;             /* last REG nnz (BETTY_PLAN_REG) */
    int64_t arena_bytes;         /* device bytes held by the plan */
    int32_t kernels_per_step;    /* library kernel launches per betty_step */
} betty_plan_info;
BETTY_API betty_status betty_plan_create(betty_ctx* ctx, const betty_model* model, const betty_block* full, int32_t L,
                               const int32_t* part, int64_t n_out, int32_t K, const int32_t* my_k, int32_t n_my,
                               int32_t group, int32_t flags, betty_plan** out, betty_stream stream);
BETTY_API betty_status betty_plan_info_get(const betty_plan* plan, betty_plan_info* info);
/* Restrict the in-step REG rebuild (BETTY_PLAN_REG) of this plan to output rows [row0, row1):
 * with R ranks, rank r takes rows [r n_out / R, (r+1) n_out / R) so the REG work is sharded
 * instead of repeated on every rank.  Synchronises `stream`, re-sizes the REG buffers (one
 * sizing pass) and drops a captured graph (re-captured by the next betty_step).  EINVAL for a
 * plan created without BETTY_PLAN_REG or a bad range. */
BETTY_API betty_status betty_plan_set_reg_rows(betty_ctx* ctx, betty_plan* plan, int64_t row0, int64_t row1,
                                               betty_stream stream);
BETTY_API void betty_plan_destroy(betty_ctx* ctx, betty_plan* plan);

/* Feature table sharded by rows across R device buffers (BASELINE.json configs[4]: "features sharded
 * across 8 GPUs' HBM"): global row g lives in base[g / rows_per_shard] at local row
 * g % rows_per_shard, with the row stride (ld_feats) and dtype betty_step is called with.  base[]
 * (HOST array of R device pointers, 16-byte aligned) may hold other GPUs' buffers mapped with
 * betty_ipc_open: the plan's layer-0 gathers then read remote rows over NVLink (owner-computes is
 * not needed: the one gather per edge goes to the owning shard).  The feats argument of betty_step
 * is then ignored for layer 0.  R = 0 returns to one contiguous table.  Supported for an
 * aggregate-first layer 0 (mean / sum with F_in <= F_out), else BETTY_EUNSUPPORTED; EINVAL for
 * R > 64 or bad pointers.  The caller owns the buffers (they must outlive the plan's steps). */
BETTY_API betty_status betty_plan_set_feature_shards(betty_ctx* ctx, betty_plan* plan, int32_t R,
                                                     const void* const* base, int64_t rows_per_shard);
/* Device buffers other processes can map (CUDA IPC): betty_dev_alloc (cudaMalloc on the ctx's
 * device), betty_ipc_handle (64 opaque bytes, host), betty_ipc_open (maps another process's buffer
 * into this one; peer access enabled lazily), betty_ipc_close, betty_dev_free.  ECUDA on failure. */
#define BETTY_IPC_HANDLE_BYTES 64
BETTY_API betty_status betty_dev_alloc(betty_ctx* ctx, size_t bytes, void** out);
BETTY_API betty_status betty_dev_free(betty_ctx* ctx, void* p);
BETTY_API betty_status betty_ipc_handle(betty_ctx* ctx, void* dev_ptr, void* handle);
BETTY_API betty_status betty_ipc_open(betty_ctx* ctx, const void* handle, void** dev_ptr);
BETTY_API betty_status betty_ipc_close(betty_ctx* ctx, void* dev_ptr);

/* One training step on this rank: for every micro-batch of the plan,
 * extraction (a2) -> forward (a3) -> loss (a4) -> backward (a5) with the
 * gradient ADDED into grad_accum (a6).  The caller then all-reduces
 * grad_accum across ranks (NCCL) and applies betty_adam (a7). */
BETTY_API betty_status betty_step(betty_ctx* ctx, betty_plan* plan, const float* params, const void* feats,
                        int64_t ld_feats, const int32_t* labels, float loss_scale, float* grad_accum,
                        float* loss_accum, betty_stream stream);

/* a7 -- Adam (PyTorch semantics; PAPER.md:1115-1118 names Adam), one fused
 * kernel over the flat parameter vector: m = b1 m + (1-b1) g;
 * v = b2 v + (1-b2) g^2; p -= lr * (m / (1-b1^t)) / (sqrt(v / (1-b2^t)) + eps).
 * zero_grad != 0 also clears g for the next step. */
BETTY_API betty_status betty_adam(betty_ctx* ctx, float* params, float* grad, float* m, float* v, int64_t n, int32_t t,
                        float lr, float b1, float b2, float eps, int32_t zero_grad, betty_stream stream);

/* Inspection hook (tests): run the extraction of launch group g of the plan
 * and describe its group-concatenated blocks: the block-diagonal union of the
 * group's micro-batches (my_k order) with ids global within the group -- the
 * output layer lists each micro-batch's outputs in turn; every layer's src
 * list is [its dst list] ++ [new sources of micro-batch 0] ++ [of 1] ++ ...
 * (dst ids stay a prefix of src ids), and the next layer's dst list is that
 * src list.  Arrays point INTO the plan's arenas (valid until the next step);
 * sizes are host values (synchronises). */
BETTY_API betty_status betty_plan_group_blocks(betty_ctx* ctx, betty_plan* plan, int32_t g, betty_block* out,
                                               betty_stream stream);

/* Test hook for the dense kernels (fp32 result; synchronises).
 * kind 0: C[M x N] = A[M x K] . B^T with B given K-major as [N x K];
 * kind 1: C[K x N] += A[M x K]^T . B[M x N] (the dW reduction; C must be
 * [K x N] contiguous).  kind | 2: fp32 operands (FP32 mode: 3xTF32 on
 * tcgen05 when use_tc, else SIMT FFMA); otherwise bf16 operands.  use_tc
 * selects the tcgen05 path (else SIMT). */
BETTY_API betty_status betty_test_gemm(betty_ctx* ctx, int32_t kind, const void* A, int64_t lda, const void* B,
                                       int64_t ldb, int64_t M, int64_t M_cap, int32_t K, int32_t N, float* C,
                                       int64_t ldc, int32_t use_tc, betty_stream stream);

/* Measurement hook: bracket every launch of one kernel site with CUDA events
 * on the step's stream in subsequent betty_step calls (graph replays
 * included; changing the site re-captures the graph).  Sites: 0 off,
 * 1 layer-0 aggregation, 2 layer-0 forward GEMM, 3 layer-0 dW GEMM,
 * 4 extraction (whole group), 5 REG, 6 layer-1 aggregation, 7 layer-1
 * forward GEMM.  probe_read synchronises and returns the summed elapsed time
 * of the last step's bracketed launches and their number. */
enum { BETTY_PROBE_OFF = 0, BETTY_PROBE_AGG_L0 = 1, BETTY_PROBE_GEMM_FWD_L0 = 2, BETTY_PROBE_GEMM_RED_L0 = 3,
       BETTY_PROBE_EXTRACT = 4, BETTY_PROBE_REG = 5, BETTY_PROBE_AGG_L1 = 6, BETTY_PROBE_GEMM_FWD_L1 = 7 };
BETTY_API betty_status betty_plan_probe(betty_plan* plan, int32_t site);
BETTY_API betty_status betty_plan_probe_read(betty_plan* plan, float* total_ms, int32_t* launches);

/* HOST function, outside the hot path (Alg. 1 line 8, where
 * the paper calls METIS): K-way partition of a REG given as HOST arrays
 * (indptr[n+1], col[nnz], w[nnz] or NULL for unit weights) by greedy graph
 * growing on the REG weights (the most shared inputs stay together), with
 * balanced part sizes floor/ceil(n/K).  Writes part[n] (host).  Deterministic. */
BETTY_API betty_status betty_reg_partition(const int64_t* indptr, const int32_t* col, const int32_t* w, int64_t n,
                                           int32_t K, int32_t* part);

/* §4.4 memory-aware batch-level partitioning (Table 3).
 *
 * betty_mb_sizes: count-only extraction (a2 without emitting the blocks) of
 * every micro-batch k in [0,K) of the partition part[n_out] (device): writes
 * sizes[(k*L + l)*3 + {0,1,2}] = n_dst, n_src, n_edges of layer l (HOST
 * array, K*L*3 int64).  Synchronises once per micro-batch; EINVAL on bad
 * arguments or part values out of range.
 *
 * betty_mem_estimate (HOST arithmetic, no GPU): the paper's estimate of one
 * micro-batch from its per-layer sizes[L*3] (as above).  terms[9] receives
 * element counts of (1) N_P_GNN, (2) N_in x H_in, (3) N_out, (4) 3 x sum E,
 * (5) sum_l n_dst,l x dims[l+1], (6) aggregator intermediates (mean
 * sum n_dst,l x dims[l]; pool sum (n_src,l + n_dst,l) x dims[l]), (7)
 * gradients N_P_GNN + N_P_Agg, (8) Adam states 2 (N_P_GNN + N_P_Agg), and
 * terms[8] = peak = (1)+(2)+(3)+(4)+(5)+(8) + max((6),(7)) (
 * readings M1-M4 in DESIGN.md §3).  Bytes = 4 x elements.
 *
 * betty_memory_aware_k: for K = K0, K0+1, ... <= K_max (<= 0: n_out),
 * partition the REG (HOST arrays) K ways with betty_reg_partition_ex(method,
 * imbalance 0.03), size every
 * micro-batch on the GPU and estimate it; stop at the first K whose largest
 * estimate (bytes) is <= capacity_bytes.  Writes
 * part[n_out] (HOST) and *K_out = K, *peak_bytes = that K's largest
 * estimate; when no K fits, *K_out = -1, part untouched and *peak_bytes =
 * the smallest largest-estimate seen.  Synchronises. */
BETTY_API betty_status betty_mb_sizes(betty_ctx* ctx, const betty_block* full, int32_t L, const int32_t* part,
                                      int64_t n_out, int32_t K, int64_t* sizes, betty_stream stream);
BETTY_API betty_status betty_mem_estimate(const betty_model* model, const int64_t* sizes, int64_t* terms);
BETTY_API betty_status betty_memory_aware_k(betty_ctx* ctx, const betty_model* model, const betty_block* full,
                                            int32_t L, const int64_t* reg_indptr, const int32_t* reg_col,
                                            const int32_t* reg_w, int64_t n_out, int64_t capacity_bytes,
                                            int32_t K0, int32_t K_max, int32_t method, int32_t* part,
                                            int32_t* K_out, int64_t* peak_bytes, betty_stream stream);

/* HOST function, outside the hot path: K-way REG partition by `method`:
 * BETTY_PART_GREEDY = betty_reg_partition (exactly balanced sizes);
 * BETTY_PART_MULTILEVEL = the METIS scheme the paper uses (Alg. 1 line 8,
 * PAPER.md:917-941): heavy-edge-matching coarsening, greedy-growing initial
 * partition, greedy boundary refinement while uncoarsening; minimises the
 * cut REG weight (the inputs duplicated across micro-batches) subject to
 * every part holding <= ceil((1 + imbalance) n / K) outputs.  Host arrays
 * (as betty_reg_partition); deterministic; EINVAL on bad arguments. */
enum { BETTY_PART_GREEDY = 0, BETTY_PART_MULTILEVEL = 1 };
BETTY_API betty_status betty_reg_partition_ex(const int64_t* indptr, const int32_t* col, const int32_t* w, int64_t n,
                                              int32_t K, int32_t method, double imbalance, int32_t* part);

/* Synchronise `stream` and report device-side errors of earlier
 * asynchronous calls (part[] out of range -> EINVAL, capacity exceeded ->
 * EOVERFLOW, CUDA faults -> ECUDA). */
BETTY_API betty_status betty_sync_check(betty_ctx* ctx, betty_stream stream);

#ifdef __cplusplus
}
#endif
#endif /* BETTY_H */
