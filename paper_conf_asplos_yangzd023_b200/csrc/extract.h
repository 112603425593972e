// extract.h -- internal interface of the group extraction (extract.cu).
#pragma once
#include <stdint.h>
#include <cuda_runtime.h>

struct betty_ctx;
namespace betty {

struct ExtractFull {            // full-batch block l (device arrays, host sizes)
    int64_t n_dst, n_src, n_edges;
    const int64_t* indptr;
    const int32_t* nbr;         // full-batch src positions
    const int32_t* src_gid;
    const int64_t* t_indptr = nullptr;   // optional full-batch CSC (built once per plan): [n_src+1]
    const int32_t* t_nbr = nullptr;      // [n_edges] full dst rows, ascending per column
    const int32_t* egid = nullptr;       // optional [n_edges]: global id of each edge's source (src_gid[nbr])
};

struct ExtractLayer {           // group-concatenated micro-batch layer l (device arrays)
    int64_t* indptr;            // [cap_dst+1]
    int32_t* indices;           // [cap_e]   src ids, global within the group
    int32_t* src_pos;           // [cap_src]
    int32_t* src_gid;           // [cap_src]
    int32_t* src_mb;            // [cap_src] slot j of each src row
    int64_t* t_indptr;          // [cap_src+1] (null: no CSC)
    int32_t* t_indices;         // [cap_e]
    int32_t* egid;              // [cap_e] or null: global id of each edge's source (feeds the layer-0 gather)
    int64_t* cnt;               // device [4]: n_dst, n_src, n_edges, spare
    int64_t* mb_src_off;        // [c+1]
    int64_t* order_tab;         // [2*(ORDER_TAB_MAX+1)] or null: micro-batch-major dst row order (see below)
    int64_t cap_dst, cap_src, cap_e;
};

// Micro-batch-major processing order of the dst rows of a layer l < L-1.  The
// group layout lists them as [top rows] ++ [new sources of layer L-1] ++ ... ++
// [new sources of layer l+1], each phase grouped by micro-batch; kernels that
// gather per dst row (the layer-0 aggregation) visit them micro-batch by
// micro-batch so that one micro-batch's source rows stay L2-resident.  The
// table holds the virtual starts vs[0..n_seg] (ascending, at [0]), the real
// starts rs[0..n_seg) (at [ORDER_TAB_MAX+1]) and n_seg (at [2*(ORDER_TAB_MAX+1)]):
// virtual row v in [vs[i], vs[i+1]) is real row rs[i] + (v - vs[i]).
constexpr int ORDER_TAB_MAX = 1024;
__host__ __device__ inline int order_tab_segs(int c, int L, int l) { return c * (L - l); }

#ifdef __CUDACC__
constexpr int ORDER_SMEM = 256;       // segments a kernel keeps in shared memory (more: identity order)
// block-cooperative: copy the table into shared memory; returns n_seg (0 = identity order)
__device__ __forceinline__ int order_load(const int64_t* otab, int64_t* s_vs, int64_t* s_rs) {
    if (!otab) return 0;
    int nseg = (int)otab[2 * (ORDER_TAB_MAX + 1)];
    if (nseg > ORDER_SMEM) nseg = 0;
    for (int i = threadIdx.x; i <= nseg; i += blockDim.x) {
        s_vs[i] = otab[i];
        if (i < nseg) s_rs[i] = otab[ORDER_TAB_MAX + 1 + i];
    }
    __syncthreads();
    return nseg;
}
// virtual row -> real row; `seg` caches the last segment
__device__ __forceinline__ int64_t order_map(int64_t vv, int nseg, const int64_t* s_vs, const int64_t* s_rs, int& seg) {
    if (nseg == 0) return vv;
    if (!(s_vs[seg] <= vv && vv < s_vs[seg + 1])) {
        int lo = 0, hi = nseg;                          // s_vs[lo] <= vv < s_vs[hi]
        while (hi - lo > 1) {
            const int mid = (lo + hi) >> 1;
            if (s_vs[mid] <= vv) lo = mid; else hi = mid;
        }
        seg = lo;
    }
    return s_rs[seg] + (vv - s_vs[seg]);
}
#endif

struct ExtractScratch {
    uint32_t* dstbits;          // [c*Wmax]
    uint32_t* newbits;          // [c*Wmax]
    // rank structures kept for the whole extraction: per layer the new-source bitmap of
    // every slot with, per 32-bit word, the slot-relative count of set bits before it
    // ({bits, prefix}); for the top layer the same for the dst (output) bitmap.  A source's
    // local id is then computed (no position -> id map): see src_id() in extract.cu
    uint2* nrank[16];           // [c*W_l]
    uint2* drank_top;           // [c*W_{L-1}]
    int64_t* wordoff;           // [c*Wmax+1]
    int32_t* tcnt;              // [max cap_src]
    int32_t* ndeg;              // [max cap_src]: full-batch degrees of the next layer's dst rows
    int64_t* sel_cnt;           // [c*nchunks] (selection: count << 40 | degree sum, per slot and chunk)
    int64_t* sel_off;           // [c*nchunks+1]
    int32_t* top_dst_pos;       // [n_out]
    int32_t* top_row_mb;        // [n_out]
    int64_t* top_dst_off;       // [c+1]
};

struct ExtractArgs {
    int L;
    const ExtractFull* full;    // [L]
    const int32_t* part;        // [n_out] device
    int32_t K;
    const int32_t* ks;          // [c] device: micro-batch id of each slot
    int32_t c;
    ExtractLayer* layers;       // [L]
    ExtractScratch sc;
    uint32_t csc_mask;          // bit l: build the CSC of layer l
    // lean0: layer 0's sources are not materialised -- its rows (indptr, the dst prefix's src_pos /
    // src_gid) and the per-edge source gids (egid, copied row segment by row segment from the
    // full batch's full[0].egid) are all an aggregate-first layer 0 consumes: its features are
    // gathered by global id from the resident table, no kernel reads the layer's src list, local
    // indices or CSC.  The plan's step sets it; standalone / inspection extractions never do.
    bool lean0 = false;
    // egid_direct: the lean layer 0 reads each edge's source gid as src_gid[nbr[e]] of the full batch
    // instead of the per-plan full[0].egid array (a FRESH step: its blocks change every step, so the
    // array would be rebuilt first -- one more pass over the full batch's edges)
    bool egid_direct = false;
};

void extract_group(betty_ctx* ctx, const ExtractArgs& a, cudaStream_t s);
// outputs per selection chunk (one CTA each; 256: 8 serial steps per warp in the write pass)
constexpr int SEL_CHUNK = 256;
// the selection's limits (extract.cu): K <= 16384 micro-batches, launch groups of <= 512, fewer than
// 2^23 - 1 outputs and 2^40 top-layer edges
bool extract_limits_ok(int32_t K, int32_t c, int64_t n_out, int64_t top_edges);

}  // namespace betty
