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
    int64_t cap_dst, cap_src, cap_e;
};

struct ExtractScratch {
    uint32_t* dstbits;          // [c*Wmax]
    uint32_t* newbits;          // [c*Wmax]
    int32_t* map;               // [c*map_stride]
    int64_t map_stride;
    int32_t* wordcnt;           // [c*Wmax]
    int64_t* wordoff;           // [c*Wmax+1]
    int64_t* deg;               // [max cap_dst]
    int32_t* tcnt;              // [max cap_src]
    int32_t* sel_cnt;           // [c*nchunks]
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
};

void extract_group(betty_ctx* ctx, const ExtractArgs& a, cudaStream_t s);

}  // namespace betty
