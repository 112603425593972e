// reg.h -- internal interface of the REG SpGEMM (reg.cu).
#pragma once
#include <stdint.h>
#include <cuda_runtime.h>

struct betty_ctx;
namespace betty {

struct RegArgs {
    // The REG rows [row0, row0 + n_rows) of the output block: `indptr` points at the block's
    // indptr + row0 (offsets stay absolute into idx); the CSC is built from the whole block
    // (full_indptr, n_full_rows), since a row's candidates are every output sharing a source.
    const int64_t* indptr;      // output block CSR rows of the slice (rows = outputs)
    const int32_t* idx;         // full-batch src positions
    const int64_t* n_rows_dev;  // device counts: rows of the slice
    const int64_t* n_cols_dev;
    const int64_t* n_edges_dev; // edges of the whole block
    int64_t rows_cap, cols_cap, edges_cap;
    const int64_t* full_indptr; // the whole output block
    const int64_t* n_full_rows_dev;
    int64_t full_rows_cap;
    int64_t row0;               // global id of the slice's first row (diagonal exclusion)
    bool csc_ready = false;     // t_indptr / t_idx already hold the block's CSC (a plan builds it once)
    int64_t* t_indptr;          // [cols_cap+1]
    int32_t* t_idx;             // [edges_cap]
    int32_t* tcnt;              // [cols_cap]
    int64_t* ub;                // [rows_cap]
    int64_t* off;               // [rows_cap+1]
    int64_t* ub_total_dev;
    int32_t* tcol;              // [ub_cap]
    int32_t* tw;                // [ub_cap]
    int64_t* row_nnz;           // [rows_cap]
    int64_t* out_indptr;        // [rows_cap+1]
    int64_t* nnz_total_dev;
    // hub rows (more than REG_CTA_MAX candidate products): one CTA per row over a bitmap of the
    // output ids, per-CTA scratch of hub_words words (bitmap + popcount prefix) x num_sms CTAs
    uint32_t* hub_bits = nullptr;
    int32_t* hub_pre = nullptr;
    int64_t hub_words = 0;
};
// phase 1: CSC + product counts (ub) + their scan (ub_total known after it)
void reg_phase1(betty_ctx* c, const RegArgs& a, cudaStream_t s);
// phase 2: expand / sort / RLE per row into tcol/tw (sized >= ub_total) + indptr scan
void reg_phase2(betty_ctx* c, const RegArgs& a, cudaStream_t s);
// phase 3: compaction into col/w (sized >= nnz_total)
void reg_phase3(betty_ctx* c, const RegArgs& a, int32_t* col, int32_t* w, int64_t nnz_cap, cudaStream_t s);

}  // namespace betty
