// internal.h -- host-side internals of libbetty (not part of the C ABI).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <string>
#include <vector>
#include "../../include/betty.h"

struct betty_ctx {
    int device = 0;
    int num_sms = 148;
    bool use_tc = true;                          // tcgen05 GEMMs (env BETTY_NO_TC=1 disables)
    bool fp32_tc = true;                         // FP32 mode as 3xTF32 on tcgen05 (env BETTY_FP32_SIMT=1: FFMA)
    betty_alloc_fn alloc = nullptr;
    betty_free_fn dealloc = nullptr;
    void* user = nullptr;
    std::string err;
    // scratch of the stream-ordered primitives, one set per concurrent stream ("lane"):
    // lane 0 = the caller's stream, lane 1 = a plan's side stream (REG inside the step)
    struct Lane {
        unsigned long long* scan_status = nullptr;   // decoupled look-back tile status
        int64_t scan_status_cap = 0;
        unsigned* counters = nullptr;                // [64] device counters, kept zero between launches
        int64_t* big_list = nullptr;                 // work list for oversize segments
        int64_t big_list_cap = 0;
        int* big_count = nullptr;
    };
    Lane lanes[2];
    int lane = 0;                                // the set launches issued now use
    Lane& L() { return lanes[lane]; }
    int* dev_err = nullptr;                      // device-side error flags (see betty::DEVERR_*)
    std::vector<void*> retired;                  // outgrown scratch still referenced by captured graphs
};

namespace betty {

enum { DEVERR_OVERFLOW = 1, DEVERR_DUP_EDGE = 2, DEVERR_BAD_PART = 4 };
enum { CTR_SCAN = 0, CTR_SCAN_DONE = 1, CTR_LOSS = 4, CTR_LOSS_DONE = 5, CTR_AGG = 8, CTR_EXTRACT = 10, CTR_GEMM = 32 };

void* ctx_alloc(betty_ctx* c, size_t bytes, cudaStream_t s);
void ensure_scan_scratch(betty_ctx* c, int64_t n_cap, cudaStream_t s);
void init_prims_attrs();
void init_reg_attrs();
inline void init_kernel_attrs() { init_prims_attrs(); init_reg_attrs(); }
void ctx_free(betty_ctx* c, void* p, cudaStream_t s);

// ---- primitives (csrc/prims.cu) ----
// out[0] = 0, out[i+1] = sum_{j<=i} in[j] for i < n; n = *n_dev (device) or n_fixed when n_dev == null.
// If total_dev != null it receives out[n].
void scan_i64(betty_ctx* c, const int64_t* in, int64_t* out, const int64_t* n_dev, int64_t n_fixed, int64_t n_cap,
              int64_t* total_dev, cudaStream_t s);
void scan_i32(betty_ctx* c, const int32_t* in, int64_t* out, const int64_t* n_dev, int64_t n_fixed, int64_t n_cap,
              int64_t* total_dev, cudaStream_t s);
// sort each segment [ptr[i], ptr[i+1]) of keys ascending, i < *nseg_dev (or nseg_fixed)
void segsort_i32(betty_ctx* c, const int64_t* ptr, int32_t* keys, const int64_t* nseg_dev, int64_t nseg_fixed,
                 int64_t nseg_cap, cudaStream_t s);
// CSR (indptr by row, indices = column ids) -> CSC with ascending row ids per column.
// n_rows/n_cols/n_edges device counts; t_indptr [n_cols+1] int64, t_idx [n_edges];
// cnt_scratch int32 [n_cols_cap] (zeroed and used as cursor).  dup_check: flag DEVERR_DUP_EDGE
// if a column has a repeated row (i.e. a row has a repeated column).
void csr_transpose(betty_ctx* c, const int64_t* indptr, const int32_t* idx, const int64_t* n_rows_dev,
                   const int64_t* n_cols_dev, const int64_t* n_edges_dev, int64_t rows_cap, int64_t cols_cap,
                   int64_t edges_cap, int64_t* t_indptr, int32_t* t_idx, int32_t* cnt_scratch, bool dup_check,
                   cudaStream_t s);
void memset_dev(void* p, int value, const int64_t* n_dev, int64_t elem_bytes, int64_t n_cap, cudaStream_t s);

}  // namespace betty
