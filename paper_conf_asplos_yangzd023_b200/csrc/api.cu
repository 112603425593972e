// api.cu -- the C ABI of include/betty.h: validation, allocation, the
// standalone entry points, plans and the graph-captured fused step.
#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <new>
#include <vector>
#include "internal.h"
#include "extract.h"
#include "model.h"
#include "reg.h"

using namespace betty;

namespace betty {
void* ctx_alloc(betty_ctx* c, size_t bytes, cudaStream_t s) {
    if (bytes == 0) bytes = 16;
    if (c->alloc) return c->alloc(bytes, (betty_stream)s, c->user);
    void* p = nullptr;
    if (cudaMallocAsync(&p, bytes, s) != cudaSuccess) {
        // reported through the return value (BETTY_ENOMEM); consume the error so the next call's
        // launch checks do not see it as a failure of their own
        cudaGetLastError();
        return nullptr;
    }
    return p;
}
void ctx_free(betty_ctx* c, void* p, cudaStream_t s) {
    if (!p) return;
    if (c->dealloc) c->dealloc(p, (betty_stream)s, c->user);
    else cudaFreeAsync(p, s);
}
size_t extract_scratch_bytes(int64_t c, int64_t max_full_src, int64_t sel_nchunks);
}  // namespace betty

static betty_status fail(betty_ctx* c, betty_status st, const char* fmt, ...) {
    if (c) {
        char buf[512];
        va_list ap;
        va_start(ap, fmt);
        vsnprintf(buf, sizeof buf, fmt, ap);
        va_end(ap);
        c->err = buf;
    }
    return st;
}

#define CUDA_OK(ctx, expr)                                                                   \
    do {                                                                                     \
        cudaError_t _e = (expr);                                                             \
        if (_e != cudaSuccess) return fail(ctx, BETTY_ECUDA, "%s: %s", #expr, cudaGetErrorString(_e)); \
    } while (0)

static betty_status check_launch(betty_ctx* c) {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return fail(c, BETTY_ECUDA, "kernel launch: %s", cudaGetErrorString(e));
    return BETTY_OK;
}

// synchronise and translate device-side error flags
static betty_status sync_check(betty_ctx* c, cudaStream_t s) {
    CUDA_OK(c, cudaStreamSynchronize(s));
    int flags = 0;
    CUDA_OK(c, cudaMemcpy(&flags, c->dev_err, sizeof(int), cudaMemcpyDeviceToHost));
    if (flags) {
        CUDA_OK(c, cudaMemset(c->dev_err, 0, sizeof(int)));
        if (flags & DEVERR_BAD_PART) return fail(c, BETTY_EINVAL, "part[] has a value outside [0, K)");
        if (flags & DEVERR_DUP_EDGE) return fail(c, BETTY_EINVAL, "a row repeats a source (A must be binary)");
        if (flags & DEVERR_OVERFLOW) return fail(c, BETTY_EOVERFLOW, "a size exceeded a capacity / kernel limit");
    }
    return check_launch(c);
}

// ----------------------------------------------------------------- ctx
extern "C" const char* betty_version(void) { return "betty-b200 0.1 (sm_100a)"; }

extern "C" betty_status betty_ctx_create(int device, betty_alloc_fn alloc, betty_free_fn dealloc, void* user,
                                         betty_ctx** out) {
    if (!out) return BETTY_EINVAL;
    *out = nullptr;
    if ((alloc == nullptr) != (dealloc == nullptr)) return BETTY_EINVAL;
    if (cudaSetDevice(device) != cudaSuccess) return BETTY_ECUDA;
    betty_ctx* c = new (std::nothrow) betty_ctx();
    if (!c) return BETTY_ENOMEM;
    c->device = device;
    c->alloc = alloc;
    c->dealloc = dealloc;
    c->user = user;
    cudaDeviceGetAttribute(&c->num_sms, cudaDevAttrMultiProcessorCount, device);
    // per lane: counters [64 unsigned] + loss partials [2048 double], big-segment list; device error flags
    bool ok = cudaMalloc(&c->dev_err, 16) == cudaSuccess;
    for (auto& ln : c->lanes) {
        ln.big_list_cap = 1 << 20;
        ok = ok && cudaMalloc(&ln.counters, 64 * 4 + 2048 * 8) == cudaSuccess &&
             cudaMalloc(&ln.big_count, 16) == cudaSuccess &&
             cudaMalloc(&ln.big_list, sizeof(int64_t) * ln.big_list_cap) == cudaSuccess;
        if (ok) { cudaMemset(ln.counters, 0, 64 * 4 + 2048 * 8); cudaMemset(ln.big_count, 0, 16); }
    }
    if (!ok) { betty_ctx_destroy(c); return BETTY_ENOMEM; }
    init_kernel_attrs();
    const char* no_tc = getenv("BETTY_NO_TC");
    c->use_tc = !(no_tc && no_tc[0] == '1') && tc_available();
    const char* simt = getenv("BETTY_FP32_SIMT");
    c->fp32_tc = !(simt && simt[0] == '1');
    cudaMemset(c->dev_err, 0, 16);
    cudaDeviceSynchronize();
    *out = c;
    return BETTY_OK;
}

extern "C" void betty_ctx_destroy(betty_ctx* c) {
    if (!c) return;
    cudaDeviceSynchronize();
    for (auto& ln : c->lanes) {
        if (ln.scan_status) ctx_free(c, ln.scan_status, 0);
        cudaFree(ln.counters);
        cudaFree(ln.big_count);
        cudaFree(ln.big_list);
    }
    for (void* p : c->retired) ctx_free(c, p, 0);
    cudaFree(c->dev_err);
    cudaDeviceSynchronize();
    delete c;
}

extern "C" const char* betty_last_error(const betty_ctx* c) { return c ? c->err.c_str() : "null ctx"; }

extern "C" int64_t betty_num_params(const betty_model* m) {
    ModelCfg cfg;
    if (!m || !make_model_cfg(m->L, m->aggr, m->gemm, m->feat_dtype, m->dims, &cfg)) return -1;
    return cfg.n_params;
}

// ------------------------------------------------------------ extraction
struct Arena {
    betty_ctx* c;
    cudaStream_t s;
    std::vector<void*> owned;
    int64_t bytes = 0;
    bool ok = true;
    template <typename T> T* get(int64_t n) {
        const int64_t b = std::max<int64_t>(n, 1) * (int64_t)sizeof(T);
        void* p = ctx_alloc(c, (size_t)b, s);
        if (!p) ok = false; else { owned.push_back(p); bytes += b; }
        return (T*)p;
    }
    void release() { for (void* p : owned) ctx_free(c, p, s); owned.clear(); }
};

struct ExtractSet {             // arenas of one extraction configuration (c slots, given capacities)
    std::vector<ExtractLayer> layers;
    ExtractScratch sc{};
    int64_t* cnt_all = nullptr; // [L*4]
};

static bool alloc_extract(Arena& A, int L, const ExtractFull* full, int64_t n_out, int32_t c,
                          const std::vector<int64_t>& cap_dst, const std::vector<int64_t>& cap_src,
                          const std::vector<int64_t>& cap_e, uint32_t csc_mask, ExtractSet* X) {
    X->layers.assign(L, ExtractLayer{});
    X->cnt_all = A.get<int64_t>(L * 4);
    int64_t max_src = 1;
    for (int l = 0; l < L; ++l) {
        ExtractLayer& B = X->layers[l];
        B.cap_dst = std::max<int64_t>(cap_dst[l], 1);
        B.cap_src = std::max<int64_t>(cap_src[l], 1);
        B.cap_e = std::max<int64_t>(cap_e[l], 1);
        B.indptr = A.get<int64_t>(B.cap_dst + 1);
        B.indices = A.get<int32_t>(B.cap_e);
        B.src_pos = A.get<int32_t>(B.cap_src);
        B.src_gid = A.get<int32_t>(B.cap_src);
        B.src_mb = A.get<int32_t>(B.cap_src);
        if (csc_mask >> l & 1) {
            B.t_indptr = A.get<int64_t>(B.cap_src + 1);
            B.t_indices = A.get<int32_t>(B.cap_e);
        }
        B.cnt = X->cnt_all + 4 * l;
        B.mb_src_off = A.get<int64_t>(c + 1);
        if (l + 1 < L) B.order_tab = A.get<int64_t>(2 * (ORDER_TAB_MAX + 1) + 1);
        max_src = std::max(max_src, std::max(full[l].n_src, B.cap_src));
    }
    int64_t max_full = 1;
    for (int l = 0; l < L; ++l) max_full = std::max(max_full, full[l].n_src);
    const int64_t W = (max_full + 31) / 32 + 1;
    const int64_t nchunks = (n_out + SEL_CHUNK - 1) / SEL_CHUNK + 1;
    ExtractScratch& sc = X->sc;
    sc.dstbits = A.get<uint32_t>(c * W);
    sc.newbits = A.get<uint32_t>(c * W);
    for (int l = 0; l < L; ++l) sc.nrank[l] = A.get<uint2>(c * ((full[l].n_src + 31) / 32));
    sc.drank_top = A.get<uint2>(c * ((full[L - 1].n_src + 31) / 32));
    sc.wordoff = A.get<int64_t>(c * W + 1);
    sc.tcnt = A.get<int32_t>(max_src);
    sc.ndeg = A.get<int32_t>(max_src);
    sc.sel_cnt = A.get<int64_t>(c * nchunks);
    sc.sel_off = A.get<int64_t>(c * nchunks + 1);
    sc.top_dst_pos = A.get<int32_t>(std::max<int64_t>(n_out, 1));
    sc.top_row_mb = A.get<int32_t>(std::max<int64_t>(n_out, 1));
    sc.top_dst_off = A.get<int64_t>(c + 1);
    if (!A.ok) return false;
    cudaMemsetAsync(sc.dstbits, 0, sizeof(uint32_t) * c * W, A.s);
    cudaMemsetAsync(sc.newbits, 0, sizeof(uint32_t) * c * W, A.s);
    cudaMemsetAsync(X->cnt_all, 0, sizeof(int64_t) * L * 4, A.s);
    return true;
}

static betty_status check_full(betty_ctx* c, const betty_block* full, int32_t L) {
    if (!full || L < 1 || L > 16) return fail(c, BETTY_EINVAL, "full blocks / L invalid");
    for (int l = 0; l < L; ++l) {
        const betty_block& b = full[l];
        if (!b.indptr || (b.n_edges > 0 && !b.indices) || (b.n_src > 0 && !b.src_gid))
            return fail(c, BETTY_EINVAL, "full block %d: null array", l);
        if (b.n_dst < 0 || b.n_src < b.n_dst || b.n_edges < 0)
            return fail(c, BETTY_EINVAL, "full block %d: bad sizes", l);
        if (b.n_src >= INT32_MAX || b.n_edges >= ((int64_t)1 << 40))
            return fail(c, BETTY_EOVERFLOW, "full block %d: sizes exceed int32 ids", l);
        if (l + 1 < L && full[l + 1].n_src != b.n_dst)
            return fail(c, BETTY_EINVAL, "block %d dst count must equal block %d src count", l, l + 1);
    }
    return BETTY_OK;
}

static std::vector<ExtractFull> to_full(const betty_block* full, int L) {
    std::vector<ExtractFull> f(L);
    for (int l = 0; l < L; ++l) f[l] = ExtractFull{full[l].n_dst, full[l].n_src, full[l].n_edges, full[l].indptr,
                                                   full[l].indices, full[l].src_gid};
    return f;
}

extern "C" betty_status betty_extract_blocks(betty_ctx* c, const betty_block* full, int32_t L, const int32_t* part,
                                             int64_t n_out, int32_t K, int32_t k, betty_block* mb,
                                             betty_stream stream) {
    if (!c) return BETTY_EINVAL;
    cudaStream_t s = (cudaStream_t)stream;
    betty_status st = check_full(c, full, L);
    if (st) return st;
    if (!mb || (n_out > 0 && !part) || K < 1 || k < 0 || k >= K || full[L - 1].n_dst != n_out)
        return fail(c, BETTY_EINVAL, "extract: bad part / K / k / n_out");
    if (!extract_limits_ok(K, 1, n_out, full[L - 1].n_edges))
        return fail(c, BETTY_EUNSUPPORTED, "extract: K > 16384, n_out >= 2^23 or >= 2^40 top-layer edges");
    std::vector<ExtractFull> F = to_full(full, L);
    std::vector<int64_t> cd(L), cs(L), ce(L);
    for (int l = 0; l < L; ++l) { cd[l] = full[l].n_dst; cs[l] = full[l].n_src; ce[l] = full[l].n_edges; }
    Arena A{c, s};
    ExtractSet X;
    int32_t* d_k = A.get<int32_t>(1);
    if (!d_k || !alloc_extract(A, L, F.data(), n_out, 1, cd, cs, ce, (1u << L) - 1, &X)) {
        A.release();
        return fail(c, BETTY_ENOMEM, "extract: allocation failed");
    }
    cudaMemcpyAsync(d_k, &k, sizeof(int32_t), cudaMemcpyHostToDevice, s);
    ExtractArgs a{};
    a.L = L; a.full = F.data(); a.part = part; a.K = K; a.ks = d_k; a.c = 1;
    a.layers = X.layers.data(); a.sc = X.sc; a.csc_mask = (1u << L) - 1;
    extract_group(c, a, s);
    std::vector<int64_t> cnt(L * 4);
    cudaMemcpyAsync(cnt.data(), X.cnt_all, sizeof(int64_t) * L * 4, cudaMemcpyDeviceToHost, s);
    st = sync_check(c, s);
    if (st) { A.release(); return st; }
    // exact-size outputs
    for (int l = 0; l < L; ++l) {
        betty_block& o = mb[l];
        memset(&o, 0, sizeof(o));
        o.n_dst = cnt[4 * l + 0]; o.n_src = cnt[4 * l + 1]; o.n_edges = cnt[4 * l + 2];
        o.indptr = (int64_t*)ctx_alloc(c, sizeof(int64_t) * (o.n_dst + 1), s);
        o.indices = (int32_t*)ctx_alloc(c, sizeof(int32_t) * std::max<int64_t>(o.n_edges, 1), s);
        o.src_pos = (int32_t*)ctx_alloc(c, sizeof(int32_t) * std::max<int64_t>(o.n_src, 1), s);
        o.src_gid = (int32_t*)ctx_alloc(c, sizeof(int32_t) * std::max<int64_t>(o.n_src, 1), s);
        o.t_indptr = (int64_t*)ctx_alloc(c, sizeof(int64_t) * (o.n_src + 1), s);
        o.t_indices = (int32_t*)ctx_alloc(c, sizeof(int32_t) * std::max<int64_t>(o.n_edges, 1), s);
        if (!o.indptr || !o.indices || !o.src_pos || !o.src_gid || !o.t_indptr || !o.t_indices) {
            betty_block_free(c, mb, l + 1);
            A.release();
            return fail(c, BETTY_ENOMEM, "extract: output allocation failed");
        }
        const ExtractLayer& B = X.layers[l];
        cudaMemcpyAsync(o.indptr, B.indptr, sizeof(int64_t) * (o.n_dst + 1), cudaMemcpyDeviceToDevice, s);
        cudaMemcpyAsync(o.indices, B.indices, sizeof(int32_t) * o.n_edges, cudaMemcpyDeviceToDevice, s);
        cudaMemcpyAsync(o.src_pos, B.src_pos, sizeof(int32_t) * o.n_src, cudaMemcpyDeviceToDevice, s);
        cudaMemcpyAsync(o.src_gid, B.src_gid, sizeof(int32_t) * o.n_src, cudaMemcpyDeviceToDevice, s);
        cudaMemcpyAsync(o.t_indptr, B.t_indptr, sizeof(int64_t) * (o.n_src + 1), cudaMemcpyDeviceToDevice, s);
        cudaMemcpyAsync(o.t_indices, B.t_indices, sizeof(int32_t) * o.n_edges, cudaMemcpyDeviceToDevice, s);
    }
    A.release();
    return sync_check(c, s);
}

extern "C" void betty_block_free(betty_ctx* c, betty_block* b, int32_t L) {
    if (!c || !b) return;
    for (int l = 0; l < L; ++l) {
        ctx_free(c, b[l].indptr, 0); ctx_free(c, b[l].indices, 0); ctx_free(c, b[l].src_pos, 0);
        ctx_free(c, b[l].src_gid, 0); ctx_free(c, b[l].t_indptr, 0); ctx_free(c, b[l].t_indices, 0);
        memset(&b[l], 0, sizeof(betty_block));
    }
}

// ------------------------------------------------------------------ REG
struct RegBufs {
    RegArgs a{};
    int64_t* cnt = nullptr;     // [3] n_rows, n_cols, n_edges
    int32_t* col = nullptr;
    int32_t* w = nullptr;
    int64_t ub_cap = 0, nnz_cap = 0;
};

// REG rows [r0, r1) of the output block ob (the CSC always covers the whole block); uploads the
// device counts {rows of the slice, n_src, n_edges, -, n_dst} on stream s.
static bool alloc_reg_phase1(Arena& A, const betty_block* ob, int64_t r0, int64_t r1, RegBufs* R, cudaStream_t s) {
    const int64_t n = r1 - r0, ns = ob->n_src, E = ob->n_edges;
    R->cnt = A.get<int64_t>(5);
    RegArgs& a = R->a;
    a.indptr = ob->indptr + r0; a.idx = ob->indices;
    a.full_indptr = ob->indptr; a.full_rows_cap = std::max<int64_t>(ob->n_dst, 1); a.row0 = r0;
    a.n_rows_dev = R->cnt; a.n_cols_dev = R->cnt + 1; a.n_edges_dev = R->cnt + 2; a.n_full_rows_dev = R->cnt + 4;
    a.rows_cap = std::max<int64_t>(n, 1); a.cols_cap = std::max<int64_t>(ns, 1); a.edges_cap = std::max<int64_t>(E, 1);
    if (R->cnt) {
        const int64_t h[5] = {n, ns, E, 0, ob->n_dst};
        cudaMemcpyAsync(R->cnt, h, sizeof(h), cudaMemcpyHostToDevice, s);
        cudaStreamSynchronize(s);       // h is a host stack array
    }
    a.t_indptr = A.get<int64_t>(ns + 1);
    a.t_idx = A.get<int32_t>(E);
    a.tcnt = A.get<int32_t>(ns);
    a.ub = A.get<int64_t>(n);
    a.off = A.get<int64_t>(n + 1);
    a.ub_total_dev = R->cnt + 3;
    a.row_nnz = A.get<int64_t>(n);
    // hub-row scratch: a bitmap over the output ids and its popcount prefix per CTA of k_reg_rows_cta
    a.hub_words = (ob->n_dst + 31) / 32 + 1;
    a.hub_bits = A.get<uint32_t>(a.hub_words * A.c->num_sms);
    a.hub_pre = A.get<int32_t>(a.hub_words * A.c->num_sms);
    return A.ok;
}

extern "C" betty_status betty_reg_build(betty_ctx* c, const betty_block* ob, betty_csr* reg, betty_stream stream) {
    if (!c) return BETTY_EINVAL;
    if (!ob) return fail(c, BETTY_EINVAL, "reg: null argument");
    return betty_reg_build_rows(c, ob, 0, ob->n_dst, reg, stream);
}

extern "C" betty_status betty_reg_build_rows(betty_ctx* c, const betty_block* ob, int64_t row0, int64_t row1,
                                             betty_csr* reg, betty_stream stream) {
    if (!c) return BETTY_EINVAL;
    cudaStream_t s = (cudaStream_t)stream;
    if (!ob || !reg || !ob->indptr || (ob->n_edges > 0 && !ob->indices) || ob->n_dst < 0)
        return fail(c, BETTY_EINVAL, "reg: null argument");
    if (row0 < 0 || row1 < row0 || row1 > ob->n_dst) return fail(c, BETTY_EINVAL, "reg: bad row range");
    if (ob->n_src >= INT32_MAX || ob->n_dst >= INT32_MAX) return fail(c, BETTY_EOVERFLOW, "reg: sizes exceed int32");
    memset(reg, 0, sizeof(*reg));
    Arena A{c, s};
    RegBufs R;
    if (!alloc_reg_phase1(A, ob, row0, row1, &R, s)) { A.release(); return fail(c, BETTY_ENOMEM, "reg: allocation failed"); }
    reg_phase1(c, R.a, s);
    int64_t ub_total = 0;
    cudaMemcpyAsync(&ub_total, R.a.ub_total_dev, sizeof(int64_t), cudaMemcpyDeviceToHost, s);
    betty_status st = sync_check(c, s);
    if (st) { A.release(); return st; }
    R.a.tcol = A.get<int32_t>(ub_total);
    R.a.tw = A.get<int32_t>(ub_total);
    reg->indptr = (int64_t*)ctx_alloc(c, sizeof(int64_t) * (row1 - row0 + 1), s);
    R.a.out_indptr = reg->indptr;
    int64_t* nnz_dev = A.get<int64_t>(1);
    R.a.nnz_total_dev = nnz_dev;
    if (!A.ok || !reg->indptr) { A.release(); ctx_free(c, reg->indptr, s); reg->indptr = nullptr;
                                 return fail(c, BETTY_ENOMEM, "reg: allocation failed"); }
    reg_phase2(c, R.a, s);
    int64_t nnz = 0;
    cudaMemcpyAsync(&nnz, nnz_dev, sizeof(int64_t), cudaMemcpyDeviceToHost, s);
    st = sync_check(c, s);
    if (st) { A.release(); ctx_free(c, reg->indptr, s); reg->indptr = nullptr;
              return st == BETTY_EOVERFLOW ? fail(c, BETTY_EUNSUPPORTED, "reg: a row has more than 32768 candidate products") : st; }
    reg->col = (int32_t*)ctx_alloc(c, sizeof(int32_t) * std::max<int64_t>(nnz, 1), s);
    reg->w = (int32_t*)ctx_alloc(c, sizeof(int32_t) * std::max<int64_t>(nnz, 1), s);
    if (!reg->col || !reg->w) { A.release(); betty_csr_free(c, reg); return fail(c, BETTY_ENOMEM, "reg: allocation failed"); }
    reg_phase3(c, R.a, reg->col, reg->w, nnz, s);
    reg->n = row1 - row0;
    reg->nnz = nnz;
    A.release();
    return sync_check(c, s);
}

extern "C" void betty_csr_free(betty_ctx* c, betty_csr* r) {
    if (!c || !r) return;
    ctx_free(c, r->indptr, 0); ctx_free(c, r->col, 0); ctx_free(c, r->w, 0);
    memset(r, 0, sizeof(*r));
}

// ---------------------------------------------------- standalone SAGE
struct betty_saved {
    ModelCfg m;
    SageBufs b;
    std::vector<BlockView> v;
    int64_t* cnt = nullptr;
    std::vector<int64_t> hcnt;
};

static betty_status model_from(betty_ctx* c, const betty_model* model, ModelCfg* m) {
    if (!model || !make_model_cfg(model->L, model->aggr, model->gemm, model->feat_dtype, model->dims, m))
        return fail(c, BETTY_EINVAL, "invalid betty_model (L in [1,16], dims >= 1, classes <= 256)");
    return BETTY_OK;
}

static betty_status check_feats(betty_ctx* c, const ModelCfg& m, const void* feats, int64_t ld) {
    const int vw = m.feat_bf16 ? 8 : 4;
    if (!feats) return fail(c, BETTY_EINVAL, "feats is null");
    if (ld < (m.dims[0] + vw - 1) / vw * vw || ld % vw)
        return fail(c, BETTY_EINVAL, "ld_feats must be >= dims[0] rounded up to and a multiple of %d", vw);
    if (((uintptr_t)feats) % 16) return fail(c, BETTY_EINVAL, "feats must be 16-byte aligned");
    return BETTY_OK;
}

extern "C" betty_status betty_sage_fwd(betty_ctx* c, const betty_model* model, const float* params,
                                       const betty_block* mb, const void* feats, int64_t ld_feats,
                                       betty_saved** saved, float* logits, betty_stream stream) {
    if (!c) return BETTY_EINVAL;
    cudaStream_t s = (cudaStream_t)stream;
    ModelCfg m;
    betty_status st = model_from(c, model, &m);
    if (st) return st;
    if (!params || !mb || !saved) return fail(c, BETTY_EINVAL, "sage_fwd: null argument");
    if ((st = check_feats(c, m, feats, ld_feats))) return st;
    for (int l = 0; l < m.L; ++l) {
        if (!mb[l].indptr || (mb[l].n_edges && !mb[l].indices) || !mb[l].src_gid)
            return fail(c, BETTY_EINVAL, "sage_fwd: block %d has null arrays", l);
        if (m.needs_csc(l) && (!mb[l].t_indptr || (mb[l].n_edges && !mb[l].t_indices)))
            return fail(c, BETTY_EINVAL, "sage_fwd: block %d needs its CSC", l);
        if (l + 1 < m.L && mb[l + 1].n_src != mb[l].n_dst)
            return fail(c, BETTY_EINVAL, "sage_fwd: block %d dst count != block %d src count", l, l + 1);
    }
    betty_saved* sv = new (std::nothrow) betty_saved();
    if (!sv) return BETTY_ENOMEM;
    sv->m = m;
    sv->hcnt.assign(4 * m.L, 0);
    std::vector<int64_t> cd(m.L), cs(m.L);
    for (int l = 0; l < m.L; ++l) {
        sv->hcnt[4 * l] = mb[l].n_dst; sv->hcnt[4 * l + 1] = mb[l].n_src; sv->hcnt[4 * l + 2] = mb[l].n_edges;
        cd[l] = mb[l].n_dst; cs[l] = mb[l].n_src;
    }
    sv->cnt = (int64_t*)ctx_alloc(c, sizeof(int64_t) * 4 * m.L, s);
    if (!sv->cnt || !sage_alloc(c, m, cd, cs, &sv->b, s)) {
        betty_saved_free(c, sv);
        return fail(c, BETTY_ENOMEM, "sage_fwd: allocation failed");
    }
    cudaMemcpyAsync(sv->cnt, sv->hcnt.data(), sizeof(int64_t) * 4 * m.L, cudaMemcpyHostToDevice, s);
    sv->v.resize(m.L);
    for (int l = 0; l < m.L; ++l)
        sv->v[l] = BlockView{mb[l].indptr, mb[l].indices, mb[l].t_indptr, mb[l].t_indices, mb[l].src_gid,
                             sv->cnt + 4 * l, std::max<int64_t>(mb[l].n_dst, 1), std::max<int64_t>(mb[l].n_src, 1),
                             std::max<int64_t>(mb[l].n_edges, 1)};
    sage_prep(c, m, sv->b, params, s);
    sage_forward(c, m, sv->b, sv->v.data(), feats, ld_feats, s);
    if (logits && mb[m.L - 1].n_dst > 0)
        cudaMemcpy2DAsync(logits, sizeof(float) * m.dims[m.L], sv->b.logits, sizeof(float) * m.layers[m.L - 1].ld_out,
                          sizeof(float) * m.dims[m.L], mb[m.L - 1].n_dst, cudaMemcpyDeviceToDevice, s);
    if ((st = check_launch(c))) { betty_saved_free(c, sv); return st; }
    *saved = sv;
    return BETTY_OK;
}

extern "C" betty_status betty_sage_bwd(betty_ctx* c, const betty_model* model, const float* params,
                                       const betty_block* mb, const betty_saved* saved, const int32_t* labels,
                                       float loss_scale, float* grad_accum, float* loss_accum, betty_stream stream) {
    if (!c) return BETTY_EINVAL;
    cudaStream_t s = (cudaStream_t)stream;
    if (!saved || !params || !labels || !grad_accum || !loss_accum || !mb)
        return fail(c, BETTY_EINVAL, "sage_bwd: null argument");
    ModelCfg m;
    betty_status st = model_from(c, model, &m);
    if (st) return st;
    if (m.n_params != saved->m.n_params || m.L != saved->m.L) return fail(c, BETTY_EINVAL, "sage_bwd: model mismatch");
    betty_saved* sv = const_cast<betty_saved*>(saved);
    sage_prep(c, sv->m, sv->b, params, s);
    sage_loss(c, sv->m, sv->b, sv->v.data(), labels, loss_scale, loss_accum, s);
    sage_backward(c, sv->m, sv->b, sv->v.data(), nullptr, 0, grad_accum, s);
    return check_launch(c);
}

extern "C" void betty_saved_free(betty_ctx* c, betty_saved* sv) {
    if (!c || !sv) return;
    sage_free(c, &sv->b, 0);
    ctx_free(c, sv->cnt, 0);
    delete sv;
}

// ------------------------------------------------------------- plan / step
struct betty_plan {
    ModelCfg m;
    int L = 0;
    int32_t K = 0, c = 1;
    int flags = 0;
    int64_t n_out = 0;
    const int32_t* part = nullptr;
    std::vector<ExtractFull> full;
    std::vector<std::vector<int32_t>> groups;
    int32_t* d_ks = nullptr;
    Arena* arena = nullptr;
    Arena* reg_arena = nullptr;   // the in-step REG's buffers (re-sized by betty_plan_set_reg_rows)
    ExtractSet X;
    uint32_t csc_mask = 0;
    // BETTY_PLAN_FRESH: per layer in csc_mask, the device counts and scratch of the in-step rebuild of
    // the full-batch CSC
    std::vector<int64_t*> fcsc_cnt;
    std::vector<int32_t*> fcsc_tmp;
    bool lean0 = false;           // the step extracts layer 0 lean (extract.h ExtractArgs::lean0)
    SageBufs sb;
    FeatShards shards;            // layer-0 feature table sharded by rows (betty_plan_set_feature_shards)
    std::vector<BlockView> views;
    // REG inside the step
    bool with_reg = false;
    RegBufs R;
    const betty_block* reg_src = nullptr;
    betty_block reg_block{};
    // side stream: the REG rebuild overlaps the rest of the step (it shares no data with it)
    cudaStream_t side = nullptr;
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    // graph
    cudaGraphExec_t gexec = nullptr;
    cudaStream_t cap_stream = nullptr;
    const void* key[9] = {};
    betty_plan_info info{};
    Probe probe;
};

// Where the REG rebuild forks onto its side stream: 0 at the start of the step (beside the
// extraction), 1 after the first group's extraction (beside the aggregation / GEMMs), 2 (default)
// before its backward.  Measured on C3, two runs each: 4.100 / 4.115 ms (fork 0) against 4.132 / 4.129
// (fork 2), 8-rank share 0.686 against 0.698 ms; fork 1 4.25 ms.  Fork 0 is 0.5 % faster but folds the
// REG into the extraction's site time (0.77 instead of 0.51 ms), so the default keeps the sites apart.
static int reg_fork_point() {
    static const int v = getenv("BETTY_REG_FORK") ? atoi(getenv("BETTY_REG_FORK")) : 2;
    return v;
}

static void step_body(betty_ctx* c, betty_plan* p, const float* params, const void* feats, int64_t ld_feats,
                      const int32_t* labels, float scale, float* grad, float* loss, cudaStream_t s) {
    Probe* pr = p->sb.probe;
    if (pr) pr->used = 0;
    auto fork_reg = [&]() {     // REG on the side stream with its own primitive scratch (lane 1)
        cudaEventRecord(p->ev_fork, s);
        cudaStreamWaitEvent(p->side, p->ev_fork, 0);
        c->lane = 1;
        if (pr) pr->begin(PROBE_REG, p->side);
        reg_phase1(c, p->R.a, p->side);
        reg_phase2(c, p->R.a, p->side);
        reg_phase3(c, p->R.a, p->R.col, p->R.w, p->R.nnz_cap, p->side);
        if (pr) pr->end(PROBE_REG, p->side);
        c->lane = 0;
        cudaEventRecord(p->ev_join, p->side);
    };
    // FRESH: the lean layer 0 reads src_gid[nbr[e]] directly (ExtractArgs::egid_direct) instead of a
    // rebuilt full-batch edge -> gid array (one pass over the full batch's 20 M edges less per step)
    if (p->flags & BETTY_PLAN_FRESH) {        // full-batch CSCs from the current block buffers
        for (int l = 0; l < p->L; ++l) {
            if (!(p->csc_mask >> l & 1)) continue;
            const ExtractFull& fb = p->full[l];
            csr_transpose(c, fb.indptr, fb.nbr, p->fcsc_cnt[l], p->fcsc_cnt[l] + 1, p->fcsc_cnt[l] + 2,
                          std::max<int64_t>(fb.n_dst, 1), std::max<int64_t>(fb.n_src, 1),
                          std::max<int64_t>(fb.n_edges, 1), (int64_t*)fb.t_indptr, (int32_t*)fb.t_nbr,
                          p->fcsc_tmp[l], l == p->L - 1, s);
        }
    }
    const int fp = p->groups.empty() ? 0 : reg_fork_point();
    if (p->with_reg && fp == 0) fork_reg();
    sage_prep(c, p->m, p->sb, params, s);
    for (size_t g = 0; g < p->groups.size(); ++g) {
        ExtractArgs a{};
        a.L = p->L; a.full = p->full.data(); a.part = p->part; a.K = p->K;
        a.ks = p->d_ks + g * p->c; a.c = (int32_t)p->groups[g].size();
        a.layers = p->X.layers.data(); a.sc = p->X.sc; a.csc_mask = p->csc_mask;
        a.lean0 = p->lean0;
        a.egid_direct = (p->flags & BETTY_PLAN_FRESH) != 0;
        if (pr) pr->begin(PROBE_EXTRACT, s);
        extract_group(c, a, s);
        if (pr) pr->end(PROBE_EXTRACT, s);
        if (p->with_reg && fp == 1 && g == 0) fork_reg();
        sage_forward(c, p->m, p->sb, p->views.data(), feats, ld_feats, s);
        sage_loss(c, p->m, p->sb, p->views.data(), labels, scale, loss, s);
        if (p->with_reg && fp == 2 && g == 0) fork_reg();
        sage_backward(c, p->m, p->sb, p->views.data(), feats, ld_feats, grad, s);
    }
    if (p->with_reg) cudaStreamWaitEvent(s, p->ev_join, 0);   // join
}

// Count-only extraction of micro-batches ks[0..n) of a K-way partition, each alone with
// full-batch capacities (one synchronisation per micro-batch): sz[i][3l + {0,1,2}] =
// n_dst, n_src, n_edges of layer l.  Sizes plans and the memory estimate (§4.4).
static betty_status size_micro_batches(betty_ctx* c, const ExtractFull* F, const betty_block* full, int L,
                                       const int32_t* part, int64_t n_out, int32_t K, const int32_t* ks, int32_t n,
                                       std::vector<std::vector<int64_t>>* sz, cudaStream_t s) {
    sz->assign(n, std::vector<int64_t>(3 * L, 0));
    std::vector<int64_t> fd(L), fs(L), fe(L);
    for (int l = 0; l < L; ++l) { fd[l] = full[l].n_dst; fs[l] = full[l].n_src; fe[l] = full[l].n_edges; }
    Arena A{c, s};
    ExtractSet X;
    int32_t* d_k = A.get<int32_t>(std::max(1, n));
    if (!d_k || !alloc_extract(A, L, F, n_out, 1, fd, fs, fe, 0, &X)) {
        A.release();
        return fail(c, BETTY_ENOMEM, "sizing allocation failed");
    }
    if (n) cudaMemcpyAsync(d_k, ks, sizeof(int32_t) * n, cudaMemcpyHostToDevice, s);
    std::vector<int64_t> h(4 * L);
    betty_status st = BETTY_OK;
    for (int i = 0; i < n && !st; ++i) {
        ExtractArgs a{};
        a.L = L; a.full = F; a.part = part; a.K = K; a.ks = d_k + i; a.c = 1;
        a.layers = X.layers.data(); a.sc = X.sc; a.csc_mask = 0;
        extract_group(c, a, s);
        cudaMemcpyAsync(h.data(), X.cnt_all, sizeof(int64_t) * 4 * L, cudaMemcpyDeviceToHost, s);
        if ((st = sync_check(c, s))) break;
        for (int l = 0; l < L; ++l)
            for (int q = 0; q < 3; ++q) (*sz)[i][3 * l + q] = h[4 * l + q];
    }
    A.release();
    return st;
}

__global__ void k_max_deg(const int64_t* __restrict__ indptr, int64_t n, int* out) {
    int mx = 0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        { const int64_t d = indptr[i + 1] - indptr[i]; mx = max(mx, d > 1000000 ? 1000000 : (int)d); }
    atomicMax(out, mx);
}

// Size and allocate the in-step REG of output rows [r0, r1) (phases 1-2 run once here, synchronising).
static betty_status plan_reg_setup(betty_ctx* c, betty_plan* p, const betty_block* ob, int64_t r0, int64_t r1,
                                   cudaStream_t s) {
    // the REG's buffers live in their own arena: a new row share releases the previous share's
    // buffers first (set_reg_rows used to leak the all-rows REG scratch in the plan arena)
    if (p->reg_arena) { p->reg_arena->s = s; p->reg_arena->release(); p->reg_arena->bytes = 0; p->reg_arena->ok = true; }
    else p->reg_arena = new Arena{c, s};
    p->with_reg = false;
    Arena& A = *p->reg_arena;
    c->lane = 1;            // size the side lane's scan scratch with the REG's own calls
    RegBufs R;
    if (!alloc_reg_phase1(A, ob, r0, r1, &R, s)) { c->lane = 0; return fail(c, BETTY_ENOMEM, "plan: REG alloc"); }
    reg_phase1(c, R.a, s);
    int64_t ub = 0;
    cudaMemcpyAsync(&ub, R.a.ub_total_dev, sizeof(int64_t), cudaMemcpyDeviceToHost, s);
    betty_status st = sync_check(c, s);
    if (st) { c->lane = 0; return st; }
    R.ub_cap = ub;
    R.a.tcol = A.get<int32_t>(ub);
    R.a.tw = A.get<int32_t>(ub);
    R.a.out_indptr = A.get<int64_t>(r1 - r0 + 1);
    R.a.nnz_total_dev = A.get<int64_t>(1);
    if (!A.ok) { c->lane = 0; return fail(c, BETTY_ENOMEM, "plan: REG alloc"); }
    reg_phase2(c, R.a, s);
    int64_t nnz = 0;
    cudaMemcpyAsync(&nnz, R.a.nnz_total_dev, sizeof(int64_t), cudaMemcpyDeviceToHost, s);
    if ((st = sync_check(c, s))) { c->lane = 0; return st; }
    R.nnz_cap = nnz;
    R.col = A.get<int32_t>(nnz);
    R.w = A.get<int32_t>(nnz);
    c->lane = 0;
    if (!A.ok) return fail(c, BETTY_ENOMEM, "plan: REG alloc");
    // The output block's CSC (built and duplicate-checked by phase 1 above) belongs to the plan's
    // full batch, like the extraction's full-batch CSC: the step's rebuild reuses it and runs the
    // SpGEMM proper (expansion, sort, run-length encode, compaction) over the rank's rows.
    R.a.csc_ready = !(p->flags & BETTY_PLAN_FRESH);    // FRESH: the step rebuilds it from the block
    // FRESH with the output block's full-batch CSC among the step's rebuilt CSCs (same block, same
    // transpose, duplicate-checked, rebuilt on the main stream before the REG forks): the REG reads
    // that one instead of transposing the block a second time (the e2e step's duplicate ~0.2 ms)
    if ((p->flags & BETTY_PLAN_FRESH) && (p->csc_mask >> (p->L - 1) & 1) && p->full[p->L - 1].t_indptr &&
        ob == &p->reg_block) {
        R.a.t_indptr = (int64_t*)p->full[p->L - 1].t_indptr;
        R.a.t_idx = (int32_t*)p->full[p->L - 1].t_nbr;
        R.a.csc_ready = true;
    }
    p->R = R;
    p->with_reg = true;
    p->info.reg_nnz = nnz;
    p->info.arena_bytes = p->arena->bytes + A.bytes + p->sb.bytes;
    return BETTY_OK;
}

extern "C" betty_status betty_plan_set_feature_shards(betty_ctx* c, betty_plan* p, int32_t R, const void* const* base,
                                                     int64_t rows_per_shard) {
    if (!c) return BETTY_EINVAL;
    if (!p || R < 0 || R > MAX_SHARDS || (R > 0 && (!base || rows_per_shard < 1)))
        return fail(c, BETTY_EINVAL, "plan_set_feature_shards: bad arguments");
    if (R > 0 && (p->m.layers[0].kind != KIND_AGG))
        return fail(c, BETTY_EUNSUPPORTED, "plan_set_feature_shards: only an aggregate-first layer 0 (mean / sum, "
                                           "F_in <= F_out) gathers from a sharded table");
    for (int r = 0; r < R; ++r)
        if (!base[r] || ((uintptr_t)base[r] & 15)) return fail(c, BETTY_EINVAL, "plan_set_feature_shards: bad base");
    FeatShards sh;
    sh.R = R;
    sh.rps = rows_per_shard;
    for (int r = 0; r < R; ++r) sh.base[r] = base[r];
    p->shards = sh;
    p->sb.shards = R > 0 ? &p->shards : nullptr;
    if (p->gexec) { cudaGraphExecDestroy(p->gexec); p->gexec = nullptr; }     // kernel arguments change
    return BETTY_OK;
}

// ------------------------------------------ device buffers shared across processes (CUDA IPC)
extern "C" betty_status betty_dev_alloc(betty_ctx* c, size_t bytes, void** out) {
    if (!c || !out) return BETTY_EINVAL;
    *out = nullptr;
    cudaSetDevice(c->device);
    if (cudaMalloc(out, std::max<size_t>(bytes, 16)) != cudaSuccess) {
        cudaGetLastError();
        return fail(c, BETTY_ENOMEM, "dev_alloc: cudaMalloc failed");
    }
    return BETTY_OK;
}
extern "C" betty_status betty_dev_free(betty_ctx* c, void* p) {
    if (!c) return BETTY_EINVAL;
    if (p) cudaFree(p);
    return BETTY_OK;
}
extern "C" betty_status betty_ipc_handle(betty_ctx* c, void* dev_ptr, void* handle) {
    if (!c || !dev_ptr || !handle) return BETTY_EINVAL;
    cudaIpcMemHandle_t h;
    if (cudaIpcGetMemHandle(&h, dev_ptr) != cudaSuccess) {
        cudaGetLastError();
        return fail(c, BETTY_ECUDA, "ipc_handle: cudaIpcGetMemHandle failed (pointer from betty_dev_alloc?)");
    }
    static_assert(sizeof(h) == BETTY_IPC_HANDLE_BYTES, "IPC handle size");
    memcpy(handle, &h, sizeof(h));
    return BETTY_OK;
}
extern "C" betty_status betty_ipc_open(betty_ctx* c, const void* handle, void** dev_ptr) {
    if (!c || !handle || !dev_ptr) return BETTY_EINVAL;
    cudaIpcMemHandle_t h;
    memcpy(&h, handle, sizeof(h));
    cudaSetDevice(c->device);
    if (cudaIpcOpenMemHandle(dev_ptr, h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
        cudaGetLastError();
        return fail(c, BETTY_ECUDA, "ipc_open: cudaIpcOpenMemHandle failed");
    }
    return BETTY_OK;
}
extern "C" betty_status betty_ipc_close(betty_ctx* c, void* dev_ptr) {
    if (!c || !dev_ptr) return BETTY_EINVAL;
    if (cudaIpcCloseMemHandle(dev_ptr) != cudaSuccess) {
        cudaGetLastError();
        return fail(c, BETTY_ECUDA, "ipc_close failed");
    }
    return BETTY_OK;
}

extern "C" betty_status betty_plan_set_reg_rows(betty_ctx* c, betty_plan* p, int64_t row0, int64_t row1,
                                                betty_stream stream) {
    if (!c) return BETTY_EINVAL;
    if (!p || !p->side) return fail(c, BETTY_EINVAL, "plan_set_reg_rows: plan without BETTY_PLAN_REG");
    const betty_block* ob = &p->reg_block;
    if (row0 < 0 || row1 < row0 || row1 > ob->n_dst) return fail(c, BETTY_EINVAL, "plan_set_reg_rows: bad row range");
    cudaStream_t s = (cudaStream_t)stream;
    if (cudaStreamSynchronize(s) != cudaSuccess) return fail(c, BETTY_ECUDA, "plan_set_reg_rows: stream");
    if (p->gexec) { cudaGraphExecDestroy(p->gexec); p->gexec = nullptr; }     // buffers change: re-capture
    return plan_reg_setup(c, p, ob, row0, row1, s);
}

extern "C" betty_status betty_plan_create(betty_ctx* c, const betty_model* model, const betty_block* full, int32_t L,
                                          const int32_t* part, int64_t n_out, int32_t K, const int32_t* my_k,
                                          int32_t n_my, int32_t group, int32_t flags, betty_plan** out,
                                          betty_stream stream) {
    if (!c) return BETTY_EINVAL;
    cudaStream_t s = (cudaStream_t)stream;
    if (!out) return fail(c, BETTY_EINVAL, "plan: out is null");
    *out = nullptr;
    ModelCfg m;
    betty_status st = model_from(c, model, &m);
    if (st) return st;
    if ((st = check_full(c, full, L))) return st;
    if (L != m.L) return fail(c, BETTY_EINVAL, "plan: L != model.L");
    if (K < 1 || n_my < 0 || (n_my > 0 && !my_k) || full[L - 1].n_dst != n_out || (n_out > 0 && !part))
        return fail(c, BETTY_EINVAL, "plan: bad K / my_k / n_out / part");
    for (int i = 0; i < n_my; ++i)
        if (my_k[i] < 0 || my_k[i] >= K) return fail(c, BETTY_EINVAL, "plan: my_k[%d] out of range", i);
    // pool layers keep the argmax as a byte position when every row of the block has <= 254 edges
    // (micro-batch rows are full-batch rows; one reduction per pool layer, here at plan time): a
    // quarter of the int32 argmax bytes and memory.  The routing kernel finds u's position in each
    // row with one warp-wide load + ballot (C4: 135.4 vs 137.7 ms per step for int32 positions;
    // the first, serial search was 105 vs 63 ms).  BETTY_POOL_POS8=0 keeps int32 argmax ids.
    const bool pos8_on = !(getenv("BETTY_POOL_POS8") && atoi(getenv("BETTY_POOL_POS8")) == 0);
    if (m.aggr == BETTY_AGGR_POOL && pos8_on) {
        int* d_mx = nullptr;
        if (cudaMalloc(&d_mx, sizeof(int) * L) != cudaSuccess) return fail(c, BETTY_ENOMEM, "plan: max degree");
        cudaMemsetAsync(d_mx, 0, sizeof(int) * L, s);
        for (int l = 0; l < L; ++l)
            if (full[l].n_dst > 0)
                k_max_deg<<<(int)std::min<int64_t>((full[l].n_dst + 255) / 256, 4096), 256, 0, s>>>(
                    full[l].indptr, full[l].n_dst, d_mx + l);
        std::vector<int> mx(L, 0);
        cudaMemcpyAsync(mx.data(), d_mx, sizeof(int) * L, cudaMemcpyDeviceToHost, s);
        st = sync_check(c, s);
        cudaFree(d_mx);
        if (st) return st;
        m.pos8.assign(L, 0);
        for (int l = 0; l < L; ++l) m.pos8[l] = mx[l] <= 254;
    }
    betty_plan* p = new (std::nothrow) betty_plan();
    if (!p) return BETTY_ENOMEM;
    p->m = m; p->L = L; p->K = K; p->flags = flags; p->n_out = n_out; p->part = part;
    p->full = to_full(full, L);
    p->c = group <= 0 ? std::max(1, n_my) : std::min(group, std::max(1, n_my));
    if (!extract_limits_ok(K, p->c, n_out, full[L - 1].n_edges)) {
        delete p;
        return fail(c, BETTY_EUNSUPPORTED, "plan: K > 16384, launch group > 512, n_out >= 2^23 or >= 2^40 top-layer edges");
    }
    for (int i = 0; i < n_my; i += p->c)
        p->groups.emplace_back(my_k + i, my_k + std::min(n_my, i + p->c));
    p->csc_mask = 0;
    for (int l = 0; l < L; ++l) if (m.needs_csc(l)) p->csc_mask |= 1u << l;

    // ---- sizing pass: every micro-batch alone, full-batch capacities
    std::vector<std::vector<int64_t>> sz;
    if ((st = size_micro_batches(c, p->full.data(), full, L, part, n_out, K, my_k, n_my, &sz, s))) {
        delete p;
        return st;
    }
    std::vector<int64_t> cd(L, 1), cs(L, 1), ce(L, 1);
    p->info.L = L;
    p->info.n_groups = (int32_t)p->groups.size();
    for (size_t g = 0, i0 = 0; g < p->groups.size(); i0 += p->groups[g].size(), ++g) {
        std::vector<int64_t> sum(3 * L, 0);
        for (size_t t = 0; t < p->groups[g].size(); ++t)
            for (int q = 0; q < 3 * L; ++q) sum[q] += sz[i0 + t][q];
        for (int l = 0; l < L; ++l) {
            cd[l] = std::max(cd[l], sum[3 * l]); cs[l] = std::max(cs[l], sum[3 * l + 1]);
            ce[l] = std::max(ce[l], sum[3 * l + 2]);
            if (l < 16) {
                p->info.n_dst[l] += sum[3 * l]; p->info.n_src[l] += sum[3 * l + 1]; p->info.edges[l] += sum[3 * l + 2];
                p->info.max_group_edges[l] = ce[l];
            }
        }
    }
    for (int l = 0; l < L; ++l)
        if (cs[l] >= INT32_MAX) { delete p; return fail(c, BETTY_EOVERFLOW, "plan: group exceeds int32 ids"); }
    for (int l = 0; l + 1 < L; ++l) { cd[l] = std::max(cd[l], cs[l + 1]); cs[l + 1] = cd[l]; }

    // ---- arenas
    p->arena = new Arena{c, s};
    Arena& A = *p->arena;
    p->d_ks = A.get<int32_t>(std::max<int64_t>(1, (int64_t)p->groups.size() * p->c));
    if (!p->d_ks || !alloc_extract(A, L, p->full.data(), n_out, p->c, cd, cs, ce, p->csc_mask, &p->X) ||
        !sage_alloc(c, m, cd, cs, &p->sb, s)) {
        betty_plan_destroy(c, p);
        return fail(c, BETTY_ENOMEM, "plan: arena allocation failed");
    }
    if (m.layers[0].kind == KIND_AGG) p->X.layers[0].egid = A.get<int32_t>(ce[0]);   // layer-0 gather by gid
    // full-batch CSC of the layers whose micro-batch CSC is built every step (filtered from it)
    p->fcsc_cnt.assign(L, nullptr);
    p->fcsc_tmp.assign(L, nullptr);
    for (int l = 0; l < L; ++l) {
        if (!(p->csc_mask >> l & 1)) continue;
        const betty_block& fb = full[l];
        int64_t* fti = A.get<int64_t>(fb.n_src + 1);
        int32_t* ftn = A.get<int32_t>(fb.n_edges);
        int64_t* hc = A.get<int64_t>(4);
        int32_t* tc = A.get<int32_t>(fb.n_src);
        if (!A.ok) break;
        const int64_t h3[4] = {fb.n_dst, fb.n_src, fb.n_edges, 0};
        cudaMemcpyAsync(hc, h3, sizeof(h3), cudaMemcpyHostToDevice, s);
        ensure_scan_scratch(c, std::max(fb.n_src, fb.n_edges) + 1, s);
        csr_transpose(c, fb.indptr, fb.indices, hc, hc + 1, hc + 2, std::max<int64_t>(fb.n_dst, 1),
                      std::max<int64_t>(fb.n_src, 1), std::max<int64_t>(fb.n_edges, 1), fti, ftn, tc, false, s);
        if ((st = sync_check(c, s))) { betty_plan_destroy(c, p); return st; }
        p->full[l].t_indptr = fti;
        p->full[l].t_nbr = ftn;
        p->fcsc_cnt[l] = hc;
        p->fcsc_tmp[l] = tc;
    }
    // lean layer 0 (aggregate-first layer 0 without a CSC: its features are gathered by global id, no
    // kernel reads its src list): the full batch's edge -> source gid array, once per plan
    static const bool full_extract = getenv("BETTY_FULL_EXTRACT") && atoi(getenv("BETTY_FULL_EXTRACT"));
    p->lean0 = !full_extract && L >= 2 && m.layers[0].kind == KIND_AGG && !(p->csc_mask & 1) && p->X.layers[0].egid;
    if (p->lean0 && A.ok) {
        int32_t* fe = A.get<int32_t>(full[0].n_edges);
        if (fe) {
            full_egid(c, full[0].indices, full[0].src_gid, full[0].n_edges, fe, s);
            p->full[0].egid = fe;
        } else {
            p->lean0 = false;
        }
    }
    if (!A.ok) {
        betty_plan_destroy(c, p);
        return fail(c, BETTY_ENOMEM, "plan: arena allocation failed");
    }
    std::vector<int32_t> hk((size_t)p->groups.size() * p->c, 0);
    for (size_t g = 0; g < p->groups.size(); ++g)
        for (size_t t = 0; t < p->groups[g].size(); ++t) hk[g * p->c + t] = p->groups[g][t];
    if (!hk.empty()) cudaMemcpyAsync(p->d_ks, hk.data(), sizeof(int32_t) * hk.size(), cudaMemcpyHostToDevice, s);
    p->views.resize(L);
    for (int l = 0; l < L; ++l) {
        const ExtractLayer& B = p->X.layers[l];
        p->views[l] = BlockView{B.indptr, B.indices, B.t_indptr, B.t_indices, B.src_gid, B.cnt, B.cap_dst, B.cap_src,
                                B.cap_e, B.egid, B.order_tab,
                                n_my > 0 ? std::max<int64_t>(1, p->info.n_src[std::min(l, 15)] / n_my) : 1};
    }
    // scan scratch for the largest scan of a step (never grows inside a capture)
    {
        int64_t mx = 0;
        for (int l = 0; l < L; ++l) mx = std::max({mx, cd[l], cs[l], ce[l]});
        int64_t maxfull = 1;
        for (int l = 0; l < L; ++l) maxfull = std::max(maxfull, full[l].n_src);
        mx = std::max(mx, (int64_t)p->c * ((maxfull + 31) / 32 + 1));
        mx = std::max(mx, (int64_t)p->c * ((n_out + SEL_CHUNK - 1) / SEL_CHUNK + 1));
        ensure_scan_scratch(c, mx, s);
    }
    // ---- REG inside the step (once here to size its buffers): all rows until betty_plan_set_reg_rows
    if (flags & BETTY_PLAN_REG) {
        // the REG shares no data with the rest of the step: its side stream gets the LOWEST priority
        // and the step's capture stream the highest, so the block scheduler fills the main path's
        // SMs first and the REG runs in the gaps (tails, latency-bound phases)
        int prio_lo = 0, prio_hi = 0;
        cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
        if (cudaStreamCreateWithPriority(&p->side, cudaStreamNonBlocking, prio_lo) != cudaSuccess ||
            cudaEventCreateWithFlags(&p->ev_fork, cudaEventDisableTiming) != cudaSuccess ||
            cudaEventCreateWithFlags(&p->ev_join, cudaEventDisableTiming) != cudaSuccess) {
            betty_plan_destroy(c, p);
            return fail(c, BETTY_ECUDA, "plan: side stream");
        }
        p->reg_block = full[L - 1];
        if ((st = plan_reg_setup(c, p, &p->reg_block, 0, full[L - 1].n_dst, s))) { betty_plan_destroy(c, p); return st; }
    }
    // ---- launches per step: capture the body once into a throw-away graph
    {
        cudaStream_t cs2;
        cudaStreamCreateWithFlags(&cs2, cudaStreamNonBlocking);
        cudaGraph_t gr;
        if (cudaStreamBeginCapture(cs2, cudaStreamCaptureModeThreadLocal) == cudaSuccess) {
            float* dummy = (float*)p->sb.partials;
            step_body(c, p, dummy, dummy, m.feat_bf16 ? 8 : 4, (const int32_t*)dummy, 1.f, dummy, dummy, cs2);
            if (cudaStreamEndCapture(cs2, &gr) == cudaSuccess) {
                size_t n = 0;
                cudaGraphGetNodes(gr, nullptr, &n);
                std::vector<cudaGraphNode_t> nodes(n);
                int32_t nk = 0;                     // kernel nodes only (not memsets / copies / events)
                if (n && cudaGraphGetNodes(gr, nodes.data(), &n) == cudaSuccess)
                    for (size_t i = 0; i < n; ++i) {
                        cudaGraphNodeType t;
                        if (cudaGraphNodeGetType(nodes[i], &t) == cudaSuccess && t == cudaGraphNodeTypeKernel) ++nk;
                    }
                p->info.kernels_per_step = nk;
                cudaGraphDestroy(gr);
            }
        }
        cudaGetLastError();
        cudaStreamDestroy(cs2);
    }
    p->info.arena_bytes = A.bytes + (p->reg_arena ? p->reg_arena->bytes : 0) + p->sb.bytes;
    if ((st = sync_check(c, s))) { betty_plan_destroy(c, p); return st; }
    *out = p;
    return BETTY_OK;
}

extern "C" betty_status betty_plan_info_get(const betty_plan* p, betty_plan_info* info) {
    if (!p || !info) return BETTY_EINVAL;
    *info = p->info;
    return BETTY_OK;
}

extern "C" void betty_plan_destroy(betty_ctx* c, betty_plan* p) {
    if (!c || !p) return;
    cudaDeviceSynchronize();
    if (p->gexec) cudaGraphExecDestroy(p->gexec);
    if (p->cap_stream) cudaStreamDestroy(p->cap_stream);
    if (p->side) cudaStreamDestroy(p->side);
    if (p->ev_fork) cudaEventDestroy(p->ev_fork);
    if (p->ev_join) cudaEventDestroy(p->ev_join);
    p->probe.destroy();
    sage_free(c, &p->sb, 0);
    if (p->arena) { p->arena->s = 0; p->arena->release(); delete p->arena; }
    if (p->reg_arena) { p->reg_arena->s = 0; p->reg_arena->release(); delete p->reg_arena; }
    cudaDeviceSynchronize();
    delete p;
}

extern "C" betty_status betty_step(betty_ctx* c, betty_plan* p, const float* params, const void* feats,
                                   int64_t ld_feats, const int32_t* labels, float loss_scale, float* grad_accum,
                                   float* loss_accum, betty_stream stream) {
    if (!c || !p) return BETTY_EINVAL;
    cudaStream_t s = (cudaStream_t)stream;
    if (!params || !labels || !grad_accum || !loss_accum) return fail(c, BETTY_EINVAL, "step: null argument");
    betty_status st = check_feats(c, p->m, feats, ld_feats);
    if (st) return st;
    if (!(p->flags & BETTY_PLAN_GRAPH)) {
        step_body(c, p, params, feats, ld_feats, labels, loss_scale, grad_accum, loss_accum, s);
        return check_launch(c);
    }
    float sc = loss_scale;
    int32_t scbits;
    memcpy(&scbits, &sc, 4);
    const void* key[9] = {params, feats, (const void*)(intptr_t)ld_feats, labels, grad_accum, loss_accum,
                          (const void*)(intptr_t)scbits, nullptr, (const void*)(intptr_t)p->probe.site};
    if (!p->gexec || memcmp(key, p->key, sizeof key) != 0) {
        if (p->gexec) { cudaGraphExecDestroy(p->gexec); p->gexec = nullptr; }
        // capture on a private stream (the caller's may be the legacy default
        // stream, which cannot be captured); the graph is launched on `s`
        if (!p->cap_stream) {
            int prio_lo = 0, prio_hi = 0;
            cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
            CUDA_OK(c, cudaStreamCreateWithPriority(&p->cap_stream, cudaStreamNonBlocking, prio_hi));
        }
        CUDA_OK(c, cudaStreamSynchronize(s));
        cudaGraph_t g;
        CUDA_OK(c, cudaStreamBeginCapture(p->cap_stream, cudaStreamCaptureModeThreadLocal));
        step_body(c, p, params, feats, ld_feats, labels, loss_scale, grad_accum, loss_accum, p->cap_stream);
        CUDA_OK(c, cudaStreamEndCapture(p->cap_stream, &g));
        static const bool no_prio = getenv("BETTY_NO_NODE_PRIORITY") != nullptr;     // A/B switch
        cudaError_t e = cudaGraphInstantiate(&p->gexec, g, no_prio ? 0 : cudaGraphInstantiateFlagUseNodePriority);
        cudaGraphDestroy(g);
        if (e != cudaSuccess) return fail(c, BETTY_ECUDA, "graph instantiate: %s", cudaGetErrorString(e));
        memcpy(p->key, key, sizeof key);
    }
    CUDA_OK(c, cudaGraphLaunch(p->gexec, s));
    return BETTY_OK;
}

extern "C" betty_status betty_adam(betty_ctx* c, float* params, float* grad, float* m, float* v, int64_t n, int32_t t,
                                   float lr, float b1, float b2, float eps, int32_t zero_grad, betty_stream stream) {
    if (!c) return BETTY_EINVAL;
    if (!params || !grad || !m || !v || n < 0 || t < 1) return fail(c, BETTY_EINVAL, "adam: bad argument");
    adam(c, params, grad, m, v, n, t, lr, b1, b2, eps, zero_grad != 0, (cudaStream_t)stream);
    return check_launch(c);
}

extern "C" betty_status betty_plan_group_blocks(betty_ctx* c, betty_plan* p, int32_t g, betty_block* out,
                                                betty_stream stream) {
    if (!c || !p || !out || g < 0 || g >= (int32_t)p->groups.size()) return BETTY_EINVAL;
    cudaStream_t s = (cudaStream_t)stream;
    ExtractArgs a{};
    a.L = p->L; a.full = p->full.data(); a.part = p->part; a.K = p->K;
    a.ks = p->d_ks + g * p->c; a.c = (int32_t)p->groups[g].size();
    a.layers = p->X.layers.data(); a.sc = p->X.sc; a.csc_mask = p->csc_mask;
    extract_group(c, a, s);
    std::vector<int64_t> h(4 * p->L);
    cudaMemcpyAsync(h.data(), p->X.cnt_all, sizeof(int64_t) * 4 * p->L, cudaMemcpyDeviceToHost, s);
    betty_status st = sync_check(c, s);
    if (st) return st;
    for (int l = 0; l < p->L; ++l) {
        const ExtractLayer& B = p->X.layers[l];
        out[l] = betty_block{h[4 * l], h[4 * l + 1], h[4 * l + 2], B.indptr, B.indices, B.src_pos, B.src_gid,
                             B.t_indptr, B.t_indices};
    }
    return BETTY_OK;
}

// ------------------------------------------------- GEMM test hooks (bf16)
extern "C" betty_status betty_test_gemm(betty_ctx* c, int32_t kind, const void* A, int64_t lda, const void* B,
                                        int64_t ldb, int64_t M, int64_t M_cap, int32_t K, int32_t N, float* C,
                                        int64_t ldc, int32_t use_tc, betty_stream stream) {
    if (!c || !A || !B || !C || M < 0 || M_cap < M || K < 1 || N < 1) return BETTY_EINVAL;
    cudaStream_t s = (cudaStream_t)stream;
    int64_t* Md = (int64_t*)ctx_alloc(c, 8, s);
    cudaMemcpyAsync(Md, &M, 8, cudaMemcpyHostToDevice, s);
    const bool saved = c->use_tc;
    c->use_tc = use_tc && tc_available();
    betty_status st = BETTY_OK;
    const bool f32 = (kind & 2) != 0;     // fp32 operands: 3xTF32 on the tensor cores (use_tc) or SIMT FFMA
    const bool saved_f = c->fp32_tc;
    c->fp32_tc = use_tc != 0;
    if ((kind & 1) == 0) {      // C[M x N] = A[M x K] . B, B given as [N x K] (K-major)
        GemmRow g{};
        g.A = A; g.lda = lda; g.a_bf16 = !f32;
        g.B = B; g.ldb = ldb; g.b_bf16 = !f32; g.transB = true;
        g.M_dev = Md; g.M_cap = std::max<int64_t>(M_cap, 1); g.K = K; g.N = N;
        g.C = C; g.ldc = ldc; g.c_bf16 = false; g.epi = EPI_STORE;
        float* hl = nullptr;
        if (f32 && use_tc) {
            hl = (float*)ctx_alloc(c, sizeof(float) * 2 * N * ldb, s);
            split_tf32_dev((const float*)B, hl, hl + N * ldb, (int64_t)N * ldb, s);
            g.Bhi = hl; g.Blo = hl + N * ldb;
        }
        gemm_row(c, g, s);
        if (hl) ctx_free(c, hl, s);
    } else {                    // C[K x N] = A[M x K]^T . B[M x N]  (C zero-initialised by the caller: it ADDS)
        int64_t S = gemm_red_splits(M_cap, K, N);
        float* part = (float*)ctx_alloc(c, sizeof(float) * S * K * N, s);
        GemmRed r{};
        r.A = A; r.lda = lda; r.a_bf16 = !f32;
        r.B = B; r.ldb = ldb; r.b_bf16 = !f32;
        r.M_dev = Md; r.M_cap = std::max<int64_t>(M_cap, 1); r.K1 = K; r.N = N;
        r.partials = part; r.S = (int)S; r.grad = C;
        r.map = GradMap{MAP_AGG, K, N, K, N, 0, 0, 0, 0, 0};   // identity: rows < K -> off_ws + i*N + j
        r.map.Fp = 1 << 29;                                     // no neighbour / bias rows
        gemm_red(c, r, s);
        ctx_free(c, part, s);
        (void)ldc;
    }
    c->use_tc = saved;
    c->fp32_tc = saved_f;
    ctx_free(c, Md, s);
    st = sync_check(c, s);
    return st;
}

extern "C" betty_status betty_plan_probe(betty_plan* p, int32_t site) {
    if (!p || site < 0 || site > PROBE_GEMM_FWD_L1) return BETTY_EINVAL;
    p->probe.site = site;
    p->probe.used = 0;
    p->sb.probe = site ? &p->probe : nullptr;
    return BETTY_OK;
}

extern "C" betty_status betty_plan_probe_read(betty_plan* p, float* total_ms, int32_t* launches) {
    if (!p || !total_ms || !launches) return BETTY_EINVAL;
    *total_ms = 0.f;
    *launches = p->probe.used;
    for (int i = 0; i < p->probe.used; ++i) {
        if (cudaEventSynchronize(p->probe.ev[2 * i + 1]) != cudaSuccess) return BETTY_ECUDA;
        float ms = 0.f;
        if (cudaEventElapsedTime(&ms, p->probe.ev[2 * i], p->probe.ev[2 * i + 1]) != cudaSuccess) return BETTY_ECUDA;
        *total_ms += ms;
    }
    return BETTY_OK;
}

extern "C" betty_status betty_sync_check(betty_ctx* c, betty_stream stream) {
    if (!c) return BETTY_EINVAL;
    return sync_check(c, (cudaStream_t)stream);
}

// ------------------------------------------------------------------ §4.4 memory-aware K
extern "C" betty_status betty_mb_sizes(betty_ctx* c, const betty_block* full, int32_t L, const int32_t* part,
                                       int64_t n_out, int32_t K, int64_t* sizes, betty_stream stream) {
    if (!c) return BETTY_EINVAL;
    betty_status st = check_full(c, full, L);
    if (st) return st;
    if (K < 1 || !sizes || full[L - 1].n_dst != n_out || (n_out > 0 && !part))
        return fail(c, BETTY_EINVAL, "mb_sizes: bad K / sizes / n_out / part");
    if (!extract_limits_ok(K, 1, n_out, full[L - 1].n_edges))
        return fail(c, BETTY_EUNSUPPORTED, "mb_sizes: K > 16384, n_out >= 2^23 or >= 2^40 top-layer edges");
    std::vector<ExtractFull> F = to_full(full, L);
    std::vector<int32_t> ks(K);
    for (int k = 0; k < K; ++k) ks[k] = k;
    std::vector<std::vector<int64_t>> sz;
    if ((st = size_micro_batches(c, F.data(), full, L, part, n_out, K, ks.data(), K, &sz, (cudaStream_t)stream)))
        return st;
    for (int k = 0; k < K; ++k)
        for (int q = 0; q < 3 * L; ++q) sizes[(int64_t)k * 3 * L + q] = sz[k][q];
    return BETTY_OK;
}

extern "C" betty_status betty_mem_estimate(const betty_model* model, const int64_t* sizes, int64_t* terms) {
    if (!model || !model->dims || model->L < 1 || !sizes || !terms) return BETTY_EINVAL;
    const int L = model->L;
    const int32_t* d = model->dims;
    const bool pool = model->aggr == BETTY_AGGR_POOL;
    int64_t p_gnn = 0, p_agg = 0;                       // N_P_GNN, N_P_Agg (Table 3)
    int64_t blocks = 0, hidden = 0, inter = 0;
    for (int l = 0; l < L; ++l) {
        const int64_t nd = sizes[3 * l], ns = sizes[3 * l + 1], ne = sizes[3 * l + 2];
        p_gnn += (int64_t)d[l] * d[l + 1] * 2 + d[l + 1];
        if (pool) p_agg += (int64_t)d[l] * (d[l] + 1);
        blocks += 3 * ne;                               // (4): src id, dst id, weight per edge
        hidden += nd * d[l + 1];                        // (5): layer outputs
        inter += (pool ? nd + ns : nd) * d[l];          // (6): h_N (mean) / fc_pool out + max (pool)
    }
    terms[0] = p_gnn;                                   // (1)
    terms[1] = sizes[1] * d[0];                         // (2) N_in x H_in (layer-0 sources)
    terms[2] = sizes[3 * (L - 1)];                      // (3) N_out
    terms[3] = blocks;
    terms[4] = hidden;
    terms[5] = inter;
    terms[6] = p_gnn + p_agg;                           // (7) gradients
    terms[7] = 2 * (p_gnn + p_agg);                     // (8) Adam m, v
    terms[8] = terms[0] + terms[1] + terms[2] + terms[3] + terms[4] + terms[7] + std::max(terms[5], terms[6]);
    return BETTY_OK;
}

extern "C" betty_status betty_memory_aware_k(betty_ctx* c, const betty_model* model, const betty_block* full,
                                             int32_t L, const int64_t* reg_indptr, const int32_t* reg_col,
                                             const int32_t* reg_w, int64_t n_out, int64_t capacity_bytes,
                                             int32_t K0, int32_t K_max, int32_t method, int32_t* part,
                                             int32_t* K_out, int64_t* peak_bytes, betty_stream stream) {
    if (!c) return BETTY_EINVAL;
    if (!model || !part || !K_out || !peak_bytes || model->L != L || (n_out > 0 && !reg_indptr))
        return fail(c, BETTY_EINVAL, "memory_aware_k: bad arguments");
    betty_status st = check_full(c, full, L);
    if (st) return st;
    if (full[L - 1].n_dst != n_out) return fail(c, BETTY_EINVAL, "memory_aware_k: n_out != output block n_dst");
    cudaStream_t s = (cudaStream_t)stream;
    if (K_max <= 0 || K_max > n_out) K_max = (int32_t)std::max<int64_t>(1, n_out);
    *K_out = -1;
    *peak_bytes = -1;
    Arena A{c, s};
    int32_t* d_part = A.get<int32_t>(std::max<int64_t>(1, n_out));
    if (!d_part) { A.release(); return fail(c, BETTY_ENOMEM, "memory_aware_k: allocation failed"); }
    std::vector<ExtractFull> F = to_full(full, L);
    std::vector<int32_t> hp(std::max<int64_t>(1, n_out));
    std::vector<int64_t> terms(9);
    for (int32_t K = std::max(1, K0); K <= K_max; ++K) {
        if ((st = betty_reg_partition_ex(reg_indptr, reg_col, reg_w, n_out, K, method, 0.03, hp.data()))) break;
        if (n_out) cudaMemcpyAsync(d_part, hp.data(), sizeof(int32_t) * n_out, cudaMemcpyHostToDevice, s);
        std::vector<int32_t> ks(K);
        for (int k = 0; k < K; ++k) ks[k] = k;
        std::vector<std::vector<int64_t>> sz;
        if ((st = size_micro_batches(c, F.data(), full, L, d_part, n_out, K, ks.data(), K, &sz, s))) break;
        int64_t peak = 0;
        for (int k = 0; k < K; ++k) {
            betty_mem_estimate(model, sz[k].data(), terms.data());
            peak = std::max(peak, terms[8] * 4);        // 4-byte elements (reading M4)
        }
        if (*peak_bytes < 0 || peak < *peak_bytes) *peak_bytes = peak;
        if (peak <= capacity_bytes) {
            *K_out = K;
            *peak_bytes = peak;
            std::copy(hp.begin(), hp.begin() + n_out, part);
            break;
        }
    }
    A.release();
    return st;
}
