// sage.cu -- host orchestration of one (group-concatenated) micro-batch
// through the GraphSAGE forward, loss and backward (a3-a6).
//
// Per layer l (Fi -> Fo), following DGL SAGEConv's two forms (reading #11):
//   AGG  (mean, Fi <= Fo):  XA = [h_dst | mean h_N | 1]          (agg kernel)
//                           S  = XA [W_s; W_n; b]                (GEMM + ReLU/ones epilogue)
//   PF   (mean, Fi >  Fo):  Y  = [H | 1] [W_n | W_s; 0 | b]      (GEMM, all src rows)
//                           S  = Y_self + mean_u Y_neigh          (agg kernel, + ReLU)
//   POOL:                   Zp = [H | 1] [W_p; b_p] ; XA = [h_dst | max_u ReLU(Zp_u) | 1] ; S = XA W
// Backward mirrors it; dW GEMMs reduce over nodes and ADD into the flat
// gradient (fused accumulation); no gradient w.r.t. the input features.
#include <algorithm>
#include "internal.h"
#include "model.h"

namespace betty {

#define PB(site) do { if (b.probe) b.probe->begin((site), s); } while (0)
#define PE(site) do { if (b.probe) b.probe->end((site), s); } while (0)

bool make_model_cfg(int L, int aggr, int gemm, int feat_dtype, const int32_t* dims, ModelCfg* out) {
    if (L < 1 || L > 16 || !dims || aggr < 0 || aggr > 2 || (gemm != 0 && gemm != 1) ||
        (feat_dtype != 0 && feat_dtype != 1))
        return false;
    ModelCfg m;
    m.L = L;
    m.aggr = aggr;
    m.sum = aggr == 2;
    m.bf16 = gemm == 1;
    m.feat_bf16 = feat_dtype == 1;
    m.dims.assign(dims, dims + L + 1);
    for (int d : m.dims)
        if (d < 1 || d > 65536) return false;
    if (m.dims[L] > 256) return false;   // loss kernel: classes <= 256
    int64_t base = 0;
    for (int l = 0; l < L; ++l) {
        LayerCfg c{};
        c.Fi = m.dims[l];
        c.Fo = m.dims[l + 1];
        c.last = (l == L - 1);
        c.kind = aggr == 1 ? KIND_POOL : (c.Fi > c.Fo ? KIND_PF : KIND_AGG);
        c.Fp = (int)r8(c.Fi);
        c.Fop = (int)r8(c.Fo);
        if (aggr == 1) {
            c.off_wp = base;
            c.off_bp = base + (int64_t)c.Fi * c.Fi;
            c.off_ws = c.off_bp + c.Fi;
        } else {
            c.off_wp = c.off_bp = -1;
            c.off_ws = base;
        }
        c.off_wn = c.off_ws + (int64_t)c.Fi * c.Fo;
        c.off_b = c.off_wn + (int64_t)c.Fi * c.Fo;
        base = c.off_b + c.Fo;
        c.ld_xa = r8(2 * c.Fp + 1);
        c.ld_gat = r8(c.Fi + 1);
        c.ld_y = c.Fop;          // PF: Y = [H|1] [W_n; 0] over all src rows (the neighbour half only)
        c.ld_g = c.Fop;          // PF: G = P^T D+ dS over all src rows (the self half is dS itself)
        c.ld_dxa = 2 * c.Fp;
        c.ld_zp = c.Fp;
        c.ld_dzp = c.Fp;
        c.ld_arg = c.Fp;                 // 16-byte aligned rows (vectorised pool kernels)
        c.ld_out = c.last ? c.Fop : r8(c.Fo + 1);
        c.ld_ds = c.Fop;
        c.ld_B = c.kind == KIND_PF ? 2 * c.Fop : c.Fop;
        c.ld_Bp = c.Fp;
        m.layers.push_back(c);
    }
    m.n_params = base;
    *out = m;
    return true;
}

static void* balloc(betty_ctx* c, SageBufs* b, int64_t bytes, cudaStream_t s) {
    if (bytes <= 0) bytes = 16;
    void* p = ctx_alloc(c, (size_t)bytes, s);
    if (p) { b->owned.push_back(p); b->bytes += bytes; }
    return p;
}

bool sage_alloc(betty_ctx* c, const ModelCfg& m, const std::vector<int64_t>& cap_dst,
                const std::vector<int64_t>& cap_src, SageBufs* b, cudaStream_t s) {
    const int64_t ea = m.bf16 ? 2 : 4;
    const bool tf = !m.bf16 && c->use_tc && c->fp32_tc;     // FP32 mode as 3xTF32 on the tensor cores
    b->tf32 = tf;
    b->l.assign(m.L, LayerBufs{});
    int64_t part_max = 1;
    bool ok = true;
    auto A = [&](int64_t bytes) { void* p = balloc(c, b, bytes, s); ok = ok && p; return p; };
    for (int l = 0; l < m.L; ++l) {
        const LayerCfg& L = m.layers[l];
        LayerBufs& B = b->l[l];
        const int64_t nd = std::max<int64_t>(cap_dst[l], 1), ns = std::max<int64_t>(cap_src[l], 1);
        if (m.needs_gat(l)) B.gat = A(ns * L.ld_gat * ea);
        if (L.kind == KIND_AGG || L.kind == KIND_POOL) {
            B.XA = A(nd * L.ld_xa * ea);
            if (l > 0 || L.kind == KIND_POOL) B.dXA = (float*)A(nd * L.ld_dxa * 4);
            B.B = A((2 * L.Fp + 1) * L.ld_B * ea);
            if (tf) { B.Bhi = A((2 * L.Fp + 1) * L.ld_B * 4); B.Blo = A((2 * L.Fp + 1) * L.ld_B * 4); }
            B.S_main = gemm_red_splits(nd, 2 * L.Fp + 1, L.Fo);
            part_max = std::max<int64_t>(part_max, (int64_t)B.S_main * (2 * L.Fp + 1) * L.Fo);
        }
        if (L.kind == KIND_PF) {
            B.Y = (float*)A(ns * L.ld_y * 4);
            B.Ys = (float*)A(nd * L.ld_y * 4);              // [H_dst|1] [W_s; b] over the dst rows only
            B.G = A(ns * L.ld_g * ea);
            B.B = A((L.Fi + 1) * L.ld_B * ea);
            if (tf) { B.Bhi = A((L.Fi + 1) * L.ld_B * 4); B.Blo = A((L.Fi + 1) * L.ld_B * 4); }
            if (l > 0) B.R = (float*)A(nd * m.layers[l - 1].ld_ds * 4);   // dS W_s^T (dst rows), residual of dX
            B.S_main = gemm_red_splits(ns, L.Fi + 1, L.Fop);
            B.S_self = gemm_red_splits(nd, L.Fi + 1, L.Fop);
            part_max = std::max<int64_t>(part_max, (int64_t)B.S_main * (L.Fi + 1) * L.Fop);
            part_max = std::max<int64_t>(part_max, (int64_t)B.S_self * (L.Fi + 1) * L.Fop);
        }
        if (L.kind == KIND_POOL) {
            B.Zp = (float*)A(ns * L.ld_zp * 4);
            B.arg = (int32_t*)A(nd * (m.arg8(l) ? (L.Fi + 15) / 16 * 16 : L.ld_arg * 4));
            B.dZp = A(ns * L.ld_dzp * ea);
            B.Bp = A((L.Fi + 1) * L.ld_Bp * ea);
            if (tf) { B.Bphi = A((L.Fi + 1) * L.ld_Bp * 4); B.Bplo = A((L.Fi + 1) * L.ld_Bp * 4); }
            B.S_pool = gemm_red_splits(ns, L.Fi + 1, L.Fi);
            part_max = std::max<int64_t>(part_max, (int64_t)B.S_pool * (L.Fi + 1) * L.Fi);
        }
        if (m.bf16 || tf) {          // K-major (transposed) weights for the tcgen05 forward GEMMs (TF: hi + lo)
            const int64_t krows = L.kind == KIND_PF ? (L.Fi + 1) : (2 * L.Fp + 1);
            B.ldbt = r8(krows);
            B.Bt = A(L.ld_B * B.ldbt * ea);
            if (tf) B.Btlo = A(L.ld_B * B.ldbt * 4);
            if (L.kind == KIND_POOL) {
                B.ldbpt = r8(L.Fi + 1);
                B.Bpt = A((int64_t)L.ld_Bp * B.ldbpt * ea);
                if (tf) B.Bptlo = A((int64_t)L.ld_Bp * B.ldbpt * 4);
            }
        }
        if (l >= 1) B.H = A(ns * m.layers[l - 1].ld_out * ea);
        if (l >= 1 && (m.bf16 || tf)) {
            B.ldhb = (m.dims[l] + 127) / 128 * 4;
            B.Hbits = (uint32_t*)A(ns * B.ldhb * 4);
        }
        if (!L.last) B.dS = A(nd * L.ld_ds * ea);
        if (L.last) {
            b->logits = (float*)A(nd * L.ld_out * 4);
            b->dS_last = (float*)A(nd * L.Fop * 4);
            b->dS_last_act = A(nd * L.ld_ds * ea);
        }
    }
    b->partials = (float*)A(part_max * 4);
    return ok;
}

void sage_free(betty_ctx* c, SageBufs* b, cudaStream_t s) {
    for (void* p : b->owned) ctx_free(c, p, s);
    b->owned.clear();
    b->l.clear();
    b->bytes = 0;
}

void sage_prep(betty_ctx* c, const ModelCfg& m, SageBufs& b, const float* params, cudaStream_t s) {
    std::vector<PrepLayer> P(m.L);
    for (int l = 0; l < m.L; ++l) {
        const LayerCfg& L = m.layers[l];
        PrepLayer& p = P[l];
        p.kind = L.kind == KIND_PF ? 1 : (L.kind == KIND_POOL ? 2 : 0);
        p.Fi = L.Fi; p.Fo = L.Fo; p.Fp = L.Fp; p.Fop = L.Fop;
        p.off_ws = L.off_ws; p.off_wn = L.off_wn; p.off_b = L.off_b; p.off_wp = L.off_wp; p.off_bp = L.off_bp;
        p.B = b.l[l].B; p.ldb = L.ld_B;
        p.Bp = b.l[l].Bp; p.ldbp = L.ld_Bp;
        p.Bt = b.l[l].Bt; p.ldbt = b.l[l].ldbt; p.ldbt_rows = L.ld_B;
        p.Bpt = b.l[l].Bpt; p.ldbpt = b.l[l].ldbpt;
        p.Bhi = b.l[l].Bhi; p.Blo = b.l[l].Blo; p.Btlo = b.l[l].Btlo;
        p.Bphi = b.l[l].Bphi; p.Bplo = b.l[l].Bplo; p.Bptlo = b.l[l].Bptlo;
    }
    prep_weights(c, params, P.data(), m.L, m.bf16, s);
}

// the [X | 1] operand of PF / POOL layers: the gathered copy at layer 0, else H_l
static void ones_operand(const ModelCfg& m, SageBufs& b, int l, const void** A, int64_t* lda) {
    if (l == 0) { *A = b.l[0].gat; *lda = m.layers[0].ld_gat; }
    else { *A = b.l[l].H; *lda = m.layers[l - 1].ld_out; }
}

// FP32 mode (3xTF32): the hi / lo weight parts of a GemmRow whose B is the main weight (pool = false)
// or the pool weight, viewed from column col0 of B (row col0 of its K-major copy)
static void tf_weights(GemmRow& g, const LayerBufs& B, bool pool, int64_t col0) {
    void* hi = pool ? B.Bphi : B.Bhi;
    void* lo = pool ? B.Bplo : B.Blo;
    void* tlo = pool ? B.Bptlo : B.Btlo;
    const int64_t ldbt = pool ? B.ldbpt : B.ldbt;
    g.Bhi = hi ? (const char*)hi + col0 * 4 : nullptr;
    g.Blo = lo ? (const char*)lo + col0 * 4 : nullptr;
    g.Btlo = tlo ? (const char*)tlo + col0 * ldbt * 4 : nullptr;
}

static GradMap grad_map(const LayerCfg& L, int mode) {
    GradMap g;
    g.mode = mode;
    g.Fi = L.Fi; g.Fo = L.Fo; g.Fp = L.Fp; g.Fop = L.Fop;
    g.off_ws = L.off_ws; g.off_wn = L.off_wn; g.off_b = L.off_b; g.off_wp = L.off_wp; g.off_bp = L.off_bp;
    return g;
}

void sage_forward(betty_ctx* c, const ModelCfg& m, SageBufs& b, const BlockView* v, const void* feats,
                  int64_t ld_feats, cudaStream_t s) {
    for (int l = 0; l < m.L; ++l) {
        const LayerCfg& L = m.layers[l];
        LayerBufs& B = b.l[l];
        const BlockView& V = v[l];
        const void* X = l == 0 ? feats : B.H;
        const bool xbf = l == 0 ? m.feat_bf16 : m.bf16;
        const int64_t ldx = l == 0 ? ld_feats : m.layers[l - 1].ld_out;
        const int32_t* xrow = l == 0 ? V.src_gid : nullptr;
        void* out = L.last ? (void*)b.logits : b.l[l + 1].H;
        const bool out_bf = L.last ? false : m.bf16;
        const int epi = L.last ? EPI_STORE : EPI_RELU_ONES;
        const void* Ao = nullptr;
        int64_t ldao = 0;
        if (L.kind != KIND_AGG) {
            if (l == 0)
                gather_ones(c, feats, m.feat_bf16, ld_feats, V.src_gid, V.cnt + 1, V.cap_src, L.Fi, B.gat, m.bf16,
                            L.ld_gat, s);
            ones_operand(m, b, l, &Ao, &ldao);
        }
        if (L.kind == KIND_PF) {
            // Y = [H|1] [W_n; 0] over every src row; Ys = [H_dst|1] [W_s; b] over the dst rows only
            // (the combined weight matrix holds [W_n | W_s; 0 | b]: column sub-views)
            const int64_t esz = m.bf16 ? 2 : 4;
            GemmRow g{};
            g.A = Ao; g.lda = ldao; g.a_bf16 = m.bf16;
            g.B = B.B; g.ldb = L.ld_B; g.b_bf16 = m.bf16; g.transB = false;
            g.M_dev = V.cnt + 1; g.M_cap = V.cap_src; g.K = L.Fi + 1; g.N = L.Fop;
            g.Bt = B.Bt; g.ldbt = B.ldbt;
            g.C = B.Y; g.ldc = L.ld_y; g.c_bf16 = false; g.epi = EPI_STORE;
            tf_weights(g, B, false, 0);
            PB(l == 0 ? PROBE_GEMM_FWD_L0 : PROBE_GEMM_FWD_L1);
            gemm_row(c, g, s);
            PE(l == 0 ? PROBE_GEMM_FWD_L0 : PROBE_GEMM_FWD_L1);
            GemmRow gs = g;
            gs.B = (const char*)B.B + L.Fop * esz;
            gs.Bt = B.Bt ? (const void*)((const char*)B.Bt + (int64_t)L.Fop * B.ldbt * esz) : nullptr;
            gs.M_dev = V.cnt + 0; gs.M_cap = V.cap_dst;
            gs.C = B.Ys;
            tf_weights(gs, B, false, L.Fop);
            gemm_row(c, gs, s);
            PB(l == 0 ? PROBE_AGG_L0 : PROBE_AGG_L1);
            agg_mean_pf(c, B.Y, B.Ys, L.ld_y, V.indptr, V.indices, V.cnt, V.cap_dst, L.Fo, L.Fop, !L.last, out,
                        out_bf, L.ld_out, m.sum, s);
            if (!L.last) b.l[l + 1].hbits_ok = false;
            PE(l == 0 ? PROBE_AGG_L0 : PROBE_AGG_L1);
            continue;
        }
        if (L.kind == KIND_POOL) {
            GemmRow g{};
            g.A = Ao; g.lda = ldao; g.a_bf16 = m.bf16;
            g.B = B.Bp; g.ldb = L.ld_Bp; g.b_bf16 = m.bf16;
            g.M_dev = V.cnt + 1; g.M_cap = V.cap_src; g.K = L.Fi + 1; g.N = L.Fi;
            g.Bt = B.Bpt; g.ldbt = B.ldbpt;
            g.C = B.Zp; g.ldc = L.ld_zp; g.c_bf16 = false; g.epi = EPI_STORE;
            tf_weights(g, B, true, 0);
            gemm_row(c, g, s);
            PB(l == 0 ? PROBE_AGG_L0 : PROBE_AGG_L1);
            agg_pool(c, X, xbf, ldx, xrow, B.Zp, L.ld_zp, V.indptr, V.indices, V.cnt, V.cap_dst, L.Fi, L.Fp, B.XA,
                     m.bf16, L.ld_xa, B.arg, m.arg8(l) ? (L.Fi + 15) / 16 * 16 : L.ld_arg, m.arg8(l), s);
            PE(l == 0 ? PROBE_AGG_L0 : PROBE_AGG_L1);
        } else {
            PB(l == 0 ? PROBE_AGG_L0 : PROBE_AGG_L1);
            // layer 0 reads feature rows by global id: straight from the extraction's edge -> gid
            // array when present, else through src_gid
            const int32_t* erow = (l == 0 && V.egid) ? V.egid : V.indices;
            const int32_t* emap = (l == 0 && !V.egid) ? V.src_gid : nullptr;
            agg_mean_xa(c, X, xbf, ldx, xrow, erow, emap, V.indptr, V.cnt, V.order_tab, V.cap_dst,
                        V.src_per_mb > 0 ? V.src_per_mb : V.cap_src, L.Fi, L.Fp, B.XA, m.bf16, L.ld_xa, m.sum,
                        l == 0 ? b.shards : nullptr, s);
            PE(l == 0 ? PROBE_AGG_L0 : PROBE_AGG_L1);
        }
        GemmRow g{};
        g.A = B.XA; g.lda = L.ld_xa; g.a_bf16 = m.bf16;
        g.B = B.B; g.ldb = L.ld_B; g.b_bf16 = m.bf16;
        g.M_dev = V.cnt + 0; g.M_cap = V.cap_dst; g.K = 2 * L.Fp + 1; g.N = L.Fo;
        g.Bt = B.Bt; g.ldbt = B.ldbt;
        g.C = out; g.ldc = L.ld_out; g.c_bf16 = out_bf; g.epi = epi;
        tf_weights(g, B, false, 0);
        if (!L.last) { g.obits = b.l[l + 1].Hbits; g.ldob = b.l[l + 1].ldhb; }
        PB(l == 0 ? PROBE_GEMM_FWD_L0 : PROBE_GEMM_FWD_L1);
        const bool bits = gemm_row(c, g, s);
        if (!L.last) b.l[l + 1].hbits_ok = bits;
        PE(l == 0 ? PROBE_GEMM_FWD_L0 : PROBE_GEMM_FWD_L1);
    }
}

void sage_loss(betty_ctx* c, const ModelCfg& m, SageBufs& b, const BlockView* v, const int32_t* labels, float scale,
               float* loss_accum, cudaStream_t s) {
    const LayerCfg& L = m.layers[m.L - 1];
    const BlockView& V = v[m.L - 1];
    // the fp32 dS of a project-first top layer is read only by P^T D+ dS: stored pre-scaled by 1/D_v
    loss_ce(c, b.logits, L.ld_out, labels, V.src_gid, V.cnt, V.cap_dst, L.Fo, scale, b.dS_last, L.Fop,
            b.dS_last_act, m.bf16, L.ld_ds, (L.kind == KIND_PF && !m.sum) ? V.indptr : nullptr, loss_accum, s);
}

void sage_backward(betty_ctx* c, const ModelCfg& m, SageBufs& b, const BlockView* v, const void* feats,
                   int64_t ld_feats, float* grad, cudaStream_t s) {
    (void)feats; (void)ld_feats;
    for (int l = m.L - 1; l >= 0; --l) {
        const LayerCfg& L = m.layers[l];
        LayerBufs& B = b.l[l];
        const BlockView& V = v[l];
        const void* dS_act = L.last ? b.dS_last_act : B.dS;
        const void* Hmask = l > 0 ? B.H : nullptr;
        const int64_t ldh = l > 0 ? m.layers[l - 1].ld_out : 0;
        void* dS_prev = l > 0 ? b.l[l - 1].dS : nullptr;
        const int64_t ld_prev = l > 0 ? m.layers[l - 1].ld_ds : 0;
        if (L.kind == KIND_PF) {
            // G = P^T D+ dS (all src rows); dW_n += [H|1]^T G ; [dW_s; db] += [H_dst|1]^T dS (dst rows);
            // dX = G W_n^T + [dst] dS W_s^T (the second term as the epilogue residual), masked by ReLU'
            const int64_t esz = m.bf16 ? 2 : 4;
            const bool ds_f32 = L.last;
            csc_pf(c, ds_f32 ? (const void*)b.dS_last : B.dS, !ds_f32 && m.bf16, ds_f32 ? L.Fop : L.ld_ds,
                   (ds_f32 || m.sum) ? nullptr : V.indptr,      // null: no 1/D (pre-scaled, or sum)
                   V.t_indptr, V.t_indices, V.cnt, V.cap_src, L.Fo, L.Fop, B.G, m.bf16, L.ld_g, s);
            const void* Ao; int64_t ldao;
            ones_operand(m, b, l, &Ao, &ldao);
            GemmRed r{};
            r.A = Ao; r.lda = ldao; r.a_bf16 = m.bf16;
            r.B = B.G; r.ldb = L.ld_g; r.b_bf16 = m.bf16;
            r.M_dev = V.cnt + 1; r.M_cap = V.cap_src; r.K1 = L.Fi + 1; r.N = L.Fo;
            r.partials = b.partials; r.S = B.S_main; r.grad = grad; r.map = grad_map(L, MAP_PF_N);
            gemm_red(c, r, s);
            GemmRed rs = r;
            rs.B = dS_act; rs.ldb = L.ld_ds;
            rs.M_dev = V.cnt + 0; rs.M_cap = V.cap_dst; rs.S = B.S_self; rs.map = grad_map(L, MAP_PF_S);
            gemm_red(c, rs, s);
            if (l > 0) {
                GemmRow gr{};                       // R = dS W_s^T over the dst rows
                gr.A = dS_act; gr.lda = L.ld_ds; gr.a_bf16 = m.bf16;
                gr.B = (const char*)B.B + L.Fop * esz; gr.ldb = L.ld_B; gr.b_bf16 = m.bf16; gr.transB = true;
                gr.M_dev = V.cnt + 0; gr.M_cap = V.cap_dst; gr.K = L.Fo; gr.N = L.Fi;
                gr.C = B.R; gr.ldc = ld_prev; gr.c_bf16 = false; gr.epi = EPI_STORE;
                tf_weights(gr, B, false, L.Fop);
                gemm_row(c, gr, s);
                GemmRow g{};
                g.A = B.G; g.lda = L.ld_g; g.a_bf16 = m.bf16;
                g.B = B.B; g.ldb = L.ld_B; g.b_bf16 = m.bf16; g.transB = true;
                g.M_dev = V.cnt + 1; g.M_cap = V.cap_src; g.K = L.Fo; g.N = L.Fi;
                g.C = dS_prev; g.ldc = ld_prev; g.c_bf16 = m.bf16; g.epi = EPI_RES_MASK;
                g.mask = Hmask; g.ldm = ldh; g.m_bf16 = m.bf16;
                g.res = B.R; g.ldr = ld_prev; g.nres_dev = V.cnt + 0;
                if (B.hbits_ok) { g.mbits = B.Hbits; g.ldmb = B.ldhb; }
                tf_weights(g, B, false, 0);
                gemm_row(c, g, s);
            }
            continue;
        }
        // AGG / POOL share the main layer: dW += XA^T dS
        {
            GemmRed r{};
            r.A = B.XA; r.lda = L.ld_xa; r.a_bf16 = m.bf16;
            r.B = dS_act; r.ldb = L.ld_ds; r.b_bf16 = m.bf16;
            r.M_dev = V.cnt + 0; r.M_cap = V.cap_dst; r.K1 = 2 * L.Fp + 1; r.N = L.Fo;
            r.partials = b.partials; r.S = B.S_main; r.grad = grad; r.map = grad_map(L, MAP_AGG);
            if (l == 0) PB(PROBE_GEMM_RED_L0);
            gemm_red(c, r, s);
            if (l == 0) PE(PROBE_GEMM_RED_L0);
        }
        if (l == 0 && L.kind == KIND_AGG) continue;       // no gradient w.r.t. input features
        {   // dXA = dS [W_s; W_n]^T
            GemmRow g{};
            g.A = dS_act; g.lda = L.ld_ds; g.a_bf16 = m.bf16;
            g.B = B.B; g.ldb = L.ld_B; g.b_bf16 = m.bf16; g.transB = true;
            g.M_dev = V.cnt + 0; g.M_cap = V.cap_dst; g.K = L.Fo; g.N = 2 * L.Fp;
            g.C = B.dXA; g.ldc = L.ld_dxa; g.c_bf16 = false; g.epi = EPI_STORE;
            tf_weights(g, B, false, 0);
            gemm_row(c, g, s);
        }
        if (L.kind == KIND_AGG) {
            csc_mean(c, B.dXA, L.ld_dxa, m.sum ? nullptr : V.indptr, V.t_indptr, V.t_indices, V.cnt, V.cap_src, L.Fi, L.Fp, Hmask,
                     m.bf16, ldh, B.hbits_ok ? B.Hbits : nullptr, B.ldhb, dS_prev, m.bf16, ld_prev, s);
            continue;
        }
        // POOL: route to the argmax, then W_pool
        route_pool(c, B.dXA, L.ld_dxa, B.arg, m.arg8(l) ? (L.Fi + 15) / 16 * 16 : L.ld_arg, m.arg8(l), V.indptr,
                   V.indices, V.t_indptr, V.t_indices, V.cnt, V.cap_src, L.Fi, L.Fp, B.Zp, L.ld_zp, B.dZp, m.bf16,
                   L.ld_dzp, s);
        const void* Ao; int64_t ldao;
        ones_operand(m, b, l, &Ao, &ldao);
        {
            GemmRed r{};
            r.A = Ao; r.lda = ldao; r.a_bf16 = m.bf16;
            r.B = B.dZp; r.ldb = L.ld_dzp; r.b_bf16 = m.bf16;
            r.M_dev = V.cnt + 1; r.M_cap = V.cap_src; r.K1 = L.Fi + 1; r.N = L.Fi;
            r.partials = b.partials; r.S = B.S_pool; r.grad = grad; r.map = grad_map(L, MAP_POOL);
            gemm_red(c, r, s);
        }
        if (l > 0) {
            GemmRow g{};
            g.A = B.dZp; g.lda = L.ld_dzp; g.a_bf16 = m.bf16;
            g.B = B.Bp; g.ldb = L.ld_Bp; g.b_bf16 = m.bf16; g.transB = true;
            g.M_dev = V.cnt + 1; g.M_cap = V.cap_src; g.K = L.Fi; g.N = L.Fi;
            g.C = dS_prev; g.ldc = ld_prev; g.c_bf16 = m.bf16; g.epi = EPI_RES_MASK;
            g.mask = Hmask; g.ldm = ldh; g.m_bf16 = m.bf16;
            if (B.hbits_ok) { g.mbits = B.Hbits; g.ldmb = B.ldhb; }
            g.res = B.dXA; g.ldr = L.ld_dxa; g.nres_dev = V.cnt + 0;
            tf_weights(g, B, true, 0);
            gemm_row(c, g, s);
        }
    }
}

}  // namespace betty
