/*
 * oracle/oracle.c -- the CPU ORACLE for Betty's micro-batch training hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.  It
 * shares no code, header, table or helper with the CUDA path
 * (paper_conf_asplos_yangzd023_b200/csrc); neither includes the other.
 *
 * Plain, slow, obviously-correct loops in float64, one function per step of
 * the method, each citing the PAPER.md passage it follows.  No blocking,
 * fusion or reordering beyond what the definitions state.
 *
 *   oracle_reg      -- REG weights c_ij = sum_k a_ki a_kj (Eq. 2-4,
 *                      PAPER.md:794-915; Alg. 1 lines 1-7)
 *   oracle_extract  -- micro-batch k of the batch-level partition
 *                      (§4.2.3) through every layer, with
 *                      the local<->global index mapping
 *   oracle_sage     -- GraphSAGE mean / pool layers (Table 1 PAPER.md:253-259,
 *                      Eq. 1), softmax cross-entropy, and the
 *                      closed-form backward, accumulating gradients
 *
 *   oracle_step     -- one batch: all K micro-batches, gradients summed
 *                      (Fig. 6)
 *   oracle_sage_ties -- oracle_sage, also reporting every hidden ReLU decision
 *                      that finite precision can take either way (reading
 *                      #24): |S| <= tau * M with M = the sum of the magnitudes
 *                      of the terms of S, and the gradient g that the decision
 *                      gates in the backward (dS = g if S > 0 else 0)
 *
 * Readings of the paper where it is silent or garbled are listed in DESIGN.md
 * §3 and SURVEY.md §8(c); the numbers in comments (#n) refer to that table.
 *
 * Pins (tests/test_oracle_*.py, run with -m "not gpu"): brute-force shared
 * neighbour counts, scipy B.B^T, closed forms (star, K_mn, disjoint stars),
 * REG invariants, the golden example G1 (tests/golden/g1.json), exhaustive
 * k-hop closure, finite differences of the loss, dense-matrix forward
 * reductions, and Betty's invariant sum_k g_k = g_full.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

/* One bipartite layer of a (micro-)batch, CSR by dst (host arrays).
 * dst ids are src ids [0, n_dst) ("dst nodes are a prefix of the src list",
 * the DGL block convention of the paper's stack). */
typedef struct {
    int64_t n_dst, n_src, n_edges;
    int64_t* indptr;     /* [n_dst+1] */
    int32_t* indices;    /* [n_edges] src ids (local for micro-batches, full-batch positions for the full batch) */
    int32_t* src_pos;    /* [n_src] position in the full-batch src list of this layer (NULL = identity) */
    int32_t* src_gid;    /* [n_src] global node id */
    int64_t* t_indptr;   /* [n_src+1] CSC */
    int32_t* t_indices;  /* [n_edges] dst ids, ascending per column */
} oblock;

void oracle_free(void* p) { free(p); }

void oracle_block_free(oblock* b, int L) {
    for (int l = 0; l < L; ++l) {
        free(b[l].indptr); free(b[l].indices); free(b[l].src_pos); free(b[l].src_gid);
        free(b[l].t_indptr); free(b[l].t_indices);
        memset(&b[l], 0, sizeof(oblock));
    }
}

static int cmp_i32(const void* a, const void* b) {
    int32_t x = *(const int32_t*)a, y = *(const int32_t*)b;
    return (x > y) - (x < y);
}

/* ------------------------------------------------------------------------ */
/* REG (§4.3.2).  A is the binary adjacency of the output block: a_ui = 1 iff
 * the sampled edge u -> i exists (Eq. 2; multi-edges collapse to 1, reading
 * #2).  C = A^T A, c_ij = sum_u a_ui a_uj = number of shared in-neighbours
 * (Eq. 3-4).  Only output nodes are kept (Alg. 1 l.5-6) and the diagonal is
 * removed (l.7); zero entries are dropped; rows list columns ascending; both
 * triangles are stored (reading #4).
 *
 * In: n_out rows, row i = sources of output i (any ids in [0, n_src)).
 * Out (malloc'd): indptr[n_out+1], col[nnz], w[nnz].  Returns nnz (or -1). */
int64_t oracle_reg(int64_t n_out, int64_t n_src, const int64_t* indptr, const int32_t* idx,
                   int64_t** out_indptr, int32_t** out_col, int32_t** out_w) {
    /* S_i: distinct sources of output i (row of A^T) */
    int64_t* sp = (int64_t*)calloc((size_t)n_out + 1, sizeof(int64_t));
    int32_t* s = (int32_t*)malloc(sizeof(int32_t) * (size_t)(indptr[n_out] > 0 ? indptr[n_out] : 1));
    for (int64_t i = 0; i < n_out; ++i) {
        int64_t n = indptr[i + 1] - indptr[i];
        int32_t* row = s + sp[i];
        memcpy(row, idx + indptr[i], sizeof(int32_t) * (size_t)n);
        qsort(row, (size_t)n, sizeof(int32_t), cmp_i32);
        int64_t m = 0;
        for (int64_t j = 0; j < n; ++j) if (j == 0 || row[j] != row[j - 1]) row[m++] = row[j];
        sp[i + 1] = sp[i] + m;   /* row i+1 is written right after the deduplicated row i */
    }

    /* Out(u) = { i : u in S_i }  -- column u of A^T, built by counting */
    int64_t* op = (int64_t*)calloc((size_t)n_src + 1, sizeof(int64_t));
    for (int64_t e = 0; e < sp[n_out]; ++e) op[s[e] + 1]++;
    for (int64_t u = 0; u < n_src; ++u) op[u + 1] += op[u];
    int32_t* o = (int32_t*)malloc(sizeof(int32_t) * (size_t)(sp[n_out] > 0 ? sp[n_out] : 1));
    int64_t* cur = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n_src > 0 ? n_src : 1));
    memcpy(cur, op, sizeof(int64_t) * (size_t)n_src);
    for (int64_t i = 0; i < n_out; ++i)
        for (int64_t e = sp[i]; e < sp[i + 1]; ++e) o[cur[s[e]]++] = (int32_t)i;
    free(cur);

    /* c_ij for each output i: for u in S_i, for j in Out(u), j != i: cnt[j]++ */
    int32_t* cnt = (int32_t*)calloc((size_t)(n_out > 0 ? n_out : 1), sizeof(int32_t));
    int32_t* touched = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n_out > 0 ? n_out : 1));
    int64_t cap = 1024, nnz = 0;
    int32_t* col = (int32_t*)malloc(sizeof(int32_t) * cap);
    int32_t* w = (int32_t*)malloc(sizeof(int32_t) * cap);
    int64_t* rp = (int64_t*)malloc(sizeof(int64_t) * ((size_t)n_out + 1));
    rp[0] = 0;
    for (int64_t i = 0; i < n_out; ++i) {
        int64_t nt = 0;
        for (int64_t e = sp[i]; e < sp[i + 1]; ++e) {
            int32_t u = s[e];
            for (int64_t f = op[u]; f < op[u + 1]; ++f) {
                int32_t j = o[f];
                if (j == i) continue;                 /* Remove_self_loop (Alg. 1 l.7) */
                if (cnt[j] == 0) touched[nt++] = j;
                cnt[j]++;
            }
        }
        qsort(touched, (size_t)nt, sizeof(int32_t), cmp_i32);
        if (nnz + nt > cap) {
            while (nnz + nt > cap) cap *= 2;
            col = (int32_t*)realloc(col, sizeof(int32_t) * cap);
            w = (int32_t*)realloc(w, sizeof(int32_t) * cap);
        }
        for (int64_t t = 0; t < nt; ++t) { col[nnz] = touched[t]; w[nnz] = cnt[touched[t]]; nnz++; cnt[touched[t]] = 0; }
        rp[i + 1] = nnz;
    }
    free(sp); free(s); free(op); free(o); free(cnt); free(touched);
    *out_indptr = rp; *out_col = col; *out_w = w;
    return nnz;
}

/* ------------------------------------------------------------------------ */
/* Micro-batch extraction (§4.2.3; §5).
 * Partition G=(U,V,E) into G'_k=(U_k,V_k,E_k): V_k = outputs with part==k
 * (disjoint, covering V); each layer's U_k = all sources of V_k's sampled
 * rows; the next (lower) layer's V is this layer's U.  Orders (readings #9,
 * #10): outputs ascending; src = dst ++ (new sources ascending full-batch src
 * position); each row keeps its full-batch order; CSC columns list dst ids
 * ascending.
 *
 * full[l]: full-batch block l (indices = full-batch src positions; the full
 * dst list of block l is the prefix of its src list, and the full src list of
 * block l is the full dst list of block l-1).  Output blocks are malloc'd.
 * Returns 0, or -1 on bad input. */
int oracle_extract(int L, const oblock* full, const int32_t* part, int64_t n_out, int32_t K, int32_t k,
                   oblock* mb) {
    if (L < 1 || k < 0 || k >= K || full[L - 1].n_dst != n_out) return -1;
    for (int64_t i = 0; i < n_out; ++i) if (part[i] < 0 || part[i] >= K) return -1;

    /* V_k: output positions with part == k, ascending (Alg. 1 l.9-12) */
    int64_t n_dst = 0;
    int32_t* dst_pos = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n_out > 0 ? n_out : 1));
    for (int64_t i = 0; i < n_out; ++i) if (part[i] == k) dst_pos[n_dst++] = (int32_t)i;

    for (int l = L - 1; l >= 0; --l) {
        const oblock* F = &full[l];
        oblock* B = &mb[l];
        memset(B, 0, sizeof(oblock));
        /* E_k: the full-batch rows of the dst nodes (in_edges) */
        B->n_dst = n_dst;
        B->indptr = (int64_t*)malloc(sizeof(int64_t) * ((size_t)n_dst + 1));
        B->indptr[0] = 0;
        for (int64_t i = 0; i < n_dst; ++i)
            B->indptr[i + 1] = B->indptr[i] + (F->indptr[dst_pos[i] + 1] - F->indptr[dst_pos[i]]);
        B->n_edges = B->indptr[n_dst];

        /* U_k: dst prefix (a dst node's full src position is its full dst
         * position), then the other sources in ascending full src position */
        int32_t* loc = (int32_t*)malloc(sizeof(int32_t) * (size_t)(F->n_src > 0 ? F->n_src : 1));
        for (int64_t p = 0; p < F->n_src; ++p) loc[p] = -1;
        for (int64_t i = 0; i < n_dst; ++i) loc[dst_pos[i]] = (int32_t)i;
        char* seen = (char*)calloc((size_t)(F->n_src > 0 ? F->n_src : 1), 1);
        for (int64_t i = 0; i < n_dst; ++i)
            for (int64_t e = F->indptr[dst_pos[i]]; e < F->indptr[dst_pos[i] + 1]; ++e)
                if (loc[F->indices[e]] < 0) seen[F->indices[e]] = 1;
        int64_t n_src = n_dst;
        for (int64_t p = 0; p < F->n_src; ++p) n_src += seen[p];
        B->n_src = n_src;
        B->src_pos = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n_src > 0 ? n_src : 1));
        for (int64_t i = 0; i < n_dst; ++i) B->src_pos[i] = dst_pos[i];
        int64_t s = n_dst;
        for (int64_t p = 0; p < F->n_src; ++p)
            if (seen[p]) { loc[p] = (int32_t)s; B->src_pos[s++] = (int32_t)p; }

        /* relabel edges to local src ids; local -> global index map */
        B->indices = (int32_t*)malloc(sizeof(int32_t) * (size_t)(B->n_edges > 0 ? B->n_edges : 1));
        for (int64_t i = 0; i < n_dst; ++i) {
            int64_t o = B->indptr[i];
            for (int64_t e = F->indptr[dst_pos[i]]; e < F->indptr[dst_pos[i] + 1]; ++e)
                B->indices[o++] = loc[F->indices[e]];
        }
        B->src_gid = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n_src > 0 ? n_src : 1));
        for (int64_t t = 0; t < n_src; ++t) B->src_gid[t] = F->src_gid[B->src_pos[t]];

        /* CSC by a stable counting sort over dst in ascending order */
        B->t_indptr = (int64_t*)calloc((size_t)n_src + 1, sizeof(int64_t));
        for (int64_t e = 0; e < B->n_edges; ++e) B->t_indptr[B->indices[e] + 1]++;
        for (int64_t t = 0; t < n_src; ++t) B->t_indptr[t + 1] += B->t_indptr[t];
        B->t_indices = (int32_t*)malloc(sizeof(int32_t) * (size_t)(B->n_edges > 0 ? B->n_edges : 1));
        int64_t* cur = (int64_t*)malloc(sizeof(int64_t) * ((size_t)n_src + 1));
        memcpy(cur, B->t_indptr, sizeof(int64_t) * ((size_t)n_src + 1));
        for (int64_t i = 0; i < n_dst; ++i)
            for (int64_t e = B->indptr[i]; e < B->indptr[i + 1]; ++e) B->t_indices[cur[B->indices[e]]++] = (int32_t)i;
        free(cur); free(loc); free(seen);

        /* next (lower) layer: its dst list is this layer's src list */
        free(dst_pos);
        dst_pos = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n_src > 0 ? n_src : 1));
        memcpy(dst_pos, B->src_pos, sizeof(int32_t) * (size_t)n_src);
        n_dst = n_src;
    }
    free(dst_pos);
    return 0;
}

/* ------------------------------------------------------------------------ */
/* GraphSAGE layers and loss.
 *
 * bf16 mode (reading #17): every matrix product rounds both operands to
 * bfloat16 (round-to-nearest-even) and multiplies in float64; the input
 * feature table, the parameters and each hidden activation H_{l+1} are held in
 * bf16.  Aggregations, softmax and the loss stay in float64.  fp32 mode
 * rounds nothing (everything float64). */

static double bf16_round(double x) {
    if (x == 0.0 || !isfinite(x)) return x;
    int e;
    double m = frexp(x, &e);          /* x = m * 2^e, 0.5 <= |m| < 1 */
    double q = nearbyint(ldexp(m, 8)); /* 8 significant bits, ties to even */
    return ldexp(q, e - 8);
}

/* exported for the test that pins the rounding against torch.bfloat16 */
double oracle_bf16_round(double x) { return bf16_round(x); }

typedef struct { int64_t r, c; double* a; } mat;

static mat mat_new(int64_t r, int64_t c) {
    mat m; m.r = r; m.c = c;
    m.a = (double*)calloc((size_t)(r * c > 0 ? r * c : 1), sizeof(double));
    return m;
}
static void mat_free(mat* m) { free(m->a); m->a = NULL; }
#define AT(m, i, j) ((m).a[(int64_t)(i) * (m).c + (j)])

/* out[i][j] += sum_k opA(i,k) * opB(k,j), k ascending; operands optionally
 * transposed and (bf16 mode) rounded to bf16 first. */
static void mm_acc(mat* out, const mat* A, int tA, const mat* B, int tB, int bf16) {
    int64_t M = tA ? A->c : A->r, K = tA ? A->r : A->c, N = tB ? B->r : B->c;
    double* a = (double*)malloc(sizeof(double) * (size_t)(M * K > 0 ? M * K : 1));
    double* b = (double*)malloc(sizeof(double) * (size_t)(K * N > 0 ? K * N : 1));
    for (int64_t i = 0; i < M; ++i)
        for (int64_t k = 0; k < K; ++k) {
            double x = tA ? AT(*A, k, i) : AT(*A, i, k);
            a[i * K + k] = bf16 ? bf16_round(x) : x;
        }
    for (int64_t k = 0; k < K; ++k)
        for (int64_t j = 0; j < N; ++j) {
            double x = tB ? AT(*B, j, k) : AT(*B, k, j);
            b[k * N + j] = bf16 ? bf16_round(x) : x;
        }
    for (int64_t i = 0; i < M; ++i)
        for (int64_t k = 0; k < K; ++k) {
            const double aik = a[i * K + k];
            for (int64_t j = 0; j < N; ++j) AT(*out, i, j) += aik * b[k * N + j];
        }
    free(a); free(b);
}

/* out[i][j] += sum_k |opA(i,k)| * |opB(k,j)| -- the magnitude of the terms of
 * the same product (for the ReLU-decision report of oracle_sage_ties). */
static void mm_acc_abs(mat* out, const mat* A, int tA, const mat* B, int tB, int bf16) {
    int64_t M = tA ? A->c : A->r, K = tA ? A->r : A->c, N = tB ? B->r : B->c;
    for (int64_t i = 0; i < M; ++i)
        for (int64_t k = 0; k < K; ++k) {
            double a = tA ? AT(*A, k, i) : AT(*A, i, k);
            a = fabs(bf16 ? bf16_round(a) : a);
            for (int64_t j = 0; j < N; ++j) {
                double b = tB ? AT(*B, j, k) : AT(*B, k, j);
                AT(*out, i, j) += a * fabs(bf16 ? bf16_round(b) : b);
            }
        }
}

/* ReLU-decision report (oracle_sage_ties): set while that call runs */
typedef struct {
    double tau;
    int64_t cap, n, found;   /* stored entries (<= cap), decisions found */
    int32_t* level;      /* the decision is the mask of H_level (level = l + 1 for layer l's output) */
    int64_t* v;
    int32_t* j;
    double* S;           /* the pre-activation */
    double* M;           /* sum of the magnitudes of its terms */
    double* g;           /* the gradient the decision gates (dX of layer level, before the mask) */
} tie_report;
static tie_report* g_ties = NULL;

/* parameter block of layer l: (pool: W_pool [Fi x Fi], b_pool [Fi]),
 * W_self [Fi x Fo], W_neigh [Fi x Fo], b [Fo] -- flat, row-major */
typedef struct { int64_t wp, bp, ws, wn, b, end; } poff;
static poff layer_offsets(const int32_t* dims, int l, int pool, int64_t base) {
    poff o; int64_t fi = dims[l], fo = dims[l + 1];
    o.wp = base; o.bp = base + (pool ? fi * fi : 0);
    o.ws = o.bp + (pool ? fi : 0);
    o.wn = o.ws + fi * fo; o.b = o.wn + fi * fo; o.end = o.b + fo;
    return o;
}
static mat param_mat(const double* params, int64_t off, int64_t r, int64_t c, int bf16) {
    mat m = mat_new(r, c);
    for (int64_t t = 0; t < r * c; ++t) m.a[t] = bf16 ? bf16_round(params[off + t]) : params[off + t];
    return m;
}

/*
 * Forward + loss + backward of one micro-batch (its L blocks), ADDING the
 * gradient into grad[] (float64, the flat parameter layout) and the loss into
 * *loss -- gradient accumulation across micro-batches.
 *
 * Layer l (block mb[l]; X = H_l [n_src x Fi], X_d = X[0:n_dst];
 * P = binary n_dst x n_src CSR, D+ = diag(1/deg) with 1/0 := 0, reading #12):
 *   mean (Table 1 "Mean", Eq. 1; DGL SAGEConv form, reading #11):
 *     A = D+ P X ;  S = X_d W_s + A W_n + b
 *     DGL's SAGEConv applies W_n before the aggregation when Fi > Fo
 *     (D+ P (X W_n), equal in exact arithmetic); the oracle follows the same
 *     two forms so that bf16 rounding points coincide with the GPU's.
 *   pool (Table 1 "Pooling", reading #14):
 *     Zp = X W_p + b_p ; Z = ReLU(Zp) ; A[v,f] = max_{u in N(v)} Z[u,f]
 *     (0 for an empty row; the first maximum in row order is the argmax)
 *     S = X_d W_s + A W_n + b
 *   H_{l+1} = ReLU(S) for l < L-1; S = logits for l = L-1.
 * Loss (reading #15): loss += s * sum_{v} [logsumexp(S_v) - S_v[y_v]],
 * s = loss_scale = 1 / n_out(full batch), y_v = labels[gid(v)];
 * dS = s * (softmax(S) - onehot(y)).
 * Backward (closed form of the above; ReLU'(0) = 0):
 *   dW_s += X_d^T dS ; db += 1^T dS
 *   mean, aggregate-first: dW_n += A^T dS ; dX = [dS W_s^T ; 0] + P^T D+ (dS W_n^T)
 *   mean, project-first:   dZ = P^T D+ dS ; dW_n += X^T dZ ; dX = [dS W_s^T ; 0] + dZ W_n^T
 *   pool: dW_n += A^T dS ; dA = dS W_n^T ; dZ[u,f] = sum_{v: arg[v,f]=u} dA[v,f] ;
 *         dZp = dZ (.) [Zp > 0] ; dW_p += X^T dZp ; db_p += 1^T dZp ;
 *         dX = [dS W_s^T ; 0] + dZp W_p^T
 *   dS_{l-1} = dX (.) [H_l > 0]; no gradient w.r.t. the input features.
 *
 * params: float64 in the flat layout (the caller widens fp32 parameters;
 * float64 lets the finite-difference pins perturb them exactly).
 * aggr: 0 mean, 1 pool, 2 sum.  force_form: -1 DGL rule, 0 aggregate-first,
 * 1 project-first (mean only; for the tests that pin the two forms equal).
 * logits_out: optional [n_dst(L-1) x dims[L]].  Returns 0.
 */
int oracle_sage(int L, const int32_t* dims, int aggr, int bf16, int force_form, const oblock* mb,
                const double* params, const float* feats, int64_t ld, const int32_t* labels, double loss_scale,
                double* grad, double* loss, double* logits_out) {
    const int pool = (aggr == 1);
    /* Table 1 "Sum": h_N = sum_u h_u, i.e. the mean without 1/D_v; the same
     * SAGEConv form and project-first rule (reading #11) */
    const int sum = (aggr == 2);
    mat* H = (mat*)calloc((size_t)L + 1, sizeof(mat));       /* H[l] = input of layer l, [n_src(l) x dims[l]] */
    mat* Aagg = (mat*)calloc((size_t)L, sizeof(mat));        /* aggregated neighbour features (or D+P(XWn)) */
    mat* Zp = (mat*)calloc((size_t)L, sizeof(mat));          /* pool pre-activation */
    int32_t** arg = (int32_t**)calloc((size_t)L, sizeof(int32_t*));
    int* projf = (int*)calloc((size_t)L, sizeof(int));
    mat S = {0, 0, NULL};

    /* H_0 = features of the layer-0 sources (bf16: the feature table is bf16) */
    H[0] = mat_new(mb[0].n_src, dims[0]);
    for (int64_t u = 0; u < mb[0].n_src; ++u)
        for (int32_t f = 0; f < dims[0]; ++f) {
            double x = (double)feats[(int64_t)mb[0].src_gid[u] * ld + f];
            AT(H[0], u, f) = bf16 ? bf16_round(x) : x;
        }

    int64_t base = 0;
    for (int l = 0; l < L; ++l) {
        const oblock* B = &mb[l];
        const int64_t fi = dims[l], fo = dims[l + 1], nd = B->n_dst, ns = B->n_src;
        poff o = layer_offsets(dims, l, pool, base);
        base = o.end;
        mat Ws = param_mat(params, o.ws, fi, fo, bf16), Wn = param_mat(params, o.wn, fi, fo, bf16);
        mat bb = param_mat(params, o.b, 1, fo, bf16);
        mat X = H[l];
        mat Xd = { nd, fi, X.a };                            /* dst prefix rows */
        S = mat_new(nd, fo);
        mat ones = mat_new(nd, 1);
        for (int64_t v = 0; v < nd; ++v) ones.a[v] = 1.0;
        mm_acc(&S, &Xd, 0, &Ws, 0, bf16);                    /* X_d W_s */
        mm_acc(&S, &ones, 0, &bb, 0, bf16);                  /* + 1 b^T */
        if (!pool) {
            projf[l] = force_form >= 0 ? force_form : (fi > fo);
            if (!projf[l]) {
                Aagg[l] = mat_new(nd, fi);                  /* A = D+ P X */
                for (int64_t v = 0; v < nd; ++v) {
                    int64_t deg = B->indptr[v + 1] - B->indptr[v];
                    for (int64_t e = B->indptr[v]; e < B->indptr[v + 1]; ++e)
                        for (int64_t f = 0; f < fi; ++f) AT(Aagg[l], v, f) += AT(X, B->indices[e], f);
                    for (int64_t f = 0; f < fi && deg > 0 && !sum; ++f) AT(Aagg[l], v, f) /= (double)deg;
                }
                mm_acc(&S, &Aagg[l], 0, &Wn, 0, bf16);      /* + A W_n */
            } else {
                mat Z = mat_new(ns, fo);                      /* Z = X W_n */
                mm_acc(&Z, &X, 0, &Wn, 0, bf16);
                Aagg[l] = mat_new(nd, fo);                  /* D+ P Z */
                for (int64_t v = 0; v < nd; ++v) {
                    int64_t deg = B->indptr[v + 1] - B->indptr[v];
                    for (int64_t e = B->indptr[v]; e < B->indptr[v + 1]; ++e)
                        for (int64_t f = 0; f < fo; ++f) AT(Aagg[l], v, f) += AT(Z, B->indices[e], f);
                    for (int64_t f = 0; f < fo && deg > 0 && !sum; ++f) AT(Aagg[l], v, f) /= (double)deg;
                }
                for (int64_t t = 0; t < nd * fo; ++t) S.a[t] += Aagg[l].a[t];
                mat_free(&Z);
            }
        } else {
            mat Wp = param_mat(params, o.wp, fi, fi, bf16), bp = param_mat(params, o.bp, 1, fi, bf16);
            mat onesS = mat_new(ns, 1);
            for (int64_t u = 0; u < ns; ++u) onesS.a[u] = 1.0;
            Zp[l] = mat_new(ns, fi);                          /* Zp = X W_p + 1 b_p^T */
            mm_acc(&Zp[l], &X, 0, &Wp, 0, bf16);
            mm_acc(&Zp[l], &onesS, 0, &bp, 0, bf16);
            Aagg[l] = mat_new(nd, fi);
            arg[l] = (int32_t*)malloc(sizeof(int32_t) * (size_t)(nd * fi > 0 ? nd * fi : 1));
            for (int64_t v = 0; v < nd; ++v)
                for (int64_t f = 0; f < fi; ++f) {
                    double best = 0.0; int32_t a = -1;
                    for (int64_t e = B->indptr[v]; e < B->indptr[v + 1]; ++e) {
                        double z = AT(Zp[l], B->indices[e], f);
                        z = z > 0.0 ? z : 0.0;               /* ReLU */
                        if (a < 0 || z > best) { best = z; a = B->indices[e]; }
                    }
                    AT(Aagg[l], v, f) = best;
                    arg[l][v * fi + f] = a;
                }
            mm_acc(&S, &Aagg[l], 0, &Wn, 0, bf16);
            mat_free(&Wp); mat_free(&bp); mat_free(&onesS);
        }
        if (g_ties && l < L - 1) {
            /* M = the same sum over magnitudes: |X_d||W_s| + |A||W_n| (or D+ P |X||W_n|) + |b| */
            mat Mg = mat_new(nd, fo);
            mm_acc_abs(&Mg, &Xd, 0, &Ws, 0, bf16);
            mm_acc_abs(&Mg, &ones, 0, &bb, 0, bf16);
            if (!pool && projf[l]) {
                mat Za = mat_new(ns, fo);
                mm_acc_abs(&Za, &X, 0, &Wn, 0, bf16);
                for (int64_t v = 0; v < nd; ++v) {
                    int64_t deg = B->indptr[v + 1] - B->indptr[v];
                    for (int64_t e = B->indptr[v]; e < B->indptr[v + 1]; ++e)
                        for (int64_t f = 0; f < fo; ++f)
                            AT(Mg, v, f) += sum ? AT(Za, B->indices[e], f) : AT(Za, B->indices[e], f) / (double)deg;
                }
                mat_free(&Za);
            } else {
                mat Aa = mat_new(nd, fi);
                for (int64_t t = 0; t < nd * fi; ++t) Aa.a[t] = fabs(Aagg[l].a[t]);
                mm_acc_abs(&Mg, &Aa, 0, &Wn, 0, bf16);
                mat_free(&Aa);
            }
            for (int64_t v = 0; v < nd; ++v)
                for (int64_t f = 0; f < fo; ++f) {
                    if (!(fabs(AT(S, v, f)) <= g_ties->tau * AT(Mg, v, f))) continue;
                    g_ties->found++;
                    if (g_ties->n < g_ties->cap) {
                        int64_t q = g_ties->n++;
                        g_ties->level[q] = l + 1; g_ties->v[q] = v; g_ties->j[q] = (int32_t)f;
                        g_ties->S[q] = AT(S, v, f); g_ties->M[q] = AT(Mg, v, f); g_ties->g[q] = 0.0;
                    }
                }
            mat_free(&Mg);
        }
        mat_free(&Ws); mat_free(&Wn); mat_free(&bb); mat_free(&ones);
        if (l < L - 1) {
            H[l + 1] = S;                                     /* ReLU; bf16: stored in bf16 */
            for (int64_t t = 0; t < nd * fo; ++t) {
                double h = S.a[t] > 0.0 ? S.a[t] : 0.0;
                H[l + 1].a[t] = bf16 ? bf16_round(h) : h;
            }
            S.a = NULL;
        }
    }

    /* softmax cross-entropy on the outputs of this micro-batch */
    const oblock* Bo = &mb[L - 1];
    const int64_t C = dims[L], no = Bo->n_dst;
    mat dS = mat_new(no, C);
    for (int64_t v = 0; v < no; ++v) {
        double mx = -INFINITY;
        for (int64_t c = 0; c < C; ++c) if (AT(S, v, c) > mx) mx = AT(S, v, c);
        double se = 0.0;
        for (int64_t c = 0; c < C; ++c) se += exp(AT(S, v, c) - mx);
        double lse = mx + log(se);
        int32_t y = labels[Bo->src_gid[v]];
        *loss += loss_scale * (lse - AT(S, v, y));
        for (int64_t c = 0; c < C; ++c)
            AT(dS, v, c) = loss_scale * (exp(AT(S, v, c) - lse) - (c == y ? 1.0 : 0.0));
        if (logits_out) for (int64_t c = 0; c < C; ++c) logits_out[v * C + c] = AT(S, v, c);
    }
    mat_free(&S);

    /* backward, layer L-1 down to 0 */
    for (int l = L - 1; l >= 0; --l) {
        const oblock* B = &mb[l];
        const int64_t fi = dims[l], fo = dims[l + 1], nd = B->n_dst, ns = B->n_src;
        int64_t lb = 0;
        for (int j = 0; j < l; ++j) lb = layer_offsets(dims, j, pool, lb).end;
        poff o = layer_offsets(dims, l, pool, lb);
        mat Ws = param_mat(params, o.ws, fi, fo, bf16), Wn = param_mat(params, o.wn, fi, fo, bf16);
        mat X = H[l];
        mat Xd = { nd, fi, X.a };
        mat gWs = mat_new(fi, fo), gWn = mat_new(fi, fo), gb = mat_new(1, fo);
        mat ones = mat_new(nd, 1);
        for (int64_t v = 0; v < nd; ++v) ones.a[v] = 1.0;
        mm_acc(&gWs, &Xd, 1, &dS, 0, bf16);                  /* dW_s += X_d^T dS */
        mm_acc(&gb, &ones, 1, &dS, 0, bf16);                 /* db += 1^T dS */
        mat dX = mat_new(ns, fi);
        if (l > 0) {
            mat dXd = { nd, fi, dX.a };
            mm_acc(&dXd, &dS, 0, &Ws, 1, bf16);              /* dX[0:nd] += dS W_s^T */
        }
        if (!pool && !projf[l]) {
            mm_acc(&gWn, &Aagg[l], 1, &dS, 0, bf16);         /* dW_n += A^T dS */
            if (l > 0) {
                mat dA = mat_new(nd, fi);
                mm_acc(&dA, &dS, 0, &Wn, 1, bf16);           /* dA = dS W_n^T */
                for (int64_t v = 0; v < nd; ++v) {           /* dX += P^T D+ dA */
                    int64_t deg = B->indptr[v + 1] - B->indptr[v];
                    for (int64_t e = B->indptr[v]; e < B->indptr[v + 1]; ++e)
                        for (int64_t f = 0; f < fi; ++f)
                            AT(dX, B->indices[e], f) += sum ? AT(dA, v, f) : AT(dA, v, f) / (double)deg;
                }
                mat_free(&dA);
            }
        } else if (!pool) {
            mat dZ = mat_new(ns, fo);                         /* dZ = P^T D+ dS */
            for (int64_t v = 0; v < nd; ++v) {
                int64_t deg = B->indptr[v + 1] - B->indptr[v];
                for (int64_t e = B->indptr[v]; e < B->indptr[v + 1]; ++e)
                    for (int64_t f = 0; f < fo; ++f)
                        AT(dZ, B->indices[e], f) += sum ? AT(dS, v, f) : AT(dS, v, f) / (double)deg;
            }
            mm_acc(&gWn, &X, 1, &dZ, 0, bf16);               /* dW_n += X^T dZ */
            if (l > 0) mm_acc(&dX, &dZ, 0, &Wn, 1, bf16);    /* dX += dZ W_n^T */
            mat_free(&dZ);
        } else {
            mat Wp = param_mat(params, o.wp, fi, fi, bf16);
            mm_acc(&gWn, &Aagg[l], 1, &dS, 0, bf16);         /* dW_n += A^T dS */
            mat dA = mat_new(nd, fi);
            mm_acc(&dA, &dS, 0, &Wn, 1, bf16);
            mat dZp = mat_new(ns, fi);
            for (int64_t v = 0; v < nd; ++v)                  /* route to the argmax */
                for (int64_t f = 0; f < fi; ++f) {
                    int32_t a = arg[l][v * fi + f];
                    if (a >= 0) AT(dZp, a, f) += AT(dA, v, f);
                }
            for (int64_t t = 0; t < ns * fi; ++t) if (!(Zp[l].a[t] > 0.0)) dZp.a[t] = 0.0;  /* ReLU' */
            mat gWp = mat_new(fi, fi), gbp = mat_new(1, fi);
            mat onesS = mat_new(ns, 1);
            for (int64_t u = 0; u < ns; ++u) onesS.a[u] = 1.0;
            mm_acc(&gWp, &X, 1, &dZp, 0, bf16);              /* dW_p += X^T dZp */
            mm_acc(&gbp, &onesS, 1, &dZp, 0, bf16);          /* db_p += 1^T dZp */
            if (l > 0) mm_acc(&dX, &dZp, 0, &Wp, 1, bf16);   /* dX += dZp W_p^T */
            for (int64_t t = 0; t < fi * fi; ++t) grad[o.wp + t] += gWp.a[t];
            for (int64_t t = 0; t < fi; ++t) grad[o.bp + t] += gbp.a[t];
            mat_free(&Wp); mat_free(&dA); mat_free(&dZp); mat_free(&gWp); mat_free(&gbp); mat_free(&onesS);
        }
        for (int64_t t = 0; t < fi * fo; ++t) { grad[o.ws + t] += gWs.a[t]; grad[o.wn + t] += gWn.a[t]; }
        for (int64_t t = 0; t < fo; ++t) grad[o.b + t] += gb.a[t];
        mat_free(&Ws); mat_free(&Wn); mat_free(&gWs); mat_free(&gWn); mat_free(&gb); mat_free(&ones);
        mat_free(&dS);
        if (l > 0) {                                          /* dS_{l-1} = dX (.) [H_l > 0] */
            if (g_ties)
                for (int64_t q = 0; q < g_ties->n; ++q)
                    if (g_ties->level[q] == l) g_ties->g[q] = AT(dX, g_ties->v[q], g_ties->j[q]);
            for (int64_t t = 0; t < ns * fi; ++t) if (!(X.a[t] > 0.0)) dX.a[t] = 0.0;
            dS = dX;
        } else {
            mat_free(&dX);
        }
    }

    for (int l = 0; l <= L; ++l) mat_free(&H[l]);
    for (int l = 0; l < L; ++l) { mat_free(&Aagg[l]); mat_free(&Zp[l]); free(arg[l]); }
    free(H); free(Aagg); free(Zp); free(arg); free(projf);
    return 0;
}

/* oracle_sage plus the report of the hidden ReLU decisions within tau of the
 * boundary (reading #24): up to cap entries (level, v, j, S, M, g); returns
 * the number of such decisions (if it exceeds cap only the first cap are stored). */
int64_t oracle_sage_ties(int L, const int32_t* dims, int aggr, int bf16, const oblock* mb, const double* params,
                         const float* feats, int64_t ld, const int32_t* labels, double loss_scale, double* grad,
                         double* loss, double tau, int64_t cap, int32_t* level, int64_t* v, int32_t* j, double* S,
                         double* M, double* g) {
    tie_report r = {tau, cap, 0, 0, level, v, j, S, M, g};
    g_ties = &r;
    oracle_sage(L, dims, aggr, bf16, -1, mb, params, feats, ld, labels, loss_scale, grad, loss, NULL);
    g_ties = NULL;
    return r.found;
}

/* ------------------------------------------------------------------------ */
/* One batch (Fig. 6): for every micro-batch k in ks[],
 * extract it and add its gradient and loss.  grad[] / *loss are accumulated
 * (+=) in micro-batch order. */
int oracle_step(int L, const int32_t* dims, int aggr, int bf16, const oblock* full, const int32_t* part,
                int64_t n_out, int32_t K, const int32_t* ks, int32_t n_ks, const double* params,
                const float* feats, int64_t ld, const int32_t* labels, double loss_scale,
                double* grad, double* loss) {
    oblock* mb = (oblock*)calloc((size_t)L, sizeof(oblock));
    for (int32_t t = 0; t < n_ks; ++t) {
        if (oracle_extract(L, full, part, n_out, K, ks[t], mb) != 0) { free(mb); return -1; }
        oracle_sage(L, dims, aggr, bf16, -1, mb, params, feats, ld, labels, loss_scale, grad, loss, NULL);
        oracle_block_free(mb, L);
    }
    free(mb);
    return 0;
}

/* ------------------------------------------------------------------------ */
/* Memory estimate of one micro-batch, "Partition memory estimation"
 * (§4.4, notation Table 3).
 * Element counts, written in the paper's order:
 *   t[0] (1) N_P_GNN              parameters without the aggregator's (W_self,
 *                                 W_neigh, b of every layer; reading M3)
 *   t[1] (2) N_in x H_in          input features: n_src of layer 0 x dims[0]
 *   t[2] (3) N_out                output labels: n_dst of layer L-1
 *   t[3] (4) sum over blocks E x 3 "two node IDs ... and a weight" per edge
 *
 *   t[4] (5) sum_i N_i x h_i      every layer's output, n_dst,l x dims[l+1]
 *                                 (reading M1)
 *   t[5] (6) aggregator intermediates: the paper gives only LSTM's (Eq. 5);
 *                                 mean: sum_l n_dst,l x dims[l] (h_N); pool:
 *                                 sum_l (n_src,l + n_dst,l) x dims[l]
 *                                 (fc_pool output + max) (reading M2)
 *   t[6] (7) N_P_GNN + N_P_Agg    gradients
 *   t[7] (8) 2 (N_P_GNN + N_P_Agg) Adam's momentum and variance
 *   t[8] peak = (1)+(2)+(3)+(4)+(5)+(8) + max((6), (7)): "(6) can be freed
 *        during the backward propagation where ... (7) starts to dominate ...
 *        the peak memory consumption comes from the maximum of (6) and (7)
 *        plus other tensors".
 * Sizes per layer l: n_dst[l], n_src[l], n_edges[l].  Bytes = 4 x elements
 * (reading M4).  Returns 0. */
int oracle_mem_estimate(int L, const int32_t* dims, int aggr, const int64_t* n_dst, const int64_t* n_src,
                        const int64_t* n_edges, int64_t* t) {
    int64_t np_gnn = 0, np_agg = 0;
    for (int l = 0; l < L; ++l) {
        int64_t fi = dims[l], fo = dims[l + 1];
        np_gnn += 2 * fi * fo + fo;                /* W_self, W_neigh, b */
        if (aggr == 1) np_agg += fi * fi + fi;     /* W_pool, b_pool */
    }
    for (int q = 0; q < 9; ++q) t[q] = 0;
    t[0] = np_gnn;
    t[1] = n_src[0] * dims[0];
    t[2] = n_dst[L - 1];
    for (int l = 0; l < L; ++l) t[3] += n_edges[l] * 3;
    for (int l = 0; l < L; ++l) t[4] += n_dst[l] * dims[l + 1];
    for (int l = 0; l < L; ++l) t[5] += (aggr == 1 ? n_src[l] + n_dst[l] : n_dst[l]) * dims[l];
    t[6] = np_gnn + np_agg;
    t[7] = 2 * (np_gnn + np_agg);
    t[8] = t[0] + t[1] + t[2] + t[3] + t[4] + t[7] + (t[5] > t[6] ? t[5] : t[6]);
    return 0;
}
