/*
 * synth/gen.c -- seeded synthetic INPUT generator shared by the CUDA path and
 * the CPU oracle.  It holds none of Betty's arithmetic (no REG, no
 * micro-batch extraction, no SAGE): it only produces
 *   (1) a degree-corrected SBM power-law graph shaped like the paper's datasets
 *       (Table 4), as a symmetric CSR without self loops;
 *   (2) node features and labels;
 *   (3) the training seeds (output nodes) of one large batch;
 *   (4) the canonical FULL-BATCH sampled blocks (DGL-style neighbour sampling
 *       with a fanout bound, §2.1; the artifact samples the
 *       full batch once, PAPER.md:1893-1897 A.4).  Sampling is the input to the
 *       method, outside its hot path.
 *
 * Every random draw is a counter-based hash (splitmix64 finaliser), so the
 * result is independent of the OpenMP thread count.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#ifdef _OPENMP
#include <omp.h>
#endif

static inline uint64_t sm_mix(uint64_t z) {
    z += 0x9e3779b97f4a7c15ULL;
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
    return z ^ (z >> 31);
}
static inline uint64_t key3(uint64_t a, uint64_t b, uint64_t c) {
    return sm_mix(sm_mix(sm_mix(a) ^ b) ^ c);
}
static inline double u01(uint64_t r) { return (double)(r >> 11) * (1.0 / 9007199254740992.0); }

/* smallest i in [0,n) with cum[i] > x (cum strictly increasing, cum[n-1] > x) */
static inline int64_t cdf_search(const double* cum, int64_t n, double x) {
    int64_t lo = 0, hi = n - 1;
    while (lo < hi) {
        int64_t mid = lo + ((hi - lo) >> 1);
        if (cum[mid] > x) hi = mid; else lo = mid + 1;
    }
    return lo;
}

typedef struct { uint64_t k; int64_t i; } kv_t;
static int cmp_kv(const void* a, const void* b) {
    const kv_t* x = (const kv_t*)a; const kv_t* y = (const kv_t*)b;
    if (x->k != y->k) return x->k < y->k ? -1 : 1;
    return x->i < y->i ? -1 : (x->i > y->i);
}
static int cmp_i32(const void* a, const void* b) {
    int32_t x = *(const int32_t*)a, y = *(const int32_t*)b;
    return (x > y) - (x < y);
}
static void sort_i32(int32_t* a, int64_t n) {
    if (n < 24) {                         /* insertion sort for short rows */
        for (int64_t i = 1; i < n; ++i) {
            int32_t v = a[i]; int64_t j = i - 1;
            while (j >= 0 && a[j] > v) { a[j + 1] = a[j]; --j; }
            a[j + 1] = v;
        }
    } else {
        qsort(a, (size_t)n, sizeof(int32_t), cmp_i32);
    }
}

void synth_free(void* p) { free(p); }

int synth_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/*
 * DC-SBM with Chung-Lu weights w = (rank+1)^(-beta), rank a seeded random
 * permutation; communities uniform; a fraction mu of edge endpoints is drawn
 * globally, the rest inside the first endpoint's community.  M candidate
 * pairs are drawn, self loops dropped, then the graph is symmetrised and
 * deduplicated.  Returns the number of CSR entries (= 2 x undirected pairs),
 * or -1 on allocation failure.  comm_out[N] receives the community ids.
 */
int64_t synth_graph(int64_t N, int64_t M, int32_t n_comm, double mu, double beta, uint64_t seed,
                    int64_t** indptr_out, int32_t** indices_out, int32_t* comm_out) {
    int32_t* comm = comm_out;
    double* w = (double*)malloc(sizeof(double) * N);
    kv_t* kv = (kv_t*)malloc(sizeof(kv_t) * N);
    if (!w || !kv) return -1;
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < N; ++i) {
        comm[i] = (int32_t)(key3(seed, 11, (uint64_t)i) % (uint64_t)n_comm);
        kv[i].k = key3(seed, 12, (uint64_t)i); kv[i].i = i;
    }
    qsort(kv, (size_t)N, sizeof(kv_t), cmp_kv);
    for (int64_t r = 0; r < N; ++r) w[kv[r].i] = pow((double)(r + 1), -beta);
    free(kv);

    double* cum = (double*)malloc(sizeof(double) * N);
    int64_t* coff = (int64_t*)calloc((size_t)n_comm + 1, sizeof(int64_t));
    int32_t* cmem = (int32_t*)malloc(sizeof(int32_t) * N);
    double* ccum = (double*)malloc(sizeof(double) * N);
    if (!cum || !coff || !cmem || !ccum) return -1;
    double acc = 0.0;
    for (int64_t i = 0; i < N; ++i) { acc += w[i]; cum[i] = acc; }
    const double total = acc;
    for (int64_t i = 0; i < N; ++i) coff[comm[i] + 1]++;
    for (int32_t c = 0; c < n_comm; ++c) coff[c + 1] += coff[c];
    {
        int64_t* cur = (int64_t*)malloc(sizeof(int64_t) * n_comm);
        memcpy(cur, coff, sizeof(int64_t) * n_comm);
        for (int64_t i = 0; i < N; ++i) cmem[cur[comm[i]]++] = (int32_t)i;
        free(cur);
    }
    for (int32_t c = 0; c < n_comm; ++c) {
        double a = 0.0;
        for (int64_t j = coff[c]; j < coff[c + 1]; ++j) { a += w[cmem[j]]; ccum[j] = a; }
    }

    int32_t* eu = (int32_t*)malloc(sizeof(int32_t) * M);
    int32_t* ev = (int32_t*)malloc(sizeof(int32_t) * M);
    if (!eu || !ev) return -1;
    #pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < M; ++e) {
        int64_t u = cdf_search(cum, N, u01(key3(seed, 13, (uint64_t)e)) * total);
        int64_t v;
        if (u01(key3(seed, 14, (uint64_t)e)) < mu) {
            v = cdf_search(cum, N, u01(key3(seed, 15, (uint64_t)e)) * total);
        } else {
            int32_t c = comm[u];
            int64_t n_c = coff[c + 1] - coff[c];
            const double* cc = ccum + coff[c];
            v = cmem[coff[c] + cdf_search(cc, n_c, u01(key3(seed, 15, (uint64_t)e)) * cc[n_c - 1])];
        }
        if (u == v) { eu[e] = -1; ev[e] = -1; }
        else { eu[e] = (int32_t)u; ev[e] = (int32_t)v; }
    }
    free(w); free(cum); free(coff); free(cmem); free(ccum);

    int64_t* deg = (int64_t*)calloc((size_t)N + 1, sizeof(int64_t));
    #pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < M; ++e) {
        if (eu[e] < 0) continue;
        #pragma omp atomic
        deg[eu[e] + 1]++;
        #pragma omp atomic
        deg[ev[e] + 1]++;
    }
    for (int64_t i = 0; i < N; ++i) deg[i + 1] += deg[i];
    int64_t raw_n = deg[N];
    int32_t* raw = (int32_t*)malloc(sizeof(int32_t) * (raw_n > 0 ? raw_n : 1));
    int64_t* cur = (int64_t*)malloc(sizeof(int64_t) * N);
    memcpy(cur, deg, sizeof(int64_t) * N);
    #pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < M; ++e) {
        if (eu[e] < 0) continue;
        int64_t p, q;
        #pragma omp atomic capture
        p = cur[eu[e]]++;
        #pragma omp atomic capture
        q = cur[ev[e]]++;
        raw[p] = ev[e]; raw[q] = eu[e];
    }
    free(eu); free(ev); free(cur);

    int64_t* nd = (int64_t*)calloc((size_t)N + 1, sizeof(int64_t));
    #pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t i = 0; i < N; ++i) {
        int32_t* r = raw + deg[i];
        int64_t n = deg[i + 1] - deg[i];
        sort_i32(r, n);
        int64_t m = 0;
        for (int64_t j = 0; j < n; ++j) if (j == 0 || r[j] != r[j - 1]) r[m++] = r[j];
        nd[i + 1] = m;
    }
    for (int64_t i = 0; i < N; ++i) nd[i + 1] += nd[i];
    int64_t nnz = nd[N];
    int32_t* ind = (int32_t*)malloc(sizeof(int32_t) * (nnz > 0 ? nnz : 1));
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < N; ++i)
        memcpy(ind + nd[i], raw + deg[i], sizeof(int32_t) * (size_t)(nd[i + 1] - nd[i]));
    free(raw); free(deg);
    *indptr_out = nd; *indices_out = ind;
    return nnz;
}

static inline double gauss(uint64_t seed, uint64_t a, uint64_t b) {
    double u1 = u01(key3(seed, a, 2 * b)) + 1e-300;
    double u2 = u01(key3(seed, a, 2 * b + 1));
    return sqrt(-2.0 * log(u1)) * cos(6.283185307179586 * u2);
}

/* kind 0: N(0,1) + signal * community centroid (centroid ~ N(0,1) per (c,f));
 * kind 1: sparse 0/1 bag of words, Bernoulli(p) with community-specific words
 *         4x more likely (Cora-shaped).  Padding columns [F, ld) are zero.
 * Row i is a pure function of (seed, node id, its community), so any subset of
 * rows can be generated on its own (synth_features_ids). */
static void feature_row(int64_t node, int32_t c, int32_t F, int64_t ld, int32_t kind, double signal, double p,
                        uint64_t seed, float* row) {
    for (int32_t f = 0; f < F; ++f) {
        if (kind == 0) {
            double v = gauss(seed, (uint64_t)node + 1000, (uint64_t)f) +
                       signal * gauss(seed ^ 0xC0FFEEULL, (uint64_t)c, (uint64_t)f);
            row[f] = (float)v;
        } else {
            double pf = ((f * 7 + c) % 16 == 0) ? 4.0 * p : 0.8 * p;
            row[f] = u01(key3(seed, (uint64_t)node + 7, (uint64_t)f)) < pf ? 1.0f : 0.0f;
        }
    }
    for (int64_t f = F; f < ld; ++f) row[f] = 0.0f;
}

void synth_features(int64_t N, int32_t F, int64_t ld, const int32_t* comm, int32_t kind,
                    double signal, double p, uint64_t seed, float* out) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < N; ++i) feature_row(i, comm[i], F, ld, kind, signal, p, seed, out + i * ld);
}

/* rows of the nodes ids[0..n) (ids == NULL: nodes row0 .. row0+n-1); comm is
 * indexed by node id.  Row j of out is node ids[j]'s row of synth_features. */
void synth_features_ids(const int32_t* ids, int64_t row0, int64_t n, int32_t F, int64_t ld, const int32_t* comm,
                        int32_t kind, double signal, double p, uint64_t seed, float* out) {
    #pragma omp parallel for schedule(static)
    for (int64_t j = 0; j < n; ++j) {
        const int64_t node = ids ? (int64_t)ids[j] : row0 + j;
        feature_row(node, comm[node], F, ld, kind, signal, p, seed, out + j * ld);
    }
}

/* n_out distinct training seeds: the n_out smallest hash keys, returned in
 * ascending node id. */
void synth_seeds(int64_t N, int64_t n_out, uint64_t seed, int32_t* out) {
    kv_t* kv = (kv_t*)malloc(sizeof(kv_t) * N);
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < N; ++i) { kv[i].k = key3(seed, 21, (uint64_t)i); kv[i].i = i; }
    qsort(kv, (size_t)N, sizeof(kv_t), cmp_kv);
    for (int64_t j = 0; j < n_out; ++j) out[j] = (int32_t)kv[j].i;
    free(kv);
    sort_i32(out, n_out);
}

/*
 * Multi-layer full-batch neighbour sampling.
 * Blocks are numbered l = 0 (input) .. L-1 (output).  The dst list of block
 * L-1 is `seeds`; the dst list of block l-1 is the src list of block l.
 * For block l each dst v keeps all in-neighbours if deg(v) <= fanout[l] (or
 * fanout[l] < 0), else the fanout[l] candidates with the smallest keys
 * key3(seed ^ l, v, p) (ties by row position p; without replacement).  Each
 * row is sorted by ascending global id.  src = dst ++ (new neighbours in
 * ascending global id); edges are stored as full-batch src positions.
 * Output arrays are malloc'd; the caller frees them with synth_free.
 */
typedef struct {
    int64_t n_dst, n_src, n_edges;
    int64_t* indptr;     /* [n_dst+1] */
    int32_t* nbr_pos;    /* [n_edges] */
    int32_t* src_gid;    /* [n_src] */
} synth_block;

int synth_sample(int64_t N, const int64_t* gindptr, const int32_t* gind,
                 int64_t n_seeds, const int32_t* seeds, int32_t L, const int32_t* fanout,
                 uint64_t seed, synth_block* out /* [L] */) {
    int32_t* map = (int32_t*)malloc(sizeof(int32_t) * N);
    uint8_t* flag = (uint8_t*)calloc((size_t)N, 1);
    if (!map || !flag) return -1;
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < N; ++i) map[i] = -1;

    int64_t n_dst = n_seeds;
    int32_t* dst_gid = (int32_t*)malloc(sizeof(int32_t) * (n_seeds > 0 ? n_seeds : 1));
    memcpy(dst_gid, seeds, sizeof(int32_t) * n_seeds);

    for (int32_t l = L - 1; l >= 0; --l) {
        const int32_t f = fanout[l];
        int64_t* ip = (int64_t*)malloc(sizeof(int64_t) * (n_dst + 1));
        ip[0] = 0;
        #pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < n_dst; ++i) {
            int64_t d = gindptr[dst_gid[i] + 1] - gindptr[dst_gid[i]];
            ip[i + 1] = (f < 0 || d <= f) ? d : f;
        }
        for (int64_t i = 0; i < n_dst; ++i) ip[i + 1] += ip[i];
        const int64_t E = ip[n_dst];
        int32_t* nbr = (int32_t*)malloc(sizeof(int32_t) * (E > 0 ? E : 1));
        #pragma omp parallel
        {
            int64_t cap = 0; kv_t* buf = NULL;
            #pragma omp for schedule(dynamic, 256)
            for (int64_t i = 0; i < n_dst; ++i) {
                const int32_t v = dst_gid[i];
                const int64_t b = gindptr[v], d = gindptr[v + 1] - b;
                int32_t* o = nbr + ip[i];
                if (f < 0 || d <= f) { memcpy(o, gind + b, sizeof(int32_t) * d); continue; }
                if (d > cap) { cap = d; buf = (kv_t*)realloc(buf, sizeof(kv_t) * cap); }
                const uint64_t hv = sm_mix(sm_mix(seed ^ (uint64_t)l) ^ (uint64_t)v);
                for (int64_t p = 0; p < d; ++p) { buf[p].k = sm_mix(hv ^ (uint64_t)p); buf[p].i = p; }
                qsort(buf, (size_t)d, sizeof(kv_t), cmp_kv);
                for (int32_t j = 0; j < f; ++j) o[j] = gind[b + buf[j].i];
                sort_i32(o, f);
            }
            free(buf);
        }
        /* src list: dst prefix, then unseen neighbours in ascending global id */
        #pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < n_dst; ++i) map[dst_gid[i]] = (int32_t)i;
        #pragma omp parallel for schedule(static)
        for (int64_t e = 0; e < E; ++e) if (map[nbr[e]] < 0) flag[nbr[e]] = 1;
        int64_t n_new = 0;
        for (int64_t g = 0; g < N; ++g) n_new += flag[g];
        const int64_t n_src = n_dst + n_new;
        int32_t* src_gid = (int32_t*)malloc(sizeof(int32_t) * (n_src > 0 ? n_src : 1));
        memcpy(src_gid, dst_gid, sizeof(int32_t) * n_dst);
        int64_t pos = n_dst;
        for (int64_t g = 0; g < N; ++g)
            if (flag[g]) { flag[g] = 0; map[g] = (int32_t)pos; src_gid[pos++] = (int32_t)g; }
        #pragma omp parallel for schedule(static)
        for (int64_t e = 0; e < E; ++e) nbr[e] = map[nbr[e]];
        #pragma omp parallel for schedule(static)
        for (int64_t s = 0; s < n_src; ++s) map[src_gid[s]] = -1;

        out[l].n_dst = n_dst; out[l].n_src = n_src; out[l].n_edges = E;
        out[l].indptr = ip; out[l].nbr_pos = nbr; out[l].src_gid = src_gid;
        free(dst_gid);
        dst_gid = (int32_t*)malloc(sizeof(int32_t) * (n_src > 0 ? n_src : 1));
        memcpy(dst_gid, src_gid, sizeof(int32_t) * n_src);
        n_dst = n_src;
    }
    free(dst_gid); free(map); free(flag);
    return 0;
}
