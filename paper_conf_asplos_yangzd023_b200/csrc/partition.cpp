// partition.cpp -- host-side K-way partitioner of the REG (outside the hot
// path: Alg. 1 line 8, uses METIS; METIS is not available in
// this image).  Greedy graph growing, the initial-partitioning
// scheme of multilevel partitioners: each part grows from the lowest-id
// unassigned output by repeatedly absorbing the unassigned output with the
// largest total REG weight to the part (= the most shared inputs, so the
// fewest duplicated inputs when it is cut off), up to a balanced size
// ceil-or-floor(n/K).  Deterministic (ties: smaller id).  Host pointers.
#include <cmath>
#include <cstdint>
#include <cstring>
#include <queue>
#include <utility>
#include <vector>
#include "../../include/betty.h"

extern "C" BETTY_API betty_status betty_reg_partition(const int64_t* indptr, const int32_t* col, const int32_t* w,
                                                      int64_t n, int32_t K, int32_t* part) {
    if (n < 0 || K < 1 || (n > 0 && (!indptr || !part))) return BETTY_EINVAL;
    if (n == 0) return BETTY_OK;
    std::vector<int64_t> gain(n, 0);
    std::vector<int32_t> touched;
    for (int64_t v = 0; v < n; ++v) part[v] = -1;
    int64_t next_seed = 0, done = 0;
    typedef std::pair<int64_t, int64_t> Item;           // (gain, -id): max-heap pops largest gain, then smallest id
    for (int32_t k = 0; k < K && done < n; ++k) {
        const int64_t target = (n * (k + 1)) / K - (n * k) / K;
        int64_t size = 0;
        std::priority_queue<Item> heap;
        while (size < target && done < n) {
            if (heap.empty()) {
                while (next_seed < n && part[next_seed] >= 0) ++next_seed;
                if (next_seed >= n) break;
                heap.push(Item(0, -next_seed));
            }
            Item it = heap.top();
            heap.pop();
            const int64_t v = -it.second;
            if (part[v] >= 0 || it.first != gain[v]) continue;   // stale entry
            part[v] = k;
            ++size;
            ++done;
            for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e) {
                const int32_t u = col[e];
                if (part[u] >= 0) continue;
                if (gain[u] == 0) touched.push_back(u);
                gain[u] += w ? w[e] : 1;
                heap.push(Item(gain[u], -(int64_t)u));
            }
        }
        for (int32_t u : touched) gain[u] = 0;
        touched.clear();
    }
    for (int64_t v = 0; v < n; ++v)
        if (part[v] < 0) part[v] = K - 1;
    return BETTY_OK;
}

// ---------------------------------------------------------------------------------------------
// Multilevel K-way partitioner (the METIS scheme the paper calls, Alg. 1 line 8 PAPER.md:941;
// SURVEY.md §8(f) #2), minimising the cut REG weight = the inputs duplicated across micro-batches
// (Eq. 4).  Host code, outside the hot path, deterministic:
//  1. coarsening by heavy-edge matching (vertices visited in a fixed hashed order, each matched to
//     its unmatched neighbour of largest edge weight, vertex weight capped) until the graph has
//     <= max(40 K, 1000) vertices or stops shrinking; parallel edges are merged (weights summed);
//  2. initial partition of the coarsest graph by weighted greedy graph growing (several starts,
//     the smallest cut wins);
//  3. uncoarsening: the partition is projected level by level and refined by greedy boundary
//     moves (largest cut reduction first, ties to the lighter part) under the balance bound
//     max part weight <= (1 + imbalance) * n / K, plus a rebalancing pass for overweight parts.
#include <algorithm>
#include <numeric>

namespace {
struct WGraph {
    int64_t n = 0;
    std::vector<int64_t> ip;      // [n+1]
    std::vector<int32_t> adj;     // neighbours (no self loops)
    std::vector<int64_t> ew;      // edge weights
    std::vector<int64_t> vw;      // vertex weights (outputs represented)
};

inline uint64_t mix64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

// heavy-edge matching; cmap[v] = coarse vertex of v; returns the coarse graph
WGraph coarsen(const WGraph& g, std::vector<int32_t>& cmap, int64_t max_vw, uint64_t seed) {
    const int64_t n = g.n;
    std::vector<int32_t> order(n), match(n, -1);
    std::iota(order.begin(), order.end(), 0);
    std::vector<uint64_t> key(n);
    for (int64_t v = 0; v < n; ++v) key[v] = mix64((uint64_t)v ^ seed);
    std::sort(order.begin(), order.end(), [&](int32_t a, int32_t b) { return key[a] < key[b]; });
    for (int32_t v : order) {
        if (match[v] >= 0) continue;
        int32_t best = -1;
        int64_t bw = -1;
        for (int64_t e = g.ip[v]; e < g.ip[v + 1]; ++e) {
            const int32_t u = g.adj[e];
            if (match[u] >= 0 || u == v || g.vw[u] + g.vw[v] > max_vw) continue;
            if (g.ew[e] > bw || (g.ew[e] == bw && u < best)) { bw = g.ew[e]; best = u; }
        }
        if (best >= 0) { match[v] = best; match[best] = v; }
        else match[v] = v;
    }
    cmap.assign(n, -1);
    int64_t nc = 0;
    for (int64_t v = 0; v < n; ++v) {            // coarse ids in order of the smaller member
        if (cmap[v] >= 0) continue;
        cmap[v] = (int32_t)nc;
        if (match[v] != v) cmap[match[v]] = (int32_t)nc;
        ++nc;
    }
    WGraph c;
    c.n = nc;
    c.vw.assign(nc, 0);
    for (int64_t v = 0; v < n; ++v) c.vw[cmap[v]] += g.vw[v];
    // members of each coarse vertex
    std::vector<int32_t> first(nc, -1), second(nc, -1);
    for (int64_t v = 0; v < n; ++v) {
        const int32_t cv = cmap[v];
        if (first[cv] < 0) first[cv] = (int32_t)v; else second[cv] = (int32_t)v;
    }
    c.ip.assign(nc + 1, 0);
    std::vector<int64_t> acc(nc, 0);
    std::vector<int32_t> mark(nc, -1), list;
    c.adj.reserve(g.adj.size() / 2 + 16);
    c.ew.reserve(g.adj.size() / 2 + 16);
    for (int64_t cv = 0; cv < nc; ++cv) {
        list.clear();
        for (int32_t v : {first[cv], second[cv]}) {
            if (v < 0) continue;
            for (int64_t e = g.ip[v]; e < g.ip[v + 1]; ++e) {
                const int32_t cu = cmap[g.adj[e]];
                if (cu == cv) continue;
                if (mark[cu] != cv) { mark[cu] = (int32_t)cv; acc[cu] = 0; list.push_back(cu); }
                acc[cu] += g.ew[e];
            }
        }
        std::sort(list.begin(), list.end());
        for (int32_t cu : list) { c.adj.push_back(cu); c.ew.push_back(acc[cu]); }
        c.ip[cv + 1] = (int64_t)c.adj.size();
    }
    return c;
}

int64_t cut_of(const WGraph& g, const std::vector<int32_t>& part) {
    int64_t cut = 0;
    for (int64_t v = 0; v < g.n; ++v)
        for (int64_t e = g.ip[v]; e < g.ip[v + 1]; ++e)
            if (part[g.adj[e]] != part[v]) cut += g.ew[e];
    return cut / 2;
}

// weighted greedy growing from `start` (then lowest unassigned ids); targets by vertex weight
void grow(const WGraph& g, int32_t K, int64_t start, std::vector<int32_t>& part) {
    const int64_t n = g.n;
    const int64_t total = std::accumulate(g.vw.begin(), g.vw.end(), (int64_t)0);
    part.assign(n, -1);
    std::vector<int64_t> gain(n, 0);
    std::vector<int32_t> touched, skip(n, -1);   // skip[v] = k: v would overshoot part k
    int64_t done_w = 0;
    bool first = true;
    typedef std::pair<int64_t, int64_t> Item;
    for (int32_t k = 0; k < K; ++k) {
        const int64_t target = (total * (k + 1)) / K - done_w;
        int64_t wsum = 0, next_seed = 0;
        std::priority_queue<Item> heap;
        while (wsum < target) {
            if (heap.empty()) {
                int64_t sv = -1;
                if (first && start >= 0 && start < n && part[start] < 0) sv = start;
                first = false;
                if (sv < 0) {
                    while (next_seed < n && (part[next_seed] >= 0 || skip[next_seed] == k)) ++next_seed;
                    if (next_seed >= n) break;
                    sv = next_seed;
                }
                heap.push(Item(gain[sv], -sv));
            }
            const Item it = heap.top();
            heap.pop();
            const int64_t v = -it.second;
            if (part[v] >= 0 || skip[v] == k || it.first != gain[v]) continue;
            if (wsum > 0 && wsum + g.vw[v] > target + g.vw[v] / 2) { skip[v] = k; continue; }   // would overshoot
            part[v] = k;
            wsum += g.vw[v];
            for (int64_t e = g.ip[v]; e < g.ip[v + 1]; ++e) {
                const int32_t u = g.adj[e];
                if (part[u] >= 0) continue;
                if (gain[u] == 0) touched.push_back(u);
                gain[u] += g.ew[e];
                heap.push(Item(gain[u], -(int64_t)u));
            }
        }
        done_w += wsum;
        for (int32_t u : touched) gain[u] = 0;
        touched.clear();
    }
    // leftovers (skipped by the overshoot rule): the lightest part each
    std::vector<int64_t> pw(K, 0);
    for (int64_t v = 0; v < n; ++v) if (part[v] >= 0) pw[part[v]] += g.vw[v];
    for (int64_t v = 0; v < n; ++v)
        if (part[v] < 0) {
            const int32_t k = (int32_t)(std::min_element(pw.begin(), pw.end()) - pw.begin());
            part[v] = k;
            pw[k] += g.vw[v];
        }
}

// greedy boundary refinement + rebalancing under max part weight maxpw
void refine(const WGraph& g, int32_t K, int64_t maxpw, std::vector<int32_t>& part, int passes) {
    const int64_t n = g.n;
    std::vector<int64_t> pw(K, 0);
    for (int64_t v = 0; v < n; ++v) pw[part[v]] += g.vw[v];
    std::vector<int64_t> conn(K, 0);
    std::vector<int32_t> seen;
    for (int pass = 0; pass < passes; ++pass) {
        int64_t moves = 0;
        for (int64_t v = 0; v < n; ++v) {
            const int32_t a = part[v];
            seen.clear();
            int64_t own = 0;
            bool boundary = false;
            for (int64_t e = g.ip[v]; e < g.ip[v + 1]; ++e) {
                const int32_t p = part[g.adj[e]];
                if (p == a) { own += g.ew[e]; continue; }
                boundary = true;
                if (conn[p] == 0) seen.push_back(p);
                conn[p] += g.ew[e];
            }
            const bool over = pw[a] > maxpw;
            if (!boundary && !over) continue;
            int32_t best = -1;
            int64_t bgain = 0;
            for (int32_t p : seen) {
                if (pw[p] + g.vw[v] > maxpw) continue;
                const int64_t gain = conn[p] - own;
                const bool better = best < 0 ? (gain > 0 || (gain == 0 && pw[p] + g.vw[v] < pw[a]) || over)
                                             : (gain > bgain || (gain == bgain && pw[p] < pw[best]));
                if (better) { best = p; bgain = gain; }
            }
            if (best < 0 && over) {                 // overweight part with no adjacent room: lightest part
                const int32_t p = (int32_t)(std::min_element(pw.begin(), pw.end()) - pw.begin());
                if (p != a && pw[p] + g.vw[v] <= maxpw) best = p;
            }
            for (int32_t p : seen) conn[p] = 0;
            if (best >= 0) {
                part[v] = best;
                pw[a] -= g.vw[v];
                pw[best] += g.vw[v];
                ++moves;
            }
        }
        if (moves == 0) break;
    }
}
}  // namespace

extern "C" BETTY_API betty_status betty_reg_partition_ex(const int64_t* indptr, const int32_t* col, const int32_t* w,
                                                         int64_t n, int32_t K, int32_t method, double imbalance,
                                                         int32_t* part) {
    if (n < 0 || K < 1 || imbalance < 0 || (n > 0 && (!indptr || !part))) return BETTY_EINVAL;
    if (method == BETTY_PART_GREEDY) return betty_reg_partition(indptr, col, w, n, K, part);
    if (method != BETTY_PART_MULTILEVEL) return BETTY_EINVAL;
    if (n == 0) return BETTY_OK;
    if (K == 1) { for (int64_t v = 0; v < n; ++v) part[v] = 0; return BETTY_OK; }
    // level 0: the REG itself (unit vertex weights)
    std::vector<WGraph> levels(1);
    WGraph& g0 = levels[0];
    g0.n = n;
    g0.ip.assign(indptr, indptr + n + 1);
    const int64_t nnz = indptr[n] - indptr[0];
    g0.adj.resize(nnz);
    g0.ew.resize(nnz);
    for (int64_t v = 0; v < n; ++v)
        for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e) {
            if (col[e] < 0 || col[e] >= n) return BETTY_EINVAL;
            g0.adj[e - indptr[0]] = col[e];
            g0.ew[e - indptr[0]] = w ? w[e] : 1;
        }
    for (int64_t v = 0; v <= n; ++v) g0.ip[v] -= indptr[0];
    g0.vw.assign(n, 1);
    const int64_t coarse_to = std::max<int64_t>(1000, 40 * (int64_t)K);
    const int64_t max_vw = std::max<int64_t>(1, (int64_t)(1.5 * (double)n / (double)coarse_to));
    std::vector<std::vector<int32_t>> cmaps;
    for (int lvl = 0; levels.back().n > coarse_to && lvl < 40; ++lvl) {
        std::vector<int32_t> cm;
        WGraph c = coarsen(levels.back(), cm, max_vw, (uint64_t)lvl * 7919u + 17u);
        if (c.n > levels.back().n * 0.95) break;      // stopped shrinking
        cmaps.push_back(std::move(cm));
        levels.push_back(std::move(c));
    }
    const int64_t maxpw = (int64_t)std::ceil((1.0 + imbalance) * (double)n / (double)K);
    // initial partition of the coarsest graph: several starts, best cut after refinement
    const WGraph& gc = levels.back();
    std::vector<int32_t> best, cur;
    int64_t best_cut = -1;
    const int tries = 8;
    for (int t = 0; t < tries; ++t) {
        const int64_t start = t == 0 ? 0 : (int64_t)(mix64((uint64_t)t) % (uint64_t)gc.n);
        grow(gc, K, start, cur);
        refine(gc, K, maxpw, cur, 10);
        const int64_t cut = cut_of(gc, cur);
        if (best_cut < 0 || cut < best_cut) { best_cut = cut; best = cur; }
    }
    // uncoarsen + refine
    for (int lvl = (int)levels.size() - 2; lvl >= 0; --lvl) {
        const std::vector<int32_t>& cm = cmaps[lvl];
        std::vector<int32_t> fine(levels[lvl].n);
        for (int64_t v = 0; v < levels[lvl].n; ++v) fine[v] = best[cm[v]];
        best.swap(fine);
        refine(levels[lvl], K, maxpw, best, 8);
    }
    for (int64_t v = 0; v < n; ++v) part[v] = best[v];
    return BETTY_OK;
}
