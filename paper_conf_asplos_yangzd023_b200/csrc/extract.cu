// extract.cu -- a2: micro-batch block extraction on the GPU.
//
// Batch-level partitioning (§4.2.3): micro-batch k keeps the
// outputs V_k = {i : part[i] == k}; layer by layer (output -> input) its dst
// list is the previous layer's src list and its src list is
//     U_k = dst ++ (sources of the dst rows not in dst, ascending full-batch
//            src position)                                 (readings #9/#10)
// with edges relabelled to local src ids and the local -> global index map
// (src_pos, src_gid) of PAPER.md:1167-1187.
//
// B200 design: a GROUP of c micro-batches is extracted by the same launches
// (block-diagonal union, each micro-batch with its own dedupe state).  The
// dedupe uses two bitmaps per micro-batch over the FULL-batch src positions of
// the layer (n_src_full/8 bytes each: 306 KB for the products shape, L2
// resident): `dstbits` marks the dst prefix, `newbits` the other sources.
// The ascending order of new sources then falls out of a popcount scan over
// the bitmap words -- no sort, no hash, no atomics-order dependence -- and a
// new source's local id is n_dst + (#set bits before it).  Only dst nodes
// need an explicit position -> local id map.  All sizes stay on the device.
//
// Group layout (what the SAGE kernels see): rows = the dst rows of all c
// micro-batches; src ids = [all dst rows (same order)] ++ [new sources of
// micro-batch 0] ++ [new of 1] ++ ..., so that dst ids remain a prefix of the
// src ids (the self term of SAGE needs it).  Per micro-batch this is exactly
// its canonical block under a renumbering; for c = 1 it IS the canonical block.
#include <cstring>
#include "common.cuh"
#include "internal.h"
#include "extract.h"

namespace betty {

// ----------------------------------------------------------- output select
// Output selection V_k (Alg. 1 line 9: the outputs of micro-batch k, ascending),
// for all c slots of a launch group at once, with the top layer's indptr and dst bitmap produced on
// the way.  Two passes over part[], one CTA per SEL_CHUNK-output chunk; an output's slot comes from
// a K-entry table in shared memory.  Pass 1 accumulates, per slot, the chunk's selected outputs and
// their top-layer degrees, packed as count << SEL_SHIFT | degree sum, so that ONE int64 scan gives
// both the dst positions and the indptr offsets.  Pass 2 (one warp per chunk, SEL_CHUNK / 32 steps
// of 32 outputs, ascending) writes each selected output's position, slot, indptr entry and dst bit.
constexpr int SEL_KMAX = 16384, SEL_CMAX = 512, SEL_SHIFT = 40;
constexpr int64_t SEL_DEG_MASK = (1ll << SEL_SHIFT) - 1;

__device__ __forceinline__ void sel_slot_table(int16_t* tab, const int32_t* __restrict__ ks, int c, int K) {
    for (int k = threadIdx.x; k < K; k += blockDim.x) tab[k] = -1;
    __syncthreads();
    for (int j = threadIdx.x; j < c; j += blockDim.x) tab[ks[j]] = (int16_t)j;
    __syncthreads();
}

__global__ void __launch_bounds__(256) k_sel_count(const int32_t* __restrict__ part, int64_t n_out, int32_t K,
                                                   const int32_t* __restrict__ ks, int32_t c,
                                                   const int64_t* __restrict__ findptr, int64_t* __restrict__ sel_cnt,
                                                   int64_t nchunks, int* dev_err) {
    __shared__ int16_t s_tab[SEL_KMAX];
    __shared__ unsigned long long s_acc[SEL_CMAX];
    sel_slot_table(s_tab, ks, c, K);
    for (int j = threadIdx.x; j < c; j += blockDim.x) s_acc[j] = 0ull;
    __syncthreads();
    const int64_t ch = blockIdx.x;
    const int64_t end = mn64((ch + 1) * SEL_CHUNK, n_out);
    constexpr int PER = SEL_CHUNK / 256;
    int32_t p[PER];
#pragma unroll
    for (int t = 0; t < PER; ++t) {                    // all loads in flight at once
        const int64_t i = ch * SEL_CHUNK + t * 256 + threadIdx.x;
        p[t] = i < end ? part[i] : -2;
    }
    int j[PER];
    int64_t d[PER];
#pragma unroll
    for (int t = 0; t < PER; ++t) {
        const int64_t i = ch * SEL_CHUNK + t * 256 + threadIdx.x;
        j[t] = -1;
        d[t] = 0;
        if (p[t] == -2) continue;
        if (p[t] < 0 || p[t] >= K) { atomicOr(dev_err, DEVERR_BAD_PART); continue; }
        j[t] = s_tab[p[t]];
        if (j[t] >= 0) d[t] = findptr[i + 1] - findptr[i];
    }
#pragma unroll
    for (int t = 0; t < PER; ++t)
        if (j[t] >= 0) atomicAdd(&s_acc[j[t]], (1ull << SEL_SHIFT) + (unsigned long long)d[t]);
    __syncthreads();
    for (int j = threadIdx.x; j < c; j += blockDim.x) sel_cnt[(int64_t)j * nchunks + ch] = (int64_t)s_acc[j];
}

__global__ void __launch_bounds__(32) k_sel_write(const int32_t* __restrict__ part, int64_t n_out, int32_t K,
                                                  const int32_t* __restrict__ ks, int32_t c,
                                                  const int64_t* __restrict__ findptr, const int64_t* __restrict__ off,
                                                  int64_t nchunks, int32_t* __restrict__ dst_pos,
                                                  int32_t* __restrict__ row_mb, int64_t* __restrict__ indptr,
                                                  int64_t cap_d, uint32_t* dstbits, int64_t W,
                                                  int64_t* __restrict__ mb_dst_off, int64_t* cnt, int* dev_err) {
    __shared__ int16_t s_tab[SEL_KMAX];
    __shared__ int64_t s_pos[SEL_CMAX], s_deg[SEL_CMAX];
    __shared__ int64_t s_d[32];
    sel_slot_table(s_tab, ks, c, K);
    const int lane = threadIdx.x;
    const int64_t ch = blockIdx.x;
    for (int j = lane; j < c; j += 32) {
        const int64_t o = off[(int64_t)j * nchunks + ch];
        s_pos[j] = o >> SEL_SHIFT;
        s_deg[j] = o & SEL_DEG_MASK;
    }
    if (ch == 0) {                                      // per-slot offsets, totals, indptr[n]
        for (int j = lane; j <= c; j += 32) mb_dst_off[j] = off[(int64_t)j * nchunks] >> SEL_SHIFT;
        if (lane == 0) {
            const int64_t t = off[(int64_t)c * nchunks], n = t >> SEL_SHIFT;
            if (n <= cap_d) {
                cnt[0] = n;
                cnt[2] = t & SEL_DEG_MASK;
                indptr[n] = t & SEL_DEG_MASK;
            } else {                                    // EOVERFLOW; the group runs empty (see k_counts)
                atomicOr(dev_err, DEVERR_OVERFLOW);
                cnt[0] = 0; cnt[2] = 0; indptr[0] = 0;
            }
        }
    }
    const int64_t base = ch * SEL_CHUNK;
    const int nloc = (int)mn64(SEL_CHUNK, n_out - base);
    // the chunk's slots and degrees first, every load in flight at once (lane = output of a step)
    constexpr int STEPS = SEL_CHUNK / 32;
    int32_t pp[STEPS], ds[STEPS];
#pragma unroll
    for (int t = 0; t < STEPS; ++t) {
        const int64_t i = base + t * 32 + lane;
        const bool in = t * 32 + lane < nloc;
        pp[t] = in ? part[i] : -1;
        ds[t] = in ? (int32_t)(findptr[i + 1] - findptr[i]) : 0;
    }
    int16_t js[STEPS];
#pragma unroll
    for (int t = 0; t < STEPS; ++t) js[t] = (pp[t] >= 0 && pp[t] < K) ? s_tab[pp[t]] : (int16_t)-1;
    __syncwarp();
#pragma unroll
    for (int t = 0; t < STEPS; ++t) {
        if (t * 32 >= nloc) break;
        const int64_t i = base + t * 32 + lane;
        const int j = js[t];
        const int64_t d = j >= 0 ? ds[t] : 0;
        const unsigned m = __match_any_sync(0xffffffffu, j);
        const unsigned lower = m & ((1u << lane) - 1u);
        s_d[lane] = d;
        __syncwarp();
        if (j >= 0) {
            int64_t db = 0;                             // degrees of the same slot's earlier outputs in this step
            for (unsigned b = lower; b; b &= b - 1u) db += s_d[__ffs(b) - 1];
            const int64_t pos = s_pos[j] + __popc(lower);
            if (pos < cap_d) {
                dst_pos[pos] = (int32_t)i;
                row_mb[pos] = j;
                indptr[pos] = s_deg[j] + db;
            }
            if (dstbits) atomicOr(&dstbits[(int64_t)j * W + (i >> 5)], 1u << (i & 31));
            __syncwarp(m);
            if (lane == 31 - __clz(m)) { s_pos[j] += __popc(m); s_deg[j] += db + d; }
        }
        __syncwarp();
    }
}

// ------------------------------------------------------------ per layer
__global__ void k_mark_dst(const int32_t* __restrict__ dst_pos, const int32_t* __restrict__ row_mb,
                           const int64_t* cnt, uint32_t* dstbits, int64_t W) {
    const int64_t n = cnt[0];
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
        const int j = row_mb[r];
        const int32_t p = dst_pos[r];
        atomicOr(&dstbits[j * W + (p >> 5)], 1u << (p & 31));
    }
}

// Rank words {bits, slot-relative popcount prefix} of c slots x W bitmap words, in two fully
// parallel passes (no look-back chain): chunk popcount sums, then each chunk adds the sums of
// the slot's earlier chunks and scans its own words.  slot_total[j] (optional) = set bits of j.
constexpr int RANK_THREADS = 256, RANK_ITEMS = 16, RANK_CHUNK = RANK_THREADS * RANK_ITEMS;
__global__ void __launch_bounds__(RANK_THREADS) k_rank_sums(const uint32_t* __restrict__ bits,
                                                             const uint32_t* __restrict__ mask, int64_t W,
                                                             int64_t* __restrict__ csum) {
    __shared__ int64_t s_warp[RANK_THREADS / 32 + 1];
    const int j = blockIdx.y;
    const int64_t c0 = (int64_t)blockIdx.x * RANK_CHUNK;
    const uint32_t* b = bits + (int64_t)j * W;
    const uint32_t* m = mask ? mask + (int64_t)j * W : nullptr;
    int64_t cnt = 0;
#pragma unroll
    for (int i = 0; i < RANK_ITEMS; ++i) {              // coalesced: word c0 + i * RANK_THREADS + t
        const int64_t w = c0 + i * RANK_THREADS + threadIdx.x;
        if (w < W) cnt += __popc(b[w] & (m ? ~m[w] : ~0u));
    }
    int64_t tot;
    block_excl_scan(cnt, s_warp, &tot);
    if (threadIdx.x == 0) csum[(int64_t)j * gridDim.x + blockIdx.x] = tot;
}
// padded shared index: thread t's 16 consecutive words fall in distinct banks
__device__ __forceinline__ int rpad(int w) { return w + (w >> 4); }
__global__ void __launch_bounds__(RANK_THREADS) k_rank_write(const uint32_t* __restrict__ bits,
                                                              const uint32_t* __restrict__ mask, int64_t W,
                                                              const int64_t* __restrict__ csum, uint2* __restrict__ out,
                                                              int64_t* __restrict__ slot_total) {
    __shared__ int64_t s_warp[RANK_THREADS / 32 + 1];
    __shared__ int64_t s_base;
    __shared__ uint32_t s_bits[RANK_CHUNK + RANK_CHUNK / 16], s_pre[RANK_CHUNK + RANK_CHUNK / 16];
    const int j = blockIdx.y;
    const int nch = gridDim.x;
    if (threadIdx.x < 32) {                             // sums of the slot's earlier chunks (and all of them)
        int64_t pre = 0, all = 0;
        for (int q = threadIdx.x; q < nch; q += 32) {
            const int64_t v = csum[(int64_t)j * nch + q];
            all += v;
            if (q < (int)blockIdx.x) pre += v;
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            pre += __shfl_xor_sync(0xffffffffu, pre, o);
            all += __shfl_xor_sync(0xffffffffu, all, o);
        }
        if (threadIdx.x == 0) {
            s_base = pre;
            if (slot_total && blockIdx.x == 0) slot_total[j] = all;
        }
    }
    const int64_t c0 = (int64_t)blockIdx.x * RANK_CHUNK;
    const uint32_t* b = bits + (int64_t)j * W;
    const uint32_t* m = mask ? mask + (int64_t)j * W : nullptr;
#pragma unroll
    for (int i = 0; i < RANK_ITEMS; ++i) {              // coalesced load -> shared
        const int wl = i * RANK_THREADS + threadIdx.x;
        const int64_t w = c0 + wl;
        s_bits[rpad(wl)] = w < W ? b[w] & (m ? ~m[w] : ~0u) : 0u;
    }
    __syncthreads();
    uint32_t v[RANK_ITEMS];
    int64_t cnt = 0;
#pragma unroll
    for (int i = 0; i < RANK_ITEMS; ++i) { v[i] = s_bits[rpad(threadIdx.x * RANK_ITEMS + i)]; cnt += __popc(v[i]); }
    int64_t tot;
    const int64_t ex = block_excl_scan(cnt, s_warp, &tot);    // (syncs: s_base visible)
    uint32_t run = (uint32_t)(s_base + ex);
#pragma unroll
    for (int i = 0; i < RANK_ITEMS; ++i) { s_pre[rpad(threadIdx.x * RANK_ITEMS + i)] = run; run += __popc(v[i]); }
    __syncthreads();
    uint2* o = out + (int64_t)j * W;
#pragma unroll
    for (int i = 0; i < RANK_ITEMS; ++i) {              // coalesced store
        const int wl = i * RANK_THREADS + threadIdx.x;
        const int64_t w = c0 + wl;
        if (w < W) o[w] = make_uint2(s_bits[rpad(wl)], s_pre[rpad(wl)]);
    }
}
// bits & ~mask (mask optional)
static void slot_rank(const uint32_t* bits, const uint32_t* mask, int32_t c, int64_t W, int64_t* csum, uint2* out,
                      int64_t* slot_total, cudaStream_t s) {
    const dim3 g((unsigned)std::max<int64_t>(1, (W + RANK_CHUNK - 1) / RANK_CHUNK), (unsigned)c);
    k_rank_sums<<<g, RANK_THREADS, 0, s>>>(bits, mask, W, csum);
    k_rank_write<<<g, RANK_THREADS, 0, s>>>(bits, mask, W, csum, out, slot_total);
}

// Local ids without a map.  Slot j's src list at layer l is [dst rows of layer l] ++ [new
// sources, ascending position]; its dst rows ARE its src list at layer l+1 (same positions),
// and at the top layer its outputs in ascending position.  So for a source p of slot j:
//   new at layer l           -> n_dst(l) + off_l(j) + rank of p in j's new bitmap of layer l
//   else new at layer q > l  -> the same at layer q (first such q)
//   else (an output)         -> top_off(j) + rank of p in j's output bitmap
struct RankSet {
    const uint2* nr[16];
    int64_t W[16];
    const int64_t* cnt[16];     // layer counts (cnt[0] = group dst total)
    const int64_t* off[16];     // per-slot offsets of the new sources
    const uint2* dr;            // top layer output bitmap ranks
    int64_t Wt;
    const int64_t* top_off;
    int L;
};
__device__ __forceinline__ int64_t rank_in(uint2 r, int32_t p) {
    return (int64_t)r.y + __popc(r.x & ((1u << (p & 31)) - 1u));
}
// nr_l: the caller's (already loaded) word of layer l's new-rank array for (j, p)
__device__ __forceinline__ int64_t src_id(const RankSet& R, int l, int j, int32_t p, uint2 nr_l) {
    const uint32_t bit = 1u << (p & 31);
    if (nr_l.x & bit) return R.cnt[l][0] + R.off[l][j] + rank_in(nr_l, p);
    for (int q = l + 1; q < R.L; ++q) {
        const uint2 nr = R.nr[q][(int64_t)j * R.W[q] + (p >> 5)];
        if (nr.x & bit) return R.cnt[q][0] + R.off[q][j] + rank_in(nr, p);
    }
    return R.top_off[j] + rank_in(R.dr[(int64_t)j * R.Wt + (p >> 5)], p);
}
// id of dst row q of slot j at layer l (= its src id at layer l + 1, or its output rank)
__device__ __forceinline__ int64_t dst_id(const RankSet& R, int l, int j, int32_t q) {
    if (l + 1 >= R.L) return R.top_off[j] + rank_in(R.dr[(int64_t)j * R.Wt + (q >> 5)], q);
    return src_id(R, l + 1, j, q, R.nr[l + 1][(int64_t)j * R.W[l + 1] + (q >> 5)]);
}

// Warp-flattened edge loops: a warp takes 32 consecutive (virtual) dst rows, lane
// i loads row i's extent, a warp scan of the degrees gives each row's edge
// offset, and the warp then walks the rows' edges as one flat range, UNR edges
// per lane in flight (independent load chains), every lane busy whatever the
// degree mix.  Row data live in a per-warp shared slice.
#ifndef BETTY_FLAT_UNR             // (overridable at build time for tuning sweeps)
#define BETTY_FLAT_UNR 4
#endif
#ifndef BETTY_RL_UNR
#define BETTY_RL_UNR 4
#endif
constexpr int FLAT_UNR = BETTY_FLAT_UNR;
constexpr int RL_UNR = BETTY_RL_UNR;   // relabel chains per lane (8: 128 registers, measured slower)
struct FlatRows {
    int pre[33];        // exclusive edge offsets of the warp's rows (pre[32] = total)
    int64_t fb[32];     // full-batch row start of each row
    int64_t ob[32];     // output offset (relabel) of each row
    int j[32];          // slot (micro-batch) of each row
};
__device__ __forceinline__ int flat_row(const FlatRows& F, int f) {
    int lo = 0, hi = 32;                                 // F.pre[lo] <= f < F.pre[hi]
#pragma unroll
    for (int step = 0; step < 5; ++step) {
        const int mid = (lo + hi) >> 1;
        if (F.pre[mid] <= f) lo = mid; else hi = mid;
    }
    return lo;
}

__global__ void __launch_bounds__(256) k_mark_new(const int32_t* __restrict__ dst_pos, const int32_t* __restrict__ row_mb,
                                                  const int64_t* cnt, const int64_t* __restrict__ findptr,
                                                  const int32_t* __restrict__ fnbr, const uint32_t* __restrict__ dstbits,
                                                  uint32_t* newbits, int64_t W, const int64_t* __restrict__ otab,
                                                  unsigned* ctr, int claim) {
    __shared__ int64_t s_vs[ORDER_SMEM + 1], s_rs[ORDER_SMEM];
    __shared__ FlatRows s_rows[8];
    const int nseg = order_load(otab, s_vs, s_rs);
    int seg = 0;
    const int64_t n = cnt[0];
    const int lane = lane_id();
    FlatRows& F = s_rows[warp_id()];
    // dynamic schedule (claims of `claim` <= 32 rows, lane = row): the rows in flight stay a narrow
    // window of the micro-batch-major order, so one micro-batch's bitmaps / map stay in L2; small
    // layers use shorter claims so that more warps share the (latency-bound) edge walk
    __shared__ int64_t s_claim[8];
    for (;;) {
        if (lane == 0) s_claim[warp_id()] = (int64_t)atomicAdd(ctr, 1u) * claim;
        __syncwarp();
        const int64_t v0 = s_claim[warp_id()];
        __syncwarp();
        if (v0 >= n) break;
        const int64_t vv = v0 + lane;
        int d = 0;
        if (lane < claim && vv < n) {
            const int64_t r = order_map(vv, nseg, s_vs, s_rs, seg);
            const int32_t q = dst_pos[r];
            const int64_t b = findptr[q];
            d = (int)(findptr[q + 1] - b);
            F.fb[lane] = b;
            F.j[lane] = row_mb[r];
        }
        const int incl = warp_incl_scan(d);
        F.pre[lane + 1] = incl;
        if (lane == 0) F.pre[0] = 0;
        __syncwarp();
        const int total = F.pre[32];
        for (int f0 = lane; f0 < total; f0 += 32 * FLAT_UNR) {
            int32_t p[FLAT_UNR];
            int jj[FLAT_UNR];
#pragma unroll
            for (int u = 0; u < FLAT_UNR; ++u) {
                const int f = f0 + 32 * u;
                p[u] = -1;
                if (f < total) {
                    const int k = flat_row(F, f);
                    p[u] = fnbr[F.fb[k] + (f - F.pre[k])];
                    jj[u] = F.j[k];
                }
            }
            // (measured: reading the new word too, to skip already-marked sources, is slower -- the
            // random L2 reads cost more than the fire-and-forget atomics they save)
            uint32_t dw[FLAT_UNR];
#pragma unroll
            for (int u = 0; u < FLAT_UNR; ++u)
                dw[u] = (p[u] >= 0 && dstbits) ? dstbits[(int64_t)jj[u] * W + (p[u] >> 5)] : 0u;
#pragma unroll
            for (int u = 0; u < FLAT_UNR; ++u) {
                if (p[u] >= 0) {
                    const uint32_t bit = 1u << (p[u] & 31);
                    if (!(dw[u] & bit)) atomicOr(&newbits[(int64_t)jj[u] * W + (p[u] >> 5)], bit);
                }
            }
        }
        __syncwarp();
    }
}

__global__ void __launch_bounds__(256) k_relabel(const int32_t* __restrict__ dst_pos, const int32_t* __restrict__ row_mb,
                                                 const int64_t* cnt, const int64_t* __restrict__ findptr,
                                                 const int32_t* __restrict__ fnbr, const int64_t* __restrict__ indptr,
                                                 const RankSet R, int l, int32_t* __restrict__ indices,
                                                 int64_t cap_e, const int32_t* __restrict__ fsrc_gid,
                                                 int32_t* __restrict__ egid, const int64_t* __restrict__ otab,
                                                 unsigned* ctr, int claim, int32_t* __restrict__ tcnt, int64_t cap_src) {
    __shared__ int64_t s_vs[ORDER_SMEM + 1], s_rs[ORDER_SMEM];
    __shared__ FlatRows s_rows[8];
    const int nseg = order_load(otab, s_vs, s_rs);
    int seg = 0;
    const int64_t n = cnt[0];
    const int lane = lane_id();
    FlatRows& F = s_rows[warp_id()];
    // dynamic schedule (claims of `claim` <= 32 rows, lane = row): the rows in flight stay a narrow
    // window of the micro-batch-major order, so one micro-batch's bitmaps / map stay in L2; small
    // layers use shorter claims so that more warps share the (latency-bound) edge walk
    __shared__ int64_t s_claim[8];
    for (;;) {
        if (lane == 0) s_claim[warp_id()] = (int64_t)atomicAdd(ctr, 1u) * claim;
        __syncwarp();
        const int64_t v0 = s_claim[warp_id()];
        __syncwarp();
        if (v0 >= n) break;
        const int64_t vv = v0 + lane;
        int d = 0;
        if (lane < claim && vv < n) {
            const int64_t r = order_map(vv, nseg, s_vs, s_rs, seg);
            const int32_t q = dst_pos[r];
            const int64_t b = findptr[q];
            d = (int)(findptr[q + 1] - b);
            const int j = row_mb[r];
            F.fb[lane] = b;
            F.j[lane] = j;
            F.ob[lane] = indptr[r];
        }
        const int incl = warp_incl_scan(d);
        F.pre[lane + 1] = incl;
        if (lane == 0) F.pre[0] = 0;
        __syncwarp();
        const int total = F.pre[32];
        for (int f0 = lane; f0 < total; f0 += 32 * RL_UNR) {
            int32_t p[RL_UNR];
            int kk[RL_UNR];
#pragma unroll
            for (int u = 0; u < RL_UNR; ++u) {
                const int f = f0 + 32 * u;
                p[u] = -1;
                if (f < total) {
                    const int k = flat_row(F, f);
                    kk[u] = k;
                    p[u] = fnbr[F.fb[k] + (f - F.pre[k])];
                }
            }
            uint2 nr[RL_UNR];
            int32_t id[RL_UNR], gid[RL_UNR];
#pragma unroll
            for (int u = 0; u < RL_UNR; ++u) {
                if (p[u] >= 0) {
                    nr[u] = R.nr[l][(int64_t)F.j[kk[u]] * R.W[l] + (p[u] >> 5)];
                    if (egid) gid[u] = fsrc_gid[p[u]];
                }
            }
            // src_id level by level for all RL_UNR edges at once: each level's rank-word loads are
            // issued together (independent chains), not one edge's whole chain after another
            bool done[RL_UNR];
#pragma unroll
            for (int u = 0; u < RL_UNR; ++u) {
                done[u] = p[u] < 0;
                if (!done[u] && (nr[u].x >> (p[u] & 31) & 1u)) {
                    id[u] = (int32_t)(R.cnt[l][0] + R.off[l][F.j[kk[u]]] + rank_in(nr[u], p[u]));
                    done[u] = true;
                }
            }
            for (int q = l + 1; q < R.L; ++q) {
#pragma unroll
                for (int u = 0; u < RL_UNR; ++u)
                    if (!done[u]) nr[u] = R.nr[q][(int64_t)F.j[kk[u]] * R.W[q] + (p[u] >> 5)];
#pragma unroll
                for (int u = 0; u < RL_UNR; ++u)
                    if (!done[u] && (nr[u].x >> (p[u] & 31) & 1u)) {
                        id[u] = (int32_t)(R.cnt[q][0] + R.off[q][F.j[kk[u]]] + rank_in(nr[u], p[u]));
                        done[u] = true;
                    }
            }
#pragma unroll
            for (int u = 0; u < RL_UNR; ++u)
                if (!done[u]) nr[u] = R.dr[(int64_t)F.j[kk[u]] * R.Wt + (p[u] >> 5)];
#pragma unroll
            for (int u = 0; u < RL_UNR; ++u)
                if (!done[u]) id[u] = (int32_t)(R.top_off[F.j[kk[u]]] + rank_in(nr[u], p[u]));
#pragma unroll
            for (int u = 0; u < RL_UNR; ++u) {
                if (p[u] >= 0) {
                    const int k = kk[u];
                    const int64_t o = F.ob[k] + (f0 + 32 * u - F.pre[k]);
                    if (o < cap_e) {
                        indices[o] = id[u];
                        if (egid) egid[o] = gid[u];
                        // CSC column length of the source (zeroed by the emit kernels)
                        if (tcnt && id[u] < cap_src) atomicAdd(&tcnt[id[u]], 1);
                    }
                }
            }
        }
        __syncwarp();
    }
}

// CSC of a micro-batch layer filtered from the full-batch CSC, warp-flattened: a warp takes 32
// sources, loads their full-batch columns' extents at once, then walks all their entries as one
// flat range (FLAT_UNR per lane in flight): keep an entry iff its dst is in the source's
// micro-batch.  Count pass: kept entries per source.  Fill pass: kept entries in column order
// (prefix of the keep flags within each source's run of lanes + a per-source running count).
template <bool FILL>
__global__ void __launch_bounds__(256) k_csc_flat(const int32_t* __restrict__ src_pos,
                                                  const int32_t* __restrict__ src_mb, const int64_t* cnt,
                                                  const int64_t* __restrict__ ft_indptr,
                                                  const int32_t* __restrict__ ft_nbr,
                                                  const uint32_t* __restrict__ dstbits, int64_t W, const RankSet R,
                                                  int l, const int64_t* __restrict__ t_indptr,
                                                  int32_t* __restrict__ t_idx, int32_t* __restrict__ tcnt) {
    __shared__ FlatRows s_rows[8];
    __shared__ int s_run[8][32];
    const int64_t n = cnt[1];
    const int lane = lane_id();
    FlatRows& F = s_rows[warp_id()];
    int* run = s_run[warp_id()];
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t u0 = gw * 32; u0 < n; u0 += nw * 32) {
        const int64_t u = u0 + lane;
        int d = 0;
        if (u < n) {
            const int32_t p = src_pos[u];
            const int64_t b = ft_indptr[p];
            d = (int)(ft_indptr[p + 1] - b);
            F.fb[lane] = b;
            F.j[lane] = src_mb[u];
            if (FILL) F.ob[lane] = t_indptr[u];
        }
        run[lane] = 0;
        const int incl = warp_incl_scan(d);
        F.pre[lane + 1] = incl;
        if (lane == 0) F.pre[0] = 0;
        __syncwarp();
        const int total = F.pre[32];
        for (int fb = 0; fb < total; fb += 32 * FLAT_UNR) {      // warp-uniform: collectives inside
            const int f0 = fb + lane;
            int32_t q[FLAT_UNR];
            int kk[FLAT_UNR];
            uint32_t w[FLAT_UNR];
#pragma unroll
            for (int t = 0; t < FLAT_UNR; ++t) {
                const int f = f0 + 32 * t;
                q[t] = -1;
                kk[t] = 32;
                if (f < total) {
                    const int k = flat_row(F, f);
                    kk[t] = k;
                    q[t] = ft_nbr[F.fb[k] + (f - F.pre[k])];
                }
            }
#pragma unroll
            for (int t = 0; t < FLAT_UNR; ++t)
                w[t] = q[t] >= 0 ? dstbits[(int64_t)F.j[kk[t]] * W + (q[t] >> 5)] : 0u;
#pragma unroll
            for (int t = 0; t < FLAT_UNR; ++t) {
                const bool keep = q[t] >= 0 && ((w[t] >> (q[t] & 31)) & 1u);
                const unsigned km = __ballot_sync(0xffffffffu, keep);
                const unsigned same = __match_any_sync(0xffffffffu, kk[t]);
                const int before = __popc(km & same & ((1u << lane) - 1u));
                if (FILL) {
                    if (keep) {
                        const int k = kk[t];
                        t_idx[F.ob[k] + run[k] + before] = (int32_t)dst_id(R, l, F.j[k], q[t]);
                    }
                }
                // the highest lane of each row's run adds the row's kept entries of this step
                const int hi = 31 - __clz(same);
                __syncwarp();
                if (lane == hi && kk[t] < 32) run[kk[t]] += __popc(km & same);
                __syncwarp();
            }
        }
        if (!FILL && u < n) tcnt[u] = run[lane];
        __syncwarp();
    }
}

// single CTA: per micro-batch src counts and offsets; checks capacities
__global__ void k_counts(const int64_t* __restrict__ mb_dst_off, const int64_t* __restrict__ slot_total,
                         int32_t c, int64_t* __restrict__ mb_src_off, int64_t* cnt, int64_t cap_src, int64_t cap_e,
                         int64_t* next_cnt, int* dev_err) {
    __shared__ int64_t s_warp[33];
    __shared__ int64_t s_base;
    if (threadIdx.x == 0) s_base = 0;
    __syncthreads();
    for (int j0 = 0; j0 < c; j0 += blockDim.x) {
        const int j = j0 + threadIdx.x;
        int64_t nn = 0;                                 // new sources of micro-batch j
        if (j < c) nn = slot_total[j];
        int64_t tot;
        const int64_t ex = block_excl_scan(nn, s_warp, &tot);
        if (j < c) mb_src_off[j] = s_base + ex;         // offset of j's new sources after the dst prefix
        __syncthreads();
        if (threadIdx.x == 0) s_base += tot;
        __syncthreads();
    }
    if (threadIdx.x == 0) {
        (void)mb_dst_off;
        mb_src_off[c] = s_base;
        const int64_t ns = cnt[0] + s_base;
        if (ns > cap_src || cnt[2] > cap_e) {
            // beyond the plan's capacities (a FRESH plan's batch grew): report EOVERFLOW at the next
            // synchronising call and empty this layer and the ones below, so no later kernel writes
            // past an arena buffer
            atomicOr(dev_err, DEVERR_OVERFLOW);
            cnt[0] = 0; cnt[1] = 0; cnt[2] = 0;
            if (next_cnt) next_cnt[0] = 0;
        } else {
            cnt[1] = ns;
            if (next_cnt) next_cnt[0] = ns;
        }
    }
}

// The emit kernels write a layer's src list (dst prefix, then the new sources ascending) and, on
// the way, zero the CSC column counts (tcnt) and record each source's full-batch degree in the
// layer below (ndeg: the next layer's dst degrees, so its indptr is a plain scan, not a gather).
__global__ void k_emit_new(const uint2* __restrict__ nrank, int64_t W, int32_t c, const int64_t* n_dst_tot,
                           const int64_t* __restrict__ mb_dst_off,
                           const int64_t* __restrict__ mb_src_off, const int32_t* __restrict__ fsrc_gid,
                           int32_t* __restrict__ src_pos, int32_t* __restrict__ src_gid, int32_t* __restrict__ src_mb,
                           int64_t cap_src, int32_t* __restrict__ tcnt, const int64_t* __restrict__ nfindptr,
                           int32_t* __restrict__ ndeg) {
    const int64_t n = (int64_t)c * W;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const uint2 r = nrank[i];
        uint32_t bits = r.x;
        if (!bits) continue;
        const int j = (int)(i / W);
        const int64_t w = i - (int64_t)j * W;
        int64_t s = n_dst_tot[0] + mb_src_off[j] + r.y;
        (void)mb_dst_off;
        while (bits) {
            const int b = __ffs(bits) - 1;
            bits &= bits - 1;
            const int32_t p = (int32_t)(w * 32 + b);
            if (s < cap_src) {
                src_pos[s] = p; src_gid[s] = fsrc_gid[p]; src_mb[s] = j;
                if (tcnt) tcnt[s] = 0;
                if (ndeg) ndeg[s] = (int32_t)(nfindptr[p + 1] - nfindptr[p]);
            }
            ++s;
        }
    }
}

__global__ void k_emit_dst(const int32_t* __restrict__ dst_pos, const int32_t* __restrict__ row_mb,
                           const int64_t* cnt, const int64_t* __restrict__ mb_dst_off,
                           const int64_t* __restrict__ mb_src_off, const int32_t* __restrict__ fsrc_gid,
                           int32_t* __restrict__ src_pos, int32_t* __restrict__ src_gid, int32_t* __restrict__ src_mb,
                           int64_t cap_src, int32_t* __restrict__ tcnt, const int64_t* __restrict__ nfindptr,
                           int32_t* __restrict__ ndeg) {
    const int64_t n = cnt[0];
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
        const int j = row_mb[r];
        const int64_t s = r;                            // dst prefix keeps the row order
        (void)mb_dst_off; (void)mb_src_off;
        const int32_t p = dst_pos[r];
        if (s < cap_src) {
            src_pos[s] = p; src_gid[s] = fsrc_gid[p]; src_mb[s] = j;
            if (tcnt) tcnt[s] = 0;
            if (ndeg) ndeg[s] = (int32_t)(nfindptr[p + 1] - nfindptr[p]);
        }
    }
}

// single CTA: the micro-batch-major order table of layer l (extract.h); segment (j, p), j-major
struct LayerPtrs { const int64_t* cnt[16]; const int64_t* off[16]; };
__global__ void k_order_tab(int32_t c, int L, int l, const int64_t* __restrict__ top_off, LayerPtrs lp_,
                            int64_t* tab) {
    __shared__ int64_t s_warp[33];
    const int P = L - l, nseg = c * P;
    if (nseg > ORDER_TAB_MAX) {                         // too many segments: identity order
        if (threadIdx.x == 0) tab[2 * (ORDER_TAB_MAX + 1)] = 0;
        return;
    }
    int64_t* vs = tab;
    int64_t* rs = tab + ORDER_TAB_MAX + 1;
    __shared__ int64_t s_base;
    if (threadIdx.x == 0) s_base = 0;
    __syncthreads();
    for (int i0 = 0; i0 < nseg; i0 += blockDim.x) {
        const int i = i0 + threadIdx.x;
        int64_t len = 0, start = 0;
        if (i < nseg) {
            const int j = i / P, p = i % P;
            if (p == 0) { start = top_off[j]; len = top_off[j + 1] - top_off[j]; }
            else {
                const int lp = L - p;                   // new sources of layer lp
                const int64_t* o = lp_.off[lp];
                start = lp_.cnt[lp][0] + o[j];
                len = o[j + 1] - o[j];
            }
        }
        int64_t tot;
        const int64_t ex = block_excl_scan(len, s_warp, &tot);
        if (i < nseg) { vs[i] = s_base + ex; rs[i] = start; }
        __syncthreads();
        if (threadIdx.x == 0) s_base += tot;
        __syncthreads();
    }
    if (threadIdx.x == 0) { vs[nseg] = s_base; tab[2 * (ORDER_TAB_MAX + 1)] = nseg; }
}

// lean layer 0: each dst row's full-batch edge segment of source gids -> the group's egid (rows in
// their group order; warp-flattened like the relabel, coalesced within a row); n_src := n_dst
// (fnbr, fsrc_gid non-null: the gid of edge f is fsrc_gid[fnbr[f]], read directly -- a FRESH step)
__global__ void __launch_bounds__(256) k_seg_egid(const int32_t* __restrict__ dst_pos, int64_t* cnt,
                                                  const int64_t* __restrict__ findptr,
                                                  const int32_t* __restrict__ fegid,
                                                  const int32_t* __restrict__ fnbr,
                                                  const int32_t* __restrict__ fsrc_gid,
                                                  const int64_t* __restrict__ indptr, int32_t* __restrict__ egid,
                                                  int64_t cap_e, int* dev_err) {
    __shared__ FlatRows s_rows[8];
    const int64_t n = cnt[0];
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        if (cnt[2] > cap_e) {                           // EOVERFLOW; the layer runs empty (see k_counts)
            atomicOr(dev_err, DEVERR_OVERFLOW);
            cnt[0] = 0; cnt[1] = 0; cnt[2] = 0;
        } else {
            cnt[1] = n;
        }
    }
    const int lane = lane_id();
    FlatRows& F = s_rows[warp_id()];
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t v0 = gw * 32; v0 < n; v0 += nw * 32) {
        const int64_t r = v0 + lane;
        int d = 0;
        if (r < n) {
            const int32_t q = dst_pos[r];
            const int64_t b = findptr[q];
            d = (int)(findptr[q + 1] - b);
            F.fb[lane] = b;
            F.ob[lane] = indptr[r];
        }
        const int incl = warp_incl_scan(d);
        F.pre[lane + 1] = incl;
        if (lane == 0) F.pre[0] = 0;
        __syncwarp();
        const int total = F.pre[32];
        for (int f0 = lane; f0 < total; f0 += 32 * FLAT_UNR) {
            int32_t g[FLAT_UNR];
            int64_t o[FLAT_UNR];
#pragma unroll
            for (int u = 0; u < FLAT_UNR; ++u) {
                const int f = f0 + 32 * u;
                o[u] = -1;
                if (f < total) {
                    const int k = flat_row(F, f);
                    g[u] = fnbr ? fnbr[F.fb[k] + (f - F.pre[k])] : fegid[F.fb[k] + (f - F.pre[k])];
                    o[u] = F.ob[k] + (f - F.pre[k]);
                }
            }
            if (fnbr) {
#pragma unroll
                for (int u = 0; u < FLAT_UNR; ++u) if (o[u] >= 0) g[u] = fsrc_gid[g[u]];
            }
#pragma unroll
            for (int u = 0; u < FLAT_UNR; ++u) if (o[u] >= 0 && o[u] < cap_e) egid[o[u]] = g[u];
        }
        __syncwarp();
    }
}

// full-batch edge -> source gid of a layer (once per plan; every step with BETTY_PLAN_FRESH)
__global__ void k_full_egid(const int32_t* __restrict__ nbr, const int32_t* __restrict__ src_gid, int64_t E,
                            int32_t* __restrict__ egid) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < E; e += (int64_t)gridDim.x * blockDim.x)
        egid[e] = src_gid[nbr[e]];
}
void full_egid(betty_ctx* c, const int32_t* nbr, const int32_t* src_gid, int64_t E, int32_t* egid, cudaStream_t s) {
    const int g = (int)std::max<int64_t>(1, std::min<int64_t>((E + 255) / 256, (int64_t)c->num_sms * 8));
    k_full_egid<<<g, 256, 0, s>>>(nbr, src_gid, E, egid);
}

__global__ void k_clear_bits(uint32_t* a, uint32_t* b, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        a[i] = 0u;
        b[i] = 0u;
    }
}

static inline int grid_for(betty_ctx* c, int64_t work, int threads, int per_sm = 8) {
    return (int)std::max<int64_t>(1, std::min<int64_t>((work + threads - 1) / threads, (int64_t)c->num_sms * per_sm));
}

bool extract_limits_ok(int32_t K, int32_t c, int64_t n_out, int64_t top_edges) {
    return K >= 1 && K <= SEL_KMAX && c >= 1 && c <= SEL_CMAX && n_out < (1ll << (63 - SEL_SHIFT)) - 1 &&
           top_edges < (1ll << SEL_SHIFT);
}

size_t extract_scratch_bytes(int64_t c, int64_t max_full_src, int64_t sel_nchunks) {
    const int64_t W = (max_full_src + 31) / 32 + 1;
    return (size_t)(c * W * 4 * 2 + c * max_full_src * 4 + (c * W + 1) * 8 + c * W * 4 +
                    (c * sel_nchunks + 1) * 8 + c * sel_nchunks * 8 + 4096);
}

void extract_group(betty_ctx* ctx, const ExtractArgs& a, cudaStream_t s) {
    const int32_t c = a.c;
    const int64_t n_out = a.full[a.L - 1].n_dst;
    const int64_t nchunks = (n_out + SEL_CHUNK - 1) / SEL_CHUNK;
    ExtractLayer* top = &a.layers[a.L - 1];

    // ---- V_k: outputs with part == ks[j], ascending, for every slot j (+ the top layer's indptr,
    // counts and dst bitmap; the bitmap only when the top layer is not extracted lean)
    const bool top_lean = a.L == 1 && a.lean0 && a.full[0].egid && top->egid;
    {
        const unsigned g = (unsigned)std::max<int64_t>(1, nchunks);
        k_sel_count<<<g, 256, 0, s>>>(a.part, n_out, a.K, a.ks, c, a.full[a.L - 1].indptr, a.sc.sel_cnt, nchunks,
                                      ctx->dev_err);
        scan_i64(ctx, a.sc.sel_cnt, a.sc.sel_off, nullptr, (int64_t)c * nchunks, 0, nullptr, s);
        k_sel_write<<<g, 32, 0, s>>>(a.part, n_out, a.K, a.ks, c, a.full[a.L - 1].indptr, a.sc.sel_off, nchunks,
                                     a.sc.top_dst_pos, a.sc.top_row_mb, top->indptr, top->cap_dst,
                                     top_lean ? nullptr : a.sc.dstbits, (a.full[a.L - 1].n_src + 31) / 32,
                                     a.sc.top_dst_off, top->cnt, ctx->dev_err);
    }

    const int32_t* dst_pos = a.sc.top_dst_pos;
    const int32_t* row_mb = a.sc.top_row_mb;
    const int64_t* dst_off = a.sc.top_dst_off;
    for (int l = a.L - 1; l >= 0; --l) {
        const ExtractFull& F = a.full[l];
        ExtractLayer& B = a.layers[l];
        const int64_t W = (F.n_src + 31) / 32;
        const int64_t cW = (int64_t)c * W;
        const int64_t cap_d = B.cap_dst, cap_e = B.cap_e, cap_s = B.cap_src;
        // micro-batch-major visiting order of this layer's dst rows (needs only the layers above)
        const int64_t* otab = nullptr;
        if (l + 1 < a.L && B.order_tab) {
            LayerPtrs lp{};
            for (int q = 0; q < a.L; ++q) { lp.cnt[q] = a.layers[q].cnt; lp.off[q] = a.layers[q].mb_src_off; }
            k_order_tab<<<1, 1024, 0, s>>>(c, a.L, l, a.sc.top_dst_off, lp, B.order_tab);
            otab = B.order_tab;
        }
        // rows: degree of each dst row in the full batch -> local indptr
        const bool top = l == a.L - 1;                  // its indptr / counts / dst bits come from the selection
        if (!top) scan_i32(ctx, a.sc.ndeg, B.indptr, B.cnt + 0, 0, cap_d, B.cnt + 2, s);   // degrees: emit kernels above
        if (l == 0 && a.lean0 && F.egid && B.egid) {
            // lean layer 0: the dst prefix (self rows) and the edges' source gids, nothing else
            k_emit_dst<<<grid_for(ctx, cap_d, 256), 256, 0, s>>>(dst_pos, row_mb, B.cnt, dst_off, B.mb_src_off,
                                                                 F.src_gid, B.src_pos, B.src_gid, B.src_mb, cap_s,
                                                                 nullptr, nullptr, nullptr);
            k_seg_egid<<<grid_for(ctx, (cap_d + 31) / 32 * 32, 256), 256, 0, s>>>(
                dst_pos, B.cnt, F.indptr, F.egid, a.egid_direct ? F.nbr : nullptr, a.egid_direct ? F.src_gid : nullptr,
                B.indptr, B.egid, cap_e, ctx->dev_err);
            break;
        }
        // dedupe: dst bitmap + position map, then new-source bitmap
        if (!top) k_mark_dst<<<grid_for(ctx, cap_d, 256), 256, 0, s>>>(dst_pos, row_mb, B.cnt, a.sc.dstbits, W);
        // rows per claim: 32 while the layer fills every resident warp (148 SMs x 64) with 32-row
        // claims, else fewer (down to 8) so that the edge walk spreads over more warps
        const int64_t warps_res = (int64_t)ctx->num_sms * 64;
        int claim = 32;
        static const bool fixed_claim = getenv("BETTY_CLAIM32") != nullptr;      // A/B switch
        while (!fixed_claim && claim > 8 && cap_d < warps_res * claim / 2) claim >>= 1;
        const int g_rows = grid_for(ctx, (cap_d * 32 + claim - 1) / claim, 256);
        unsigned* ctr = ctx->L().counters + CTR_EXTRACT;
        cudaMemsetAsync(ctr, 0, sizeof(unsigned), s);
        // mark_nocheck: mark every neighbour (no dst lookup per edge); the dst rows are masked out of
        // the bitmap words by the rank pass instead
        static const bool mark_nocheck = getenv("BETTY_MARK_NOCHECK") && atoi(getenv("BETTY_MARK_NOCHECK"));
        k_mark_new<<<g_rows, 256, 0, s>>>(dst_pos, row_mb, B.cnt, F.indptr, F.nbr, mark_nocheck ? nullptr : a.sc.dstbits,
                                          a.sc.newbits, W, otab, ctr, claim);
        // ascending order of new sources = popcount scan over the bitmap words
        int64_t* csum = a.sc.wordoff;                   // chunk sums, then slot totals at the end
        int64_t* slot_tot = a.sc.wordoff + (int64_t)c * ((W + RANK_CHUNK - 1) / RANK_CHUNK + 1);
        slot_rank(a.sc.newbits, mark_nocheck ? a.sc.dstbits : nullptr, c, W, csum, a.sc.nrank[l], slot_tot, s);
        // CSC column lengths of this layer: counted by the relabel pass (a histogram of the local
        // source ids it writes) unless BETTY_CSC_COUNT=flat (a separate pass over the full-batch CSC)
        const bool want_csc = B.t_indptr && (a.csc_mask >> l & 1);
        static const bool flat_count = getenv("BETTY_CSC_COUNT") && !strcmp(getenv("BETTY_CSC_COUNT"), "flat");
        int32_t* hist = (want_csc && F.t_indptr && !flat_count) ? a.sc.tcnt : nullptr;
        const int64_t* nfi = l > 0 ? a.full[l - 1].indptr : nullptr;     // the layer below's dst degrees
        int32_t* ndeg = l > 0 ? a.sc.ndeg : nullptr;
        k_counts<<<1, 1024, 0, s>>>(dst_off, slot_tot, c, B.mb_src_off, B.cnt, cap_s, cap_e,
                                    l > 0 ? a.layers[l - 1].cnt : nullptr, ctx->dev_err);
        k_emit_dst<<<grid_for(ctx, cap_d, 256), 256, 0, s>>>(dst_pos, row_mb, B.cnt, dst_off, B.mb_src_off,
                                                             F.src_gid, B.src_pos, B.src_gid, B.src_mb, cap_s, hist,
                                                             nfi, ndeg);
        k_emit_new<<<grid_for(ctx, cW, 256), 256, 0, s>>>(a.sc.nrank[l], W, c, B.cnt, dst_off, B.mb_src_off,
                                                          F.src_gid, B.src_pos, B.src_gid, B.src_mb, cap_s, hist,
                                                          nfi, ndeg);
        // rank structures of this layer (and of the outputs at the top layer)
        if (l == a.L - 1) slot_rank(a.sc.dstbits, nullptr, c, W, csum, a.sc.drank_top, nullptr, s);
        RankSet R{};
        R.L = a.L;
        for (int q = 0; q < a.L; ++q) {
            R.nr[q] = a.sc.nrank[q];
            R.W[q] = (a.full[q].n_src + 31) / 32;
            R.cnt[q] = a.layers[q].cnt;
            R.off[q] = a.layers[q].mb_src_off;
        }
        R.dr = a.sc.drank_top;
        R.Wt = (a.full[a.L - 1].n_src + 31) / 32;
        R.top_off = a.sc.top_dst_off;
        cudaMemsetAsync(ctr + 1, 0, sizeof(unsigned), s);
        k_relabel<<<g_rows, 256, 0, s>>>(dst_pos, row_mb, B.cnt, F.indptr, F.nbr, B.indptr, R, l, B.indices, cap_e,
                                         F.src_gid, B.egid, otab, ctr + 1, claim, hist, cap_s);
        if (want_csc && F.t_indptr) {           // from the full-batch CSC (needs the dst bitmap + map)
            const int g_src = grid_for(ctx, (cap_s + 31) / 32 * 32, 256);
            if (!hist)
                k_csc_flat<false><<<g_src, 256, 0, s>>>(B.src_pos, B.src_mb, B.cnt, F.t_indptr, F.t_nbr, a.sc.dstbits,
                                                        W, R, l, nullptr, nullptr, a.sc.tcnt);
            scan_i32(ctx, a.sc.tcnt, B.t_indptr, B.cnt + 1, 0, cap_s, nullptr, s);
            k_csc_flat<true><<<g_src, 256, 0, s>>>(B.src_pos, B.src_mb, B.cnt, F.t_indptr, F.t_nbr, a.sc.dstbits, W,
                                                   R, l, B.t_indptr, B.t_indices, nullptr);
            if (l + 1 < a.L)                    // below the top layer dst ids are not monotone in position
                segsort_i32(ctx, B.t_indptr, B.t_indices, B.cnt + 1, 0, cap_s, s);
        }
        k_clear_bits<<<grid_for(ctx, cW, 256), 256, 0, s>>>(a.sc.dstbits, a.sc.newbits, cW);
        if (want_csc && !F.t_indptr)
            csr_transpose(ctx, B.indptr, B.indices, B.cnt + 0, B.cnt + 1, B.cnt + 2, cap_d, cap_s, cap_e,
                          B.t_indptr, B.t_indices, a.sc.tcnt, false, s);
        dst_pos = B.src_pos;
        row_mb = B.src_mb;
        dst_off = B.mb_src_off;
    }
}

}  // namespace betty
