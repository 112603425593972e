// reg.cu -- a1: the redundancy-embedded graph (REG) as an integer SpGEMM.
//
// PAPER.md:771-945 (§4.3.2, Eq. 2-4, Alg. 1 lines 1-7): A is the binary
// adjacency of the output block (a_ui = 1 iff sampled edge u -> i), C = A^T A,
// c_ij = sum_u a_ui a_uj = number of input neighbours shared by outputs i and
// j; only output nodes are kept and self loops removed.  With B = A^T
// restricted to (outputs x sources), C = B B^T.
//
// GPU design (row-wise expansion, sort-based accumulation, bit-exact):
//   1. CSC of B (counting sort + per-column sort; rejects repeated edges)
//   2. ub_i = sum_{u in S_i} (d_u - 1): exact number of candidate products of row i
//   3. exclusive scan of ub -> a temporary slot per product
//   4. per row: expand the candidates j (from the columns of its sources,
//      skipping j = i), sort them (warp bitonic for ub <= 256, CTA bitonic
//      in shared memory up to 32768), run-length encode -> (j, c_ij) ascending;
//      hub rows (ub > 32768, no degree bound in Eq. 2-4) take a CTA each: the
//      candidates (expanded in place in the row's global slot) set bits of a
//      bitmap over the output ids, a popcount prefix over its words ranks
//      every distinct j (ascending by construction), and c_ij is counted by
//      integer atomics into its rank's slot -- no sort, exact
//   5. scan of the per-row counts -> indptr, compaction into col / w
// Every step is integer and order-independent, so the result is bit-exact.
#include <climits>
#include "common.cuh"
#include "internal.h"
#include "reg.h"

namespace betty {

constexpr int REG_WARP_MAX = 256;
constexpr int REG_CTA_MAX = 32768;

__global__ void k_reset_big(int* p) { *p = 0; }

__global__ void k_reg_ub(const int64_t* __restrict__ indptr, const int32_t* __restrict__ idx,
                         const int64_t* __restrict__ t_indptr, const int64_t* n_rows_dev, int64_t* __restrict__ ub,
                         int64_t* big, int* big_cnt, int64_t big_cap, int* dev_err) {
    const int64_t n = *n_rows_dev;
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = gw; i < n; i += nw) {
        int64_t s = 0;
        for (int64_t e = indptr[i] + lane; e < indptr[i + 1]; e += 32) {
            const int32_t u = idx[e];
            s += t_indptr[u + 1] - t_indptr[u] - 1;
        }
        s = warp_sum(s);
        if (lane == 0) {
            ub[i] = s;
            if (s > REG_WARP_MAX) {                     // CTA rows (hub rows included)
                const int k = atomicAdd(big_cnt, 1);
                if (k < big_cap) big[k] = i; else atomicOr(dev_err, DEVERR_OVERFLOW);
            }
        }
    }
}

// expand the candidate list of row i into buf[0, ub) (ub known), cooperative over `nthr` threads.
// The row's edges are taken 32 at a time: one warp loads their columns' extents and
// prefix-sums the lengths into shared memory (s_pre[0..n], s_cb[0..n)), then every
// thread handles flattened candidate positions independently (no serial chain of
// dependent loads per edge).  Column u lists i exactly once (no repeated edges) and
// is ascending, so a candidate j at offset t of its column lands at t - [j > i].
__device__ __forceinline__ void reg_expand(const int64_t* __restrict__ indptr, const int32_t* __restrict__ idx,
                                           const int64_t* __restrict__ t_indptr, const int32_t* __restrict__ t_idx,
                                           int64_t i, int64_t row0, int32_t* buf, int tid, int nthr, int* s_pre,
                                           int64_t* s_cb) {
    const int64_t rb = indptr[i], re = indptr[i + 1];
    const int32_t gi = (int32_t)(row0 + i);             // the row's global id: its own column entry
    const int lane = tid & 31;
    int64_t o = 0;
    for (int64_t e0 = rb; e0 < re; e0 += 32) {
        const int n = (int)mn64(32, re - e0);
        if (tid < 32) {
            int d = 0;
            int64_t cb = 0;
            if (lane < n) {
                const int32_t u = idx[e0 + lane];
                cb = t_indptr[u];
                d = (int)(t_indptr[u + 1] - cb);
            }
            const int incl = warp_incl_scan(d);
            if (lane == 0) s_pre[0] = 0;
            s_pre[lane + 1] = incl;
            s_cb[lane] = cb;
        }
        if (nthr > 32) __syncthreads(); else __syncwarp();
        const int total = s_pre[n];
        for (int f = tid; f < total; f += nthr) {
            int lo = 0, hi = n;                          // s_pre[lo] <= f < s_pre[hi]
            while (hi - lo > 1) {
                const int mid = (lo + hi) >> 1;
                if (s_pre[mid] <= f) lo = mid; else hi = mid;
            }
            const int t = f - s_pre[lo];
            const int32_t j = t_idx[s_cb[lo] + t];
            if (j != gi) buf[o + (s_pre[lo] - lo) + t - (j > gi ? 1 : 0)] = j;
        }
        o += total - n;
        if (nthr > 32) __syncthreads(); else __syncwarp();
    }
}

// The same expansion by one warp for a row with ub <= REG_WARP_MAX (so a 32-edge chunk spans at
// most REG_WARP_MAX + 32 candidates): each lane stamps its edge's index over the edge's flat range
// in s_seg (a short per-lane loop of shared stores), so a candidate finds its edge with one shared
// load instead of a binary search over the chunk's prefix (ncu r02r: the search was the kernel's
// hottest code).
constexpr int REG_SEG_MAX = REG_WARP_MAX + 32;
__device__ __forceinline__ void reg_expand_warp(const int32_t* __restrict__ idx, const int64_t* __restrict__ t_indptr,
                                                const int32_t* __restrict__ t_idx, int64_t i, int64_t row0,
                                                int64_t rb, int64_t re, int64_t cb0, int d0, int32_t* buf,
                                                int* s_pre, int64_t* s_cb, uint8_t* s_seg) {
    const int32_t gi = (int32_t)(row0 + i);
    const int lane = lane_id();
    int64_t o = 0;
    for (int64_t e0 = rb; e0 < re; e0 += 32) {
        const int n = (int)mn64(32, re - e0);
        int d = d0;                                     // the first chunk's columns come prefetched
        int64_t cb = cb0;
        if (e0 != rb) {
            d = 0;
            cb = 0;
            if (lane < n) {
                const int32_t u = idx[e0 + lane];
                cb = t_indptr[u];
                d = (int)(t_indptr[u + 1] - cb);
            }
        }
        const int incl = warp_incl_scan(d);
        const int total = __shfl_sync(0xffffffffu, incl, 31);
        const int start = incl - d;
        s_pre[lane] = start;
        s_cb[lane] = cb;
        for (int k = 0; k < d; ++k) s_seg[start + k] = (uint8_t)lane;
        __syncwarp();
        for (int f = lane; f < total; f += 32) {
            const int k = s_seg[f];
            const int t = f - s_pre[k];
            const int32_t j = t_idx[s_cb[k] + t];
            if (j != gi) buf[o + (s_pre[k] - k) + t - (j > gi ? 1 : 0)] = j;
        }
        o += total - n;
        __syncwarp();
    }
}

// run-length encode sorted buf[0, n) -> (col, w) at out offset; returns count (to all threads)
__device__ __forceinline__ void reg_rle_store(const int32_t* buf, int n, int32_t* __restrict__ ocol,
                                              int32_t* __restrict__ ow, int tid, int nthr, int* s_cnt) {
    // sequential over 32-element chunks per warp would be simplest; use a block-wide two-pass
    for (int base = 0; base < n; base += nthr) {
        const int t = base + tid;
        const bool head = t < n && (t == 0 || buf[t] != buf[t - 1]);
        int run = 0;
        if (head) {
            int e = t + 1;
            while (e < n && buf[e] == buf[t]) ++e;
            run = e - t;
        }
        // rank of heads before t within the whole row: count heads in [0, t)
        // (computed with an atomic counter in shared memory per chunk, ordered by ballot)
        const unsigned bal = __ballot_sync(0xffffffffu, head);
        const int wpos = __popc(bal & ((1u << lane_id()) - 1));
        __shared__ int s_wcnt[32];
        if (nthr > 32) {
            if (lane_id() == 0) s_wcnt[warp_id()] = __popc(bal);
            __syncthreads();
            int before = 0;
            for (int w = 0; w < warp_id(); ++w) before += s_wcnt[w];
            if (head) { ocol[*s_cnt + before + wpos] = buf[t]; ow[*s_cnt + before + wpos] = run; }
            __syncthreads();
            if (tid == 0) { int tot = 0; for (int w = 0; w < nthr / 32; ++w) tot += s_wcnt[w]; *s_cnt += tot; }
            __syncthreads();
        } else {
            if (head) { ocol[*s_cnt + wpos] = buf[t]; ow[*s_cnt + wpos] = run; }
            __syncwarp();
            if (tid == 0) *s_cnt += __popc(bal);
            __syncwarp();
        }
    }
}

__device__ void bitonic_sort(int32_t* s, int P, int tid, int nthr, bool warp_only) {
    for (int k = 2; k <= P; k <<= 1)
        for (int j = k >> 1; j > 0; j >>= 1) {
            for (int i = tid; i < P; i += nthr) {
                const int ixj = i ^ j;
                if (ixj > i) {
                    const int32_t a = s[i], b = s[ixj];
                    if ((a > b) == ((i & k) == 0)) { s[i] = b; s[ixj] = a; }
                }
            }
            if (warp_only) __syncwarp(); else __syncthreads();
        }
}

// ascending bitonic sort of 32*K keys held lane-major in registers (lane l holds keys
// [K*l, K*l+K)); strides >= K exchange across lanes with shuffles, smaller ones in-lane
template <int K> __device__ __forceinline__ void warp_bitonic_regs(int32_t (&x)[K]) {
    const int lane = lane_id();
#pragma unroll
    for (int size = 2; size <= 32 * K; size <<= 1) {
#pragma unroll
        for (int stride = size / 2; stride > 0; stride >>= 1) {
            if (stride >= K) {
                const int ls = stride / K;
                const bool lower = (lane & ls) == 0;
#pragma unroll
                for (int k = 0; k < K; ++k) {
                    const bool up = ((lane * K + k) & size) == 0;
                    const int32_t y = __shfl_xor_sync(0xffffffffu, x[k], ls);
                    x[k] = (lower == up) ? min(x[k], y) : max(x[k], y);
                }
            } else {
#pragma unroll
                for (int k = 0; k < K; ++k) {
                    const int q = k ^ stride;
                    if (q > k) {
                        const bool up = ((lane * K + k) & size) == 0;
                        const int32_t a = x[k], b = x[q];
                        if ((a > b) == up) { x[k] = b; x[q] = a; }
                    }
                }
            }
        }
    }
}

// sort buf[0, u) (u <= 32*K) in registers and run-length encode -> (col, w) ascending;
// returns the count.  buf (>= 32*K+1 ints) is reused for the head positions.
template <int K>
__device__ __forceinline__ int warp_sort_rle(int32_t* buf, int u, int32_t* __restrict__ ocol, int32_t* __restrict__ ow) {
    const int lane = lane_id();
    int32_t x[K];
#pragma unroll
    for (int k = 0; k < K; ++k) x[k] = lane * K + k < u ? buf[lane * K + k] : INT_MAX;
    __syncwarp();
    warp_bitonic_regs<K>(x);
    const int32_t prev_lane_last = __shfl_up_sync(0xffffffffu, x[K - 1], 1);
    bool head[K];
    int nh = 0;
#pragma unroll
    for (int k = 0; k < K; ++k) {
        const int i = lane * K + k;
        const int32_t prev = k == 0 ? prev_lane_last : x[k - 1];
        head[k] = i < u && (i == 0 || x[k] != prev);
        nh += head[k];
    }
    const int incl = warp_incl_scan(nh);
    const int total = __shfl_sync(0xffffffffu, incl, 31);
    int r = incl - nh;
    // head positions -> buf (the keys live in registers now); run length = next head - this head
#pragma unroll
    for (int k = 0; k < K; ++k)
        if (head[k]) buf[r++] = lane * K + k;
    if (lane == 0) buf[total] = u;
    __syncwarp();
    r = incl - nh;
#pragma unroll
    for (int k = 0; k < K; ++k)
        if (head[k]) { ocol[r] = x[k]; ow[r] = buf[r + 1] - buf[r]; ++r; }
    __syncwarp();
    return total;
}

__global__ void __launch_bounds__(256) k_reg_rows_warp(const int64_t* __restrict__ indptr,
                                                       const int32_t* __restrict__ idx,
                                                       const int64_t* __restrict__ t_indptr,
                                                       const int32_t* __restrict__ t_idx, const int64_t* n_rows_dev,
                                                       int64_t row0,
                                                       const int64_t* __restrict__ ub, const int64_t* __restrict__ off,
                                                       int32_t* __restrict__ tcol, int32_t* __restrict__ tw,
                                                       int64_t* __restrict__ nnz) {
    __shared__ int32_t buf[8][REG_WARP_MAX + 1];
    __shared__ int s_pre[8][33];
    __shared__ int64_t s_cb[8][32];
    __shared__ uint8_t s_seg[8][REG_SEG_MAX];
    const int64_t n = *n_rows_dev;
    const int w = warp_id(), lane = lane_id();
    const int64_t gw = blockIdx.x * 8ll + w, nw = gridDim.x * 8ll;
    // Software pipeline over the warp's rows: a row's data is a chain of four dependent loads
    // (indptr -> idx -> t_indptr -> t_idx).  The next row's first three levels are issued while this
    // row is expanded and sorted (level 1 at the top, level 2 after the expansion, level 3 after the
    // sort), so only its t_idx gathers remain on the critical path (ncu r02y: the warps waited on the
    // chain, with the grid at 4x the resident warps).
    int64_t pu = 0, prb = 0, pre = 0, poff = 0, pcb = 0;
    int32_t pidx = 0;
    int pd = 0;
    auto lvl1 = [&](int64_t r) {
        pu = 0; prb = 0; pre = 0; poff = 0;
        if (r < n) { pu = ub[r]; prb = indptr[r]; pre = indptr[r + 1]; poff = off[r]; }
    };
    auto lvl2 = [&]() { pidx = (pu > 0 && pu <= REG_WARP_MAX && lane < pre - prb) ? idx[prb + lane] : -1; };
    auto lvl3 = [&]() {
        pcb = 0; pd = 0;
        if (pidx >= 0) { pcb = t_indptr[pidx]; pd = (int)(t_indptr[pidx + 1] - pcb); }
    };
    lvl1(gw); lvl2(); lvl3();
    for (int64_t i = gw; i < n; i += nw) {
        const int64_t u = pu, rb = prb, re = pre, oi = poff, cb0 = pcb;
        const int d0 = pd;
        lvl1(i + nw);
        if (u > REG_WARP_MAX) { lvl2(); lvl3(); continue; }      // handled by the CTA kernel
        if (u == 0) { if (lane == 0) nnz[i] = 0; lvl2(); lvl3(); continue; }
        reg_expand_warp(idx, t_indptr, t_idx, i, row0, rb, re, cb0, d0, buf[w], s_pre[w], s_cb[w], s_seg[w]);
        lvl2();
        if (u <= 32) {               // sort + run-length encode in registers
            int32_t x = lane < u ? buf[w][lane] : INT_MAX;
            x = warp_bitonic32(x);
            const int32_t prev = __shfl_up_sync(0xffffffffu, x, 1);
            const bool head = lane < u && (lane == 0 || x != prev);
            const unsigned hm = __ballot_sync(0xffffffffu, head);
            const unsigned above = hm & ~((2u << lane) - 1u);
            const int nxt = above ? __ffs(above) - 1 : (int)u;
            const int pos = __popc(hm & ((1u << lane) - 1u));
            if (head) { tcol[oi + pos] = x; tw[oi + pos] = nxt - lane; }
            if (lane == 0) nnz[i] = __popc(hm);
            __syncwarp();
            lvl3();
            continue;
        }
        int cnt;
        if (u <= 64) cnt = warp_sort_rle<2>(buf[w], (int)u, tcol + oi, tw + oi);
        else if (u <= 128) cnt = warp_sort_rle<4>(buf[w], (int)u, tcol + oi, tw + oi);
        else cnt = warp_sort_rle<8>(buf[w], (int)u, tcol + oi, tw + oi);
        if (lane == 0) nnz[i] = cnt;
        lvl3();
    }
}

// exclusive scan of v over the CTA (blockDim.x a multiple of 32, <= 1024); returns the prefix,
// *total gets the sum (to every thread)
__device__ __forceinline__ int64_t cta_excl_scan(int64_t v, int64_t* total, int64_t* s_w) {
    const int lane = lane_id(), w = warp_id(), nw = blockDim.x >> 5;
    int64_t incl = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const int64_t y = __shfl_up_sync(0xffffffffu, incl, d);
        if (lane >= d) incl += y;
    }
    if (lane == 31) s_w[w] = incl;
    __syncthreads();
    if (w == 0) {
        int64_t x = lane < nw ? s_w[lane] : 0, xi = x;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const int64_t y = __shfl_up_sync(0xffffffffu, xi, d);
            if (lane >= d) xi += y;
        }
        if (lane < nw) s_w[lane] = xi - x;
        if (lane == 31) s_w[32] = xi;
    }
    __syncthreads();
    const int64_t r = s_w[w] + incl - v;
    *total = s_w[32];
    __syncthreads();
    return r;
}

// One hub row (ub > REG_CTA_MAX) by the whole CTA: the candidates are expanded into the row's
// global slot cand[0, u), marked in a bitmap over the output ids, ranked by a popcount prefix, and
// counted into w[rank] by integer atomics; finally the distinct ids overwrite cand ascending.
__device__ void reg_hub_row(const int64_t* __restrict__ indptr, const int32_t* __restrict__ idx,
                            const int64_t* __restrict__ t_indptr, const int32_t* __restrict__ t_idx, int64_t i,
                            int64_t row0, int64_t u, int32_t* cand, int32_t* wout, uint32_t* bits, int32_t* pre,
                            int64_t W, int* s_pre, int64_t* s_cb, int64_t* s_w, int64_t* nnz_out) {
    const int tid = threadIdx.x, nthr = blockDim.x;
    reg_expand(indptr, idx, t_indptr, t_idx, i, row0, cand, tid, nthr, s_pre, s_cb);
    for (int64_t q = tid; q < W; q += nthr) bits[q] = 0u;
    for (int64_t q = tid; q < u; q += nthr) wout[q] = 0;
    __syncthreads();
    for (int64_t q = tid; q < u; q += nthr) {
        const int32_t j = cand[q];
        atomicOr(&bits[j >> 5], 1u << (j & 31));
    }
    __syncthreads();
    int64_t run = 0;
    for (int64_t base = 0; base < W; base += nthr) {
        const int64_t q = base + tid;
        const int64_t v = q < W ? __popc(bits[q]) : 0;
        int64_t tot;
        const int64_t ex = cta_excl_scan(v, &tot, s_w);
        if (q < W) pre[q] = (int32_t)(run + ex);
        run += tot;
    }
    __syncthreads();
    for (int64_t q = tid; q < u; q += nthr) {
        const int32_t j = cand[q];
        const uint32_t m = bits[j >> 5] & ((1u << (j & 31)) - 1u);
        atomicAdd(&wout[pre[j >> 5] + __popc(m)], 1);
    }
    __syncthreads();
    for (int64_t q = tid; q < W; q += nthr) {
        uint32_t m = bits[q];
        int32_t r = pre[q];
        while (m) {
            const int b = __ffs(m) - 1;
            cand[r++] = (int32_t)(q * 32 + b);
            m &= m - 1u;
        }
    }
    if (tid == 0) *nnz_out = run;
    __syncthreads();
}

__global__ void __launch_bounds__(1024) k_reg_rows_cta(const int64_t* __restrict__ indptr,
                                                       const int32_t* __restrict__ idx,
                                                       const int64_t* __restrict__ t_indptr,
                                                       const int32_t* __restrict__ t_idx, int64_t row0,
                                                       const int64_t* __restrict__ ub, const int64_t* __restrict__ off,
                                                       const int64_t* big, const int* big_cnt,
                                                       int32_t* __restrict__ tcol, int32_t* __restrict__ tw,
                                                       int64_t* __restrict__ nnz, uint32_t* hub_bits, int32_t* hub_pre,
                                                       int64_t hub_words, int* dev_err) {
    extern __shared__ int32_t sbuf[];
    __shared__ int s_cnt;
    __shared__ int s_pre[33];
    __shared__ int64_t s_cb[32];
    __shared__ int64_t s_w[33];
    const int nb = *big_cnt;
    for (int t = blockIdx.x; t < nb; t += gridDim.x) {
        const int64_t i = big[t];
        const int64_t u = ub[i];
        if (u > REG_CTA_MAX) {
            if (!hub_bits) { if (threadIdx.x == 0) { nnz[i] = 0; atomicOr(dev_err, DEVERR_OVERFLOW); } continue; }
            reg_hub_row(indptr, idx, t_indptr, t_idx, i, row0, u, tcol + off[i], tw + off[i],
                        hub_bits + blockIdx.x * hub_words, hub_pre + blockIdx.x * hub_words, hub_words, s_pre, s_cb,
                        s_w, &nnz[i]);
            continue;
        }
        reg_expand(indptr, idx, t_indptr, t_idx, i, row0, sbuf, threadIdx.x, blockDim.x, s_pre, s_cb);
        int P = 1024;
        while (P < u) P <<= 1;
        for (int q = (int)u + threadIdx.x; q < P; q += blockDim.x) sbuf[q] = INT_MAX;
        __syncthreads();
        bitonic_sort(sbuf, P, threadIdx.x, blockDim.x, false);
        if (threadIdx.x == 0) s_cnt = 0;
        __syncthreads();
        reg_rle_store(sbuf, (int)u, tcol + off[i], tw + off[i], threadIdx.x, blockDim.x, &s_cnt);
        if (threadIdx.x == 0) nnz[i] = s_cnt;
        __syncthreads();
    }
}

__global__ void k_reg_compact(const int64_t* __restrict__ off, const int64_t* __restrict__ rp,
                              const int64_t* n_rows_dev, const int32_t* __restrict__ tcol,
                              const int32_t* __restrict__ tw, int32_t* __restrict__ col, int32_t* __restrict__ w,
                              int64_t nnz_cap) {
    const int64_t n = *n_rows_dev;
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = gw; i < n; i += nw) {
        const int64_t b = rp[i], len = rp[i + 1] - b, o = off[i];
        for (int64_t t = lane; t < len; t += 32)
            if (b + t < nnz_cap) { col[b + t] = tcol[o + t]; w[b + t] = tw[o + t]; }
    }
}

void init_reg_attrs() {
    cudaFuncSetAttribute(k_reg_rows_cta, cudaFuncAttributeMaxDynamicSharedMemorySize, REG_CTA_MAX * 4);
}

void reg_phase1(betty_ctx* c, const RegArgs& a, cudaStream_t s) {
    if (!a.csc_ready)
        csr_transpose(c, a.full_indptr, a.idx, a.n_full_rows_dev, a.n_cols_dev, a.n_edges_dev, a.full_rows_cap,
                      a.cols_cap, a.edges_cap, a.t_indptr, a.t_idx, a.tcnt, true, s);
    const int gw = (int)std::max<int64_t>(1, std::min<int64_t>((a.rows_cap * 32 + 255) / 256, (int64_t)c->num_sms * 16));
    k_reset_big<<<1, 1, 0, s>>>(c->L().big_count);
    k_reg_ub<<<gw, 256, 0, s>>>(a.indptr, a.idx, a.t_indptr, a.n_rows_dev, a.ub, c->L().big_list, c->L().big_count,
                                c->L().big_list_cap, c->dev_err);
    scan_i64(c, a.ub, a.off, a.n_rows_dev, 0, a.rows_cap, a.ub_total_dev, s);
}

void reg_phase2(betty_ctx* c, const RegArgs& a, cudaStream_t s) {
    const int gw = (int)std::max<int64_t>(1, std::min<int64_t>((a.rows_cap * 32 + 255) / 256, (int64_t)c->num_sms * 16));
    k_reg_rows_warp<<<gw, 256, 0, s>>>(a.indptr, a.idx, a.t_indptr, a.t_idx, a.n_rows_dev, a.row0, a.ub, a.off, a.tcol,
                                       a.tw, a.row_nnz);
    // one CTA per SM over the rows with more than REG_WARP_MAX candidates (a few hundred of 196 K on C3,
    // but most rows of a full-neighbourhood batch such as C2: a 16-CTA grid took C2 from 8.3 to 17.7 ms)
    k_reg_rows_cta<<<c->num_sms, 1024, REG_CTA_MAX * 4, s>>>(a.indptr, a.idx, a.t_indptr, a.t_idx, a.row0, a.ub, a.off,
                                                            c->L().big_list, c->L().big_count, a.tcol, a.tw, a.row_nnz,
                                                            a.hub_bits, a.hub_pre, a.hub_words, c->dev_err);
    scan_i64(c, a.row_nnz, a.out_indptr, a.n_rows_dev, 0, a.rows_cap, a.nnz_total_dev, s);
}

void reg_phase3(betty_ctx* c, const RegArgs& a, int32_t* col, int32_t* w, int64_t nnz_cap, cudaStream_t s) {
    const int gw = (int)std::max<int64_t>(1, std::min<int64_t>((a.rows_cap * 32 + 255) / 256, (int64_t)c->num_sms * 16));
    k_reg_compact<<<gw, 256, 0, s>>>(a.off, a.out_indptr, a.n_rows_dev, a.tcol, a.tw, col, w, nnz_cap);
}

}  // namespace betty
