// prims.cu -- device-wide primitives with DEVICE-resident sizes, so that a
// whole training step runs without host synchronisation (graph-capturable):
//   * single-pass exclusive scan (one chunk per CTA, aggregates exchanged through flags)
//   * segmented sort of short int32 segments (warp / CTA bitonic)
//   * CSR -> CSC transpose with ascending row ids per column
#include <climits>
#include "common.cuh"
#include "internal.h"

namespace betty {

// ------------------------------------------------------------------ scan
constexpr int SCAN_THREADS = 256;
constexpr unsigned long long ST_AGG = 1ull << 62, ST_PRE = 2ull << 62, ST_VAL = (1ull << 62) - 1;

__device__ __forceinline__ unsigned long long ld_acquire(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(unsigned long long* p, unsigned long long v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// Chunked single-pass scan: one contiguous run of 4096-element tiles per CTA (grid <= 2 x SMs; a small
// n uses fewer CTAs), claimed by ticket (so every lower chunk belongs to a CTA that is already running).
// A thread holds 16 consecutive elements of a tile in registers, loaded by independent 16-byte loads
// (one memory round trip per tile); the chunk's aggregate is published as a flag word, warp 0 sums ALL
// lower chunks' aggregates in one warp-parallel pass (no chain of inclusive prefixes), and the chunk is
// scanned with a running carry (a one-tile chunk -- n <= 1.2 M -- straight from the registers it was
// reduced from).  ncu r06: the tile-by-tile decoupled look-back took 35 us for 2.4 M int32 (prefixes
// propagated <= 32 tiles per hop) and a chunk loop with one 4-element load per thread and round trip
// 15 us for 28 K elements -- latency chains, not bytes.
constexpr int SCAN_ITEMS = 16;
constexpr int SCAN_TILE = SCAN_THREADS * SCAN_ITEMS;
template <typename Tin>
__device__ __forceinline__ void scan_ld16(const Tin* __restrict__ in, int64_t i, int64_t hi, bool vec,
                                          int64_t (&v)[SCAN_ITEMS]) {
    if (vec && i + SCAN_ITEMS <= hi) {
        if constexpr (sizeof(Tin) == 4) {
            int4 x[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) x[q] = __ldg(reinterpret_cast<const int4*>(in + i) + q);
#pragma unroll
            for (int q = 0; q < 4; ++q) { v[4 * q] = x[q].x; v[4 * q + 1] = x[q].y; v[4 * q + 2] = x[q].z; v[4 * q + 3] = x[q].w; }
        } else {
            longlong2 x[8];
#pragma unroll
            for (int q = 0; q < 8; ++q) x[q] = __ldg(reinterpret_cast<const longlong2*>(in + i) + q);
#pragma unroll
            for (int q = 0; q < 8; ++q) { v[2 * q] = x[q].x; v[2 * q + 1] = x[q].y; }
        }
    } else {
#pragma unroll
        for (int q = 0; q < SCAN_ITEMS; ++q) v[q] = i + q < hi ? (int64_t)in[i + q] : 0;
    }
}

template <typename Tin>
__global__ void __launch_bounds__(SCAN_THREADS) k_scan(const Tin* __restrict__ in, int64_t* __restrict__ out,
                                                       const int64_t* n_dev, int64_t n_fixed, int64_t* total_dev,
                                                       unsigned long long* status, unsigned* ctr) {
    __shared__ int64_t s_warp[SCAN_THREADS / 32 + 1];
    __shared__ int64_t s_prefix;
    __shared__ unsigned s_c;
    __shared__ int s_last;
    const int64_t n = n_dev ? *n_dev : n_fixed;
    const int G = (int)gridDim.x;
    const int64_t ntiles = (n + SCAN_TILE - 1) / SCAN_TILE;
    const int nch = (int)max((int64_t)1, min((int64_t)G, ntiles));     // chunks in use
    const int64_t tpc = (ntiles + nch - 1) / nch;                        // tiles per chunk
    const bool solo = G == 1;                        // one CTA: no ticket, no flags, no cleanup
    if (!solo) {
        if (threadIdx.x == 0) s_c = atomicAdd(&ctr[0], 1u);
        __syncthreads();
    }
    const int c = solo ? 0 : (int)s_c;
    if (c < nch) {
        const int64_t lo = min(n, (int64_t)c * tpc * SCAN_TILE), hi = min(n, lo + tpc * SCAN_TILE);
        const bool vec = ((uintptr_t)in & 15) == 0;                      // tiles start 64-byte aligned
        const int64_t toff = (int64_t)threadIdx.x * SCAN_ITEMS;
        // 1. the chunk's aggregate (a one-tile chunk keeps its values for step 3)
        int64_t v[SCAN_ITEMS];
        int64_t sum = 0;
        scan_ld16(in, lo + toff, hi, vec, v);
#pragma unroll
        for (int q = 0; q < SCAN_ITEMS; ++q) sum += v[q];
#pragma unroll 2
        for (int64_t base = lo + SCAN_TILE; !solo && base < hi; base += SCAN_TILE) {
            int64_t w[SCAN_ITEMS];
            scan_ld16(in, base + toff, hi, vec, w);
#pragma unroll
            for (int q = 0; q < SCAN_ITEMS; ++q) sum += w[q];
        }
        int64_t agg = 0;
        if (!solo) block_excl_scan(sum, s_warp, &agg);
        else if (threadIdx.x == 0) { s_prefix = 0; out[0] = 0; }
        // 2. publish it, then sum every lower chunk's aggregate
        if (!solo && threadIdx.x < 32) {
            const int lane = threadIdx.x;
            if (lane == 0) st_release(&status[c], ST_AGG | (unsigned long long)agg);
            int64_t p = 0;
            for (int j = lane; j < c; j += 32) {
                unsigned long long st = ld_acquire(&status[j]);
                while ((st >> 62) == 0) st = ld_acquire(&status[j]);
                p += (int64_t)(st & ST_VAL);
            }
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) p += __shfl_xor_sync(0xffffffffu, p, o);
            if (lane == 0) {
                s_prefix = p;
                if (c == nch - 1 && total_dev) *total_dev = p + agg;
                if (c == 0) out[0] = 0;
            }
        }
        __syncthreads();
        // 3. the chunk's inclusive sums, written to out[i + 1]; the next tile's loads are issued before
        // this tile's block scan (chunks of several tiles: n > 1.2 M)
        int64_t run = s_prefix;
        for (int64_t base = lo; base < hi; base += SCAN_TILE) {
            const int64_t i = base + toff;
            int64_t nx[SCAN_ITEMS];
            if (base + SCAN_TILE < hi) scan_ld16(in, i + SCAN_TILE, hi, vec, nx);
            int64_t ts = 0;
#pragma unroll
            for (int q = 0; q < SCAN_ITEMS; ++q) ts += v[q];
            int64_t tot;
            int64_t r = run + block_excl_scan(ts, s_warp, &tot);
#pragma unroll
            for (int q = 0; q < SCAN_ITEMS; ++q) {
                r += v[q];
                if (i + q < hi) out[i + q + 1] = r;
            }
            run += tot;
            if (base + SCAN_TILE < hi) {
#pragma unroll
                for (int q = 0; q < SCAN_ITEMS; ++q) v[q] = nx[q];
            }
        }
        if (solo && threadIdx.x == 0 && total_dev) *total_dev = run;
    }
    if (solo) return;
    // the last CTA to finish clears the chunk flags and the counters
    __syncthreads();
    if (threadIdx.x == 0) {
        fence_gpu();
        s_last = (atomicAdd(&ctr[1], 1u) == (unsigned)G - 1);
    }
    __syncthreads();
    if (s_last) {
        for (int j = threadIdx.x; j < nch; j += blockDim.x) status[j] = 0;
        if (threadIdx.x == 0) { ctr[0] = 0; ctr[1] = 0; }
        fence_gpu();
    }
}

void ensure_scan_scratch(betty_ctx* c, int64_t n_cap, cudaStream_t s) {
    const int64_t tiles = (n_cap + SCAN_TILE - 1) / SCAN_TILE + 1;   // >= the grid
    if (tiles > c->L().scan_status_cap) {
        // growing is only legal outside graph capture; plan creation sizes it first.  A plan's
        // instantiated CUDA graph holds the old pointer by value, so the old buffer is retired (kept
        // until the context is destroyed), never freed here (a later larger call must not turn an
        // existing graph's scratch into freed memory)
        if (c->L().scan_status) c->retired.push_back(c->L().scan_status);
        const int64_t cap = tiles * 2 + 1024;
        c->L().scan_status = (unsigned long long*)ctx_alloc(c, sizeof(unsigned long long) * cap, s);
        cudaMemsetAsync(c->L().scan_status, 0, sizeof(unsigned long long) * cap, s);
        c->L().scan_status_cap = cap;
    }
}

template <typename Tin>
static void scan_impl(betty_ctx* c, const Tin* in, int64_t* out, const int64_t* n_dev, int64_t n_fixed, int64_t n_cap,
                      int64_t* total_dev, cudaStream_t s) {
    if (!n_dev) n_cap = n_fixed;
    ensure_scan_scratch(c, n_cap, s);
    // one chunk of tiles per CTA; a one-tile scan runs on one CTA without flags or atomics (one CTA
    // walking up to 16 tiles alone was measured slower: C3 step 4.087 -> 4.117 ms)
    const int64_t chunks = (n_cap + SCAN_TILE - 1) / SCAN_TILE;
    const int grid = (int)std::min<int64_t>(std::max<int64_t>(chunks, 1), (int64_t)c->num_sms * 2);
    k_scan<Tin><<<grid, SCAN_THREADS, 0, s>>>(in, out, n_dev, n_fixed, total_dev, c->L().scan_status,
                                              c->L().counters + CTR_SCAN);
}

void scan_i64(betty_ctx* c, const int64_t* in, int64_t* out, const int64_t* n_dev, int64_t n_fixed, int64_t n_cap,
              int64_t* total_dev, cudaStream_t s) {
    scan_impl(c, in, out, n_dev, n_fixed, n_cap, total_dev, s);
}
void scan_i32(betty_ctx* c, const int32_t* in, int64_t* out, const int64_t* n_dev, int64_t n_fixed, int64_t n_cap,
              int64_t* total_dev, cudaStream_t s) {
    scan_impl(c, in, out, n_dev, n_fixed, n_cap, total_dev, s);
}

// ---------------------------------------------------------------- memset
__global__ void k_memset(uint32_t* p, uint32_t v, const int64_t* n_dev, int64_t elem_words, int64_t n_fixed) {
    const int64_t n = (n_dev ? *n_dev : n_fixed) * elem_words;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        p[i] = v;
}
void memset_dev(void* p, int value, const int64_t* n_dev, int64_t elem_bytes, int64_t n_cap, cudaStream_t s) {
    // elem_bytes must be a multiple of 4; value is replicated per byte
    const uint32_t v = (uint32_t)(value & 0xff) * 0x01010101u;
    const int64_t words = n_cap * (elem_bytes / 4);
    int grid = (int)std::min<int64_t>((words + 255) / 256 + 1, 148 * 8);
    k_memset<<<grid, 256, 0, s>>>((uint32_t*)p, v, n_dev, elem_bytes / 4, n_cap);
}

// --------------------------------------------------------- segmented sort
constexpr int SEG_WARP_MAX = 512;
constexpr int SEG_CTA_MAX = 32768;

__device__ void smem_bitonic(int32_t* s, int P, int tid, int nthreads, bool warp_only) {
    for (int k = 2; k <= P; k <<= 1) {
        for (int j = k >> 1; j > 0; j >>= 1) {
            for (int i = tid; i < P; i += nthreads) {
                const int ixj = i ^ j;
                if (ixj > i) {
                    const int32_t a = s[i], b = s[ixj];
                    const bool up = ((i & k) == 0);
                    if ((a > b) == up) { s[i] = b; s[ixj] = a; }
                }
            }
            if (warp_only) __syncwarp(); else __syncthreads();
        }
    }
}

// dup: also flag a repeated key inside a segment (DEVERR_DUP_EDGE; the transpose's repeated-edge check,
// folded into the sort instead of a separate pass over the CSC)
__global__ void __launch_bounds__(256) k_segsort_warp(const int64_t* __restrict__ ptr, int32_t* __restrict__ keys,
                                                      const int64_t* nseg_dev, int64_t nseg_fixed, int64_t* big,
                                                      int* big_cnt, int64_t big_cap, int* dev_err, int dup) {
    __shared__ int32_t buf[8][SEG_WARP_MAX];
    const int64_t nseg = nseg_dev ? *nseg_dev : nseg_fixed;
    const int w = warp_id(), lane = lane_id();
    const int64_t gw = blockIdx.x * 8ll + w, nw = gridDim.x * 8ll;
    // a warp takes 32 consecutive segments: segments of <= SEG_THREAD_MAX keys are
    // insertion-sorted by one lane each (most CSC columns of a sampled block hold
    // 1-4 entries); longer ones are sorted warp-cooperatively one at a time
    constexpr int SEG_THREAD_MAX = 8;
    for (int64_t s0 = gw * 32; s0 < nseg; s0 += nw * 32) {
        const int64_t my = s0 + lane;
        int64_t mb = 0, ml = 0;
        if (my < nseg) { mb = ptr[my]; ml = ptr[my + 1] - mb; }
        if (ml > 1 && ml <= SEG_THREAD_MAX) {
            int32_t k[SEG_THREAD_MAX];
#pragma unroll
            for (int i = 0; i < SEG_THREAD_MAX; ++i) k[i] = i < ml ? keys[mb + i] : INT_MAX;
#pragma unroll
            for (int i = 1; i < SEG_THREAD_MAX; ++i)
#pragma unroll
                for (int j = i; j > 0; --j)
                    if (k[j] < k[j - 1]) { const int32_t t = k[j]; k[j] = k[j - 1]; k[j - 1] = t; }
#pragma unroll
            for (int i = 0; i < SEG_THREAD_MAX; ++i) if (i < ml) keys[mb + i] = k[i];
            if (dup) {
                bool rep = false;
#pragma unroll
                for (int i = 1; i < SEG_THREAD_MAX; ++i) rep |= i < ml && k[i] == k[i - 1];
                if (rep) atomicOr(dev_err, DEVERR_DUP_EDGE);
            }
        }
        unsigned long_mask = __ballot_sync(0xffffffffu, ml > SEG_THREAD_MAX);
        while (long_mask) {
            const int src = __ffs(long_mask) - 1;
            long_mask &= long_mask - 1;
            const int64_t seg = s0 + src;
            const int64_t b = __shfl_sync(0xffffffffu, mb, src), len = __shfl_sync(0xffffffffu, ml, src);
            if (len <= 32) {
                int32_t x = lane < len ? keys[b + lane] : INT_MAX;
                x = warp_bitonic32(x);
                if (lane < len) keys[b + lane] = x;
                const int32_t prev = __shfl_up_sync(0xffffffffu, x, 1);
                if (dup && lane > 0 && lane < len && x == prev) atomicOr(dev_err, DEVERR_DUP_EDGE);
            } else if (len <= SEG_WARP_MAX) {
                int P = 64;
                while (P < len) P <<= 1;
                for (int i = lane; i < P; i += 32) buf[w][i] = i < len ? keys[b + i] : INT_MAX;
                __syncwarp();
                smem_bitonic(buf[w], P, lane, 32, true);
                for (int i = lane; i < len; i += 32) {
                    keys[b + i] = buf[w][i];
                    if (dup && i > 0 && buf[w][i] == buf[w][i - 1]) atomicOr(dev_err, DEVERR_DUP_EDGE);
                }
                __syncwarp();
            } else if (lane == 0) {
                const int i = atomicAdd(big_cnt, 1);
                if (i < big_cap) big[i] = seg; else atomicOr(dev_err, DEVERR_OVERFLOW);
            }
        }
    }
}

__global__ void __launch_bounds__(1024) k_segsort_big(const int64_t* __restrict__ ptr, int32_t* __restrict__ keys,
                                                      const int64_t* big, int* big_cnt, int* dev_err, int dup) {
    extern __shared__ int32_t sbuf[];
    const int n_big = *big_cnt;
    for (int t = blockIdx.x; t < n_big; t += gridDim.x) {
        const int64_t seg = big[t];
        const int64_t b = ptr[seg], len = ptr[seg + 1] - b;
        if (len > SEG_CTA_MAX) {
            if (threadIdx.x == 0) atomicOr(dev_err, DEVERR_OVERFLOW);
            continue;
        }
        int P = 1024;
        while (P < len) P <<= 1;
        for (int i = threadIdx.x; i < P; i += blockDim.x) sbuf[i] = i < len ? keys[b + i] : INT_MAX;
        __syncthreads();
        smem_bitonic(sbuf, P, threadIdx.x, blockDim.x, false);
        for (int i = threadIdx.x; i < len; i += blockDim.x) {
            keys[b + i] = sbuf[i];
            if (dup && i > 0 && sbuf[i] == sbuf[i - 1]) atomicOr(dev_err, DEVERR_DUP_EDGE);
        }
        __syncthreads();
    }
}

__global__ void k_reset_int(int* p) { *p = 0; }

void init_prims_attrs() {
    cudaFuncSetAttribute(k_segsort_big, cudaFuncAttributeMaxDynamicSharedMemorySize, SEG_CTA_MAX * 4);
}

static void segsort_impl(betty_ctx* c, const int64_t* ptr, int32_t* keys, const int64_t* nseg_dev, int64_t nseg_fixed,
                         int64_t nseg_cap, bool dup, cudaStream_t s) {
    if (!nseg_dev) nseg_cap = nseg_fixed;
    int grid = (int)std::min<int64_t>((nseg_cap + 255) / 256 + 1, (int64_t)c->num_sms * 8);
    k_reset_int<<<1, 1, 0, s>>>(c->L().big_count);
    k_segsort_warp<<<grid, 256, 0, s>>>(ptr, keys, nseg_dev, nseg_fixed, c->L().big_list, c->L().big_count, c->L().big_list_cap,
                                        c->dev_err, dup ? 1 : 0);
    k_segsort_big<<<c->num_sms, 1024, SEG_CTA_MAX * 4, s>>>(ptr, keys, c->L().big_list, c->L().big_count, c->dev_err,
                                                            dup ? 1 : 0);
}
void segsort_i32(betty_ctx* c, const int64_t* ptr, int32_t* keys, const int64_t* nseg_dev, int64_t nseg_fixed,
                 int64_t nseg_cap, cudaStream_t s) {
    segsort_impl(c, ptr, keys, nseg_dev, nseg_fixed, nseg_cap, false, s);
}

// ------------------------------------------------------------- transpose
__global__ void k_hist(const int32_t* __restrict__ idx, const int64_t* n_edges_dev, int32_t* cnt) {
    const int64_t n = *n_edges_dev;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x)
        atomicAdd(&cnt[idx[e]], 1);
}

__global__ void k_scatter_t(const int64_t* __restrict__ indptr, const int32_t* __restrict__ idx,
                            const int64_t* n_rows_dev, const int64_t* __restrict__ t_indptr, int32_t* cursor,
                            int32_t* __restrict__ t_idx) {
    const int64_t n = *n_rows_dev;
    const int lane = lane_id();
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t r = gw; r < n; r += nw) {
        const int64_t b = indptr[r], e = indptr[r + 1];
        for (int64_t i = b + lane; i < e; i += 32) {
            const int32_t col = idx[i];
            const int32_t k = atomicSub(&cursor[col], 1) - 1;     // the histogram counts down to 0
            t_idx[t_indptr[col] + k] = (int32_t)r;
        }
    }
}

void csr_transpose(betty_ctx* c, const int64_t* indptr, const int32_t* idx, const int64_t* n_rows_dev,
                   const int64_t* n_cols_dev, const int64_t* n_edges_dev, int64_t rows_cap, int64_t cols_cap,
                   int64_t edges_cap, int64_t* t_indptr, int32_t* t_idx, int32_t* cnt, bool dup_check,
                   cudaStream_t s) {
    const int g_e = (int)std::min<int64_t>((edges_cap + 255) / 256 + 1, (int64_t)c->num_sms * 8);
    const int g_r = (int)std::min<int64_t>((rows_cap * 32 + 255) / 256 + 1, (int64_t)c->num_sms * 8);
    memset_dev(cnt, 0, n_cols_dev, 4, cols_cap, s);
    k_hist<<<g_e, 256, 0, s>>>(idx, n_edges_dev, cnt);
    scan_i32(c, cnt, t_indptr, n_cols_dev, 0, cols_cap, nullptr, s);
    k_scatter_t<<<g_r, 256, 0, s>>>(indptr, idx, n_rows_dev, t_indptr, cnt, t_idx);
    segsort_impl(c, t_indptr, t_idx, n_cols_dev, 0, cols_cap, dup_check, s);   // (+ the repeated-edge check)
}

}  // namespace betty
