// partition.cpp -- host-side K-way partitioner of the REG (outside the hot
// path: Alg. 1 line 8, uses METIS; METIS is not available in
// this image).  Greedy graph growing, the initial-partitioning
// scheme of multilevel partitioners: each part grows from the lowest-id
// unassigned output by repeatedly absorbing the unassigned output with the
// largest total REG weight to the part (= the most shared inputs, so the
// fewest duplicated inputs when it is cut off), up to a balanced size
// ceil-or-floor(n/K).  Deterministic (ties: smaller id).  Host pointers.
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
