"""Pins of the oracle's memory estimate (Table 3 terms (1)-(8))
and of the memory-aware re-partitioning loop: the golden
G1 numbers hand-derived in tests/golden/g1.json, the parameter count against
the flat layout of the input generator, block sizes counted independently
from the sampled rows, and the loop's K choice on G1."""
import numpy as np
import pytest

import oracle
import synth
from tests.helpers import closure, load_golden, tiny
from tests.test_oracle_extract import golden_full


def test_golden_terms():
    g = load_golden("g1.json")
    full = golden_full(g)
    m = g["mem"]
    part = np.array(g["part"], dtype=np.int32)
    for aggr in ("mean", "pool"):
        for k in range(2):
            key = f"mb{k}"
            if key not in m[aggr]:
                continue
            t = oracle.mem_estimate(m["dims"], aggr, oracle.extract(full, part, 2, k))
            assert list(t) == m[aggr][key], (aggr, k)
    t = oracle.mem_estimate(m["dims"], "mean", full)
    assert list(t) == m["mean"]["full"]


def test_golden_loop():
    g = load_golden("g1.json")
    full = golden_full(g)
    m = g["mem"]
    parts = {1: np.zeros(2, np.int32), 2: np.array(g["part"], np.int32)}
    for cap, K in m["loop"]:
        k, part, peak = oracle.memory_aware_k(full, m["dims"], "mean", cap, lambda K_: parts[K_])
        assert k == K, (cap, k)
        if K > 0:
            assert peak <= cap


@pytest.mark.parametrize("aggr", ["mean", "pool"])
def test_terms_independent(aggr):
    """Every term re-derived from independent counts: parameters from the
    generator's flat layout, block sizes from the brute-force k-hop closure."""
    g, sd, blocks, feats, labels = tiny(n=300, pairs=900, fanouts=(3, 4, 5), n_out=30, F=6, C=4, seed=4)
    dims = [6, 8, 7, 4]
    K = 3
    part = synth.random_partition(30, K, 7)
    n_params = len(synth.init_params(dims, aggr, seed=1))
    n_agg = sum(dims[l] * dims[l] + dims[l] for l in range(3)) if aggr == "pool" else 0
    for k in range(K):
        outs = [int(sd[i]) for i in range(30) if part[i] == k]
        cl = closure(blocks, outs)
        nd = [len(cl[l][0]) for l in range(3)]
        ns = [len(cl[l][1]) for l in range(3)]
        ne = [len(cl[l][2]) for l in range(3)]
        t = oracle.mem_estimate(dims, aggr, oracle.extract(blocks, part, K, k))
        assert t[0] == n_params - n_agg
        assert t[1] == ns[0] * dims[0]
        assert t[2] == len(outs)
        assert t[3] == 3 * sum(ne)
        assert t[4] == sum(nd[l] * dims[l + 1] for l in range(3))
        inter = sum(((ns[l] + nd[l]) if aggr == "pool" else nd[l]) * dims[l] for l in range(3))
        assert t[5] == inter
        assert t[6] == n_params and t[7] == 2 * n_params
        assert t[8] == t[0] + t[1] + t[2] + t[3] + t[4] + t[7] + max(t[5], t[6])


def test_loop_monotone_capacity():
    """A larger capacity never needs more micro-batches (same partitioner);
    the chosen K is the first one whose every estimate fits."""
    g, sd, blocks, feats, labels = tiny(n=400, pairs=1600, fanouts=(3, 5), n_out=40, F=5, C=3, seed=5)
    dims = [5, 16, 3]
    fn = lambda K: synth.range_partition(40, K)
    peaks = {K: max(int(oracle.mem_estimate(dims, "mean", oracle.extract(blocks, fn(K), K, k))[8])
                    for k in range(K)) for K in range(1, 11)}
    for cap in sorted(set(peaks.values())):
        K, part, peak = oracle.memory_aware_k(blocks, dims, "mean", cap, fn, K_max=10)
        assert K == min(k for k in peaks if peaks[k] <= cap)
        assert peak == peaks[K]
    K, part, peak = oracle.memory_aware_k(blocks, dims, "mean", min(peaks.values()) - 1, fn, K_max=10)
    assert K == -1
