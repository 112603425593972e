"""Host part of §4.4: the library's Table 3 estimator
(pure host arithmetic behind the C ABI) equals the oracle's, term by term,
on the golden G1 sizes and on random sizes."""
import numpy as np
import pytest

import oracle
import paper_conf_asplos_yangzd023_b200 as B
from tests.helpers import load_golden


class _Sz:
    def __init__(self, nd, ns, ne):
        self.n_dst, self.n_src = int(nd), int(ns)
        self.indptr = np.array([0, ne], dtype=np.int64)


def test_estimate_golden():
    g = load_golden("g1.json")
    m = g["mem"]
    sizes = {"mb0": [[5, 9, 9], [1, 5, 4]], "mb1": [[5, 7, 9], [1, 5, 4]], "full": [[7, 10, 11], [2, 7, 8]]}
    for aggr in ("mean", "pool"):
        for key, want in m[aggr].items():
            t = B.betty_mem_estimate(B.Model(m["dims"], aggr), np.array(sizes[key]))
            assert list(t) == want, (aggr, key)


@pytest.mark.parametrize("aggr", ["mean", "pool"])
def test_estimate_matches_oracle_random(aggr):
    rng = np.random.default_rng(11)
    for trial in range(50):
        L = int(rng.integers(1, 6))
        dims = [int(x) for x in rng.integers(1, 600, L + 1)]
        nd = rng.integers(0, 10 ** 6, L)
        ns = nd + rng.integers(0, 10 ** 6, L)
        ne = rng.integers(0, 10 ** 8, L)
        sizes = np.stack([nd, ns, ne], axis=1)
        t = B.betty_mem_estimate(B.Model(dims, aggr), sizes)
        o = oracle.mem_estimate(dims, aggr, [_Sz(*sizes[l]) for l in range(L)])
        assert np.array_equal(t, o), (trial, t, o)
