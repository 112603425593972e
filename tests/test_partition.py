"""Host REG partitioner (outside the hot path; stands in for METIS, Alg. 1
line 8): validity, balance, and that it cuts far less REG weight -- i.e.
creates less input redundancy -- than a random partition (§4.3.2)."""
import numpy as np
import pytest

import oracle
import synth
import paper_conf_asplos_yangzd023_b200 as B
from tests.helpers import tiny


def cut_weight(rp, col, w, part):
    rows = np.repeat(np.arange(len(rp) - 1), np.diff(rp))
    return int(w[part[rows] != part[col]].sum())


@pytest.mark.parametrize("K", [1, 2, 5, 16])
def test_partition_valid_balanced(K):
    g, sd, blocks, feats, labels = tiny(n=3000, pairs=12000, fanouts=(4, 6), n_out=400, n_comm=20, mu=0.1, seed=2)
    rp, col, w = oracle.reg(blocks[-1].n_src, blocks[-1].indptr, blocks[-1].nbr_pos)
    part = B.betty_reg_partition(rp, col, w, K)
    assert part.shape == (400,) and part.min() >= 0 and part.max() < K
    sizes = np.bincount(part, minlength=K)
    assert sizes.max() - sizes.min() <= 1
    assert np.array_equal(part, B.betty_reg_partition(rp, col, w, K))   # deterministic


def test_partition_reduces_redundancy_vs_random():
    g, sd, blocks, feats, labels = tiny(n=3000, pairs=12000, fanouts=(4, 6), n_out=400, n_comm=20, mu=0.1, seed=3)
    rp, col, w = oracle.reg(blocks[-1].n_src, blocks[-1].indptr, blocks[-1].nbr_pos)
    K = 8
    ours = B.betty_reg_partition(rp, col, w, K)
    rnd = synth.random_partition(400, K, 1)
    assert cut_weight(rp, col, w, ours) < 0.8 * cut_weight(rp, col, w, rnd)
    red = [sum(oracle.extract(blocks, p, K, k)[0].n_src for k in range(K)) for p in (ours, rnd)]
    assert red[0] < red[1]


@pytest.mark.parametrize("K", [1, 2, 7, 32])
def test_multilevel_valid_bounded(K):
    g, sd, blocks, feats, labels = tiny(n=3000, pairs=12000, fanouts=(4, 6), n_out=400, n_comm=20, mu=0.1, seed=2)
    rp, col, w = oracle.reg(blocks[-1].n_src, blocks[-1].indptr, blocks[-1].nbr_pos)
    part = B.betty_reg_partition(rp, col, w, K, method="multilevel", imbalance=0.03)
    assert part.shape == (400,) and part.min() >= 0 and part.max() < K
    assert np.bincount(part, minlength=K).max() <= int(np.ceil(1.03 * 400 / K))
    assert np.array_equal(part, B.betty_reg_partition(rp, col, w, K, method="multilevel"))


@pytest.mark.parametrize("K", [4, 16, 64])
def test_multilevel_beats_greedy(K):
    """The METIS scheme (Alg. 1 line 8) cuts less REG weight than greedy growing, and so
    duplicates fewer inputs across micro-batches (Eq. 4)."""
    g, sd, blocks, feats, labels = tiny(n=30000, pairs=150000, fanouts=(5, 10), n_out=4000, n_comm=200, mu=0.1,
                                        seed=2)
    rp, col, w = oracle.reg(blocks[-1].n_src, blocks[-1].indptr, blocks[-1].nbr_pos)
    ml = B.betty_reg_partition(rp, col, w, K, method="multilevel")
    gr = B.betty_reg_partition(rp, col, w, K)
    assert cut_weight(rp, col, w, ml) < cut_weight(rp, col, w, gr)
    red = [sum(oracle.extract(blocks, p, K, k)[0].n_src for k in range(K)) for p in (ml, gr)]
    assert red[0] < red[1]


def test_multilevel_edge_cases():
    rp = np.zeros(1, np.int64)
    assert len(B.betty_reg_partition(rp, np.zeros(0, np.int32), np.zeros(0, np.int32), 3, method="multilevel")) == 0
    # no REG edges at all (every output reads distinct inputs): still a valid bounded partition
    rp = np.zeros(101, np.int64)
    part = B.betty_reg_partition(rp, np.zeros(0, np.int32), np.zeros(0, np.int32), 4, method="multilevel")
    assert np.bincount(part, minlength=4).max() <= 26
    with pytest.raises(Exception):
        B.betty_reg_partition(np.array([0, 1], np.int64), np.array([5], np.int32), np.array([1], np.int32), 2,
                              method="multilevel")


def test_induced_subgraph_brute_force():
    from paper_conf_asplos_yangzd023_b200.partition import induced_subgraph
    g = synth.graph(300, 1500, 5, 0.2, 0.4, 4)
    nodes = np.sort(np.random.default_rng(1).choice(300, 80, replace=False)).astype(np.int32)
    ip, col = induced_subgraph(g.indptr, g.indices, nodes)
    pos = {int(v): i for i, v in enumerate(nodes)}
    for i, v in enumerate(nodes):
        want = sorted(pos[int(u)] for u in g.indices[g.indptr[v]:g.indptr[v + 1]] if int(u) in pos)
        assert list(col[ip[i]:ip[i + 1]]) == want
    # symmetric (the raw graph is undirected)
    pairs = {(i, int(j)) for i in range(len(nodes)) for j in col[ip[i]:ip[i + 1]]}
    assert all((j, i) in pairs for (i, j) in pairs)


@pytest.mark.parametrize("K", [2, 8])
def test_raw_graph_partition_valid_and_REG_creates_less_redundancy(K):
    """The paper's Metis baseline (reading P2) is a valid, balanced K-way split of the outputs, and the
    REG partition (same multilevel partitioner, REG weights) creates fewer redundant inputs
    (Betty has the least redundancy in all cases)."""
    from paper_conf_asplos_yangzd023_b200.partition import raw_graph_partition
    g, sd, blocks, feats, labels = tiny(n=3000, pairs=12000, fanouts=(4, 6), n_out=400, n_comm=20, mu=0.1, seed=5)
    part = raw_graph_partition(g.indptr, g.indices, sd, K)
    assert part.shape == (400,) and part.min() >= 0 and part.max() < K
    assert np.bincount(part, minlength=K).max() <= int(np.ceil(1.03 * 400 / K)) + 1
    assert np.array_equal(part, raw_graph_partition(g.indptr, g.indices, sd, K))
    rp, col, w = oracle.reg(blocks[-1].n_src, blocks[-1].indptr, blocks[-1].nbr_pos)
    reg = B.betty_reg_partition(rp, col, w, K, method="multilevel")
    red = [sum(oracle.extract(blocks, p, K, k)[0].n_src for k in range(K)) for p in (reg, part)]
    assert red[0] <= red[1]
