"""Pins of the oracle's micro-batch extraction (batch-level partitioning,
PAPER.md:535-547 §4.2.3; block generation + index mapping PAPER.md:1141-1187):
the golden example, K=1 identity, exhaustive k-hop closure, and the
partition invariants (disjoint V_k covering V; union of U_k = U)."""
import numpy as np
import pytest

import oracle
import synth
from tests.helpers import closure, load_golden, tiny


def golden_full(g):
    rows = [{int(k): v for k, v in g["rows"][str(l)].items()} for l in (0, 1)]
    return synth.blocks_from_rows(g["seeds"], rows)


def test_golden_full_blocks():
    g = load_golden("g1.json")
    full = golden_full(g)
    for l in (0, 1):
        e = g["full"][str(l)]
        assert list(full[l].src_gid) == e["src_gid"]
        assert list(full[l].indptr) == e["indptr"]
        assert list(full[l].nbr_pos) == e["idx"]


def test_golden_micro_batches():
    g = load_golden("g1.json")
    full = golden_full(g)
    part = np.array(g["part"], dtype=np.int32)
    srcs = set()
    total = 0
    for k in range(g["K"]):
        mb = oracle.extract(full, part, g["K"], k)
        for l in (0, 1):
            e = g["mb"][str(k)][str(l)]
            b = mb[l]
            assert list(b.src_pos) == e["src_pos"], (k, l)
            assert list(b.src_gid) == e["src_gid"], (k, l)
            assert list(b.indptr) == e["indptr"], (k, l)
            assert list(b.indices) == e["idx"], (k, l)
            assert list(b.t_indptr) == e["t_indptr"], (k, l)
            assert list(b.t_indices) == e["t_idx"], (k, l)
        srcs |= set(mb[0].src_gid.tolist())
        total += mb[0].n_src
    assert len(srcs) == g["checks"]["union_src0"]
    assert total == g["checks"]["sum_src0"]
    assert total - len(srcs) == g["checks"]["redundancy"]


def test_golden_mean_values():
    """With 1-d features h(g)=g the layer-0 mean of node 4 is 16/3, of node 11
    (no sampled neighbour) 0: computed through the oracle's forward with
    W_self=0, W_neigh=1, b=0 on a 1-layer model whose outputs are 4 and 11."""
    g = load_golden("g1.json")
    rows0 = {int(k): v for k, v in g["rows"]["0"].items()}
    full = synth.blocks_from_rows([4, 11], [rows0])
    feats = np.arange(12, dtype=np.float32).reshape(12, 1)
    params = np.array([0.0, 1.0, 0.0], dtype=np.float32)  # W_self [1x1], W_neigh [1x1], b [1]
    _, _, logits = oracle.sage([1, 1], "mean", False, full, params, feats, np.zeros(12, np.int32), 1.0,
                               want_logits=True)
    assert logits[0, 0] == pytest.approx(g["checks"]["mean_l0"]["4"], rel=1e-15)
    assert logits[1, 0] == g["checks"]["mean_l0"]["11"]


def check_block_is_full(mb, full):
    for l in range(len(full)):
        a, b = mb[l], full[l]
        assert a.n_dst == b.n_dst and a.n_src == b.n_src
        np.testing.assert_array_equal(a.indptr, b.indptr)
        np.testing.assert_array_equal(a.indices, b.nbr_pos)
        np.testing.assert_array_equal(a.src_pos, np.arange(b.n_src))
        np.testing.assert_array_equal(a.src_gid, b.src_gid)


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_k1_reproduces_full_batch(seed):
    g, sd, blocks, feats, labels = tiny(n=300, pairs=900, fanouts=(3, 4, 5), n_out=40, seed=seed)
    mb = oracle.extract(blocks, np.zeros(len(sd), np.int32), 1, 0)
    check_block_is_full(mb, blocks)


def check_closure(blocks, mb, out_gids):
    ref = closure(blocks, out_gids)
    for l, b in enumerate(mb):
        dst, src, edges = ref[l]
        assert set(b.src_gid[:b.n_dst].tolist()) == dst
        assert set(b.src_gid.tolist()) == src
        assert len(set(b.src_gid.tolist())) == b.n_src          # no duplicate sources
        got = {(int(b.src_gid[b.indices[e]]), int(b.src_gid[i]))
               for i in range(b.n_dst) for e in range(b.indptr[i], b.indptr[i + 1])}
        assert got == edges
        assert b.n_edges == len(edges)
        # src_pos indexes the full-batch src list and maps to the same gid
        np.testing.assert_array_equal(blocks[l].src_gid[b.src_pos], b.src_gid)
        # canonical order: dst prefix then ascending full src position
        assert (np.diff(b.src_pos[b.n_dst:]) > 0).all()
        # CSC is the transpose with ascending dst ids per column
        pairs = sorted((int(b.indices[e]), i) for i in range(b.n_dst) for e in range(b.indptr[i], b.indptr[i + 1]))
        cols = [(s, int(b.t_indices[e])) for s in range(b.n_src) for e in range(b.t_indptr[s], b.t_indptr[s + 1])]
        assert cols == pairs


@pytest.mark.parametrize("seed", [1, 2])
def test_k_equals_n_out_is_single_output_tree(seed):
    g, sd, blocks, feats, labels = tiny(n=200, pairs=700, fanouts=(3, 4), n_out=15, seed=seed)
    n_out = len(sd)
    part = np.arange(n_out, dtype=np.int32)
    for k in range(n_out):
        mb = oracle.extract(blocks, part, n_out, k)
        check_closure(blocks, mb, [int(sd[k])])


@pytest.mark.parametrize("seed,K", [(1, 2), (2, 3), (3, 5), (4, 7)])
def test_any_partition_closure_and_cover(seed, K):
    g, sd, blocks, feats, labels = tiny(n=250, pairs=900, fanouts=(2, 3, 4), n_out=30, seed=seed)
    part = synth.random_partition(len(sd), K, seed)
    L = len(blocks)
    union = [set() for _ in range(L)]
    outs = []
    sum_src0 = 0
    for k in range(K):
        mb = oracle.extract(blocks, part, K, k)
        check_closure(blocks, mb, [int(x) for x in sd[part == k]])
        outs += mb[-1].src_gid[:mb[-1].n_dst].tolist()
        for l in range(L):
            union[l] |= set(mb[l].src_gid.tolist())
        sum_src0 += mb[0].n_src
    assert sorted(outs) == sorted(sd.tolist())                  # disjoint union of V_k is V
    for l in range(L):
        assert union[l] == set(blocks[l].src_gid.tolist())     # union of U_k is U
    assert sum_src0 >= blocks[0].n_src


def test_empty_part_and_bad_input():
    g, sd, blocks, feats, labels = tiny(seed=4)
    part = np.zeros(len(sd), np.int32)
    mb = oracle.extract(blocks, part, 3, 2)                      # part 2 is empty
    for b in mb:
        assert b.n_dst == 0 and b.n_src == 0 and b.n_edges == 0
    with pytest.raises(ValueError):
        oracle.extract(blocks, part, 3, 3)                       # k out of range
    bad = part.copy()
    bad[0] = 5
    with pytest.raises(ValueError):
        oracle.extract(blocks, bad, 3, 0)                        # part[] out of range
