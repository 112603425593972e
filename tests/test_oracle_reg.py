"""Pins of the oracle's REG (Eq. 2-4, Alg. 1 l.1-7) against
brute force, scipy, closed forms and invariants -- none of which reuse the
oracle's own loops."""
import itertools

import numpy as np
import pytest
import scipy.sparse as sp

import oracle
from tests.helpers import load_golden, tiny

pytestmark = pytest.mark.filterwarnings("ignore")


def reg_dense(indptr, col, w, n):
    C = np.zeros((n, n), dtype=np.int64)
    for i in range(n):
        for e in range(indptr[i], indptr[i + 1]):
            C[i, col[e]] = w[e]
    return C


def random_block(rng, n_out, n_src, max_deg, allow_dups=False):
    rows = []
    for _ in range(n_out):
        d = rng.integers(0, max_deg + 1)
        if allow_dups:
            r = list(rng.integers(0, n_src, d))
        else:
            r = list(rng.choice(n_src, size=min(d, n_src), replace=False))
        rows.append(r)
    indptr = np.zeros(n_out + 1, dtype=np.int64)
    for i, r in enumerate(rows):
        indptr[i + 1] = indptr[i] + len(r)
    idx = np.array([x for r in rows for x in r], dtype=np.int32)
    return rows, indptr, idx


@pytest.mark.parametrize("seed", range(8))
def test_reg_brute_force_pairs(seed):
    """c_ij == |S_i ∩ S_j| for every pair i != j (Eq. 4 read as set intersection)."""
    rng = np.random.default_rng(seed)
    n_out, n_src = int(rng.integers(1, 40)), int(rng.integers(1, 30))
    rows, indptr, idx = random_block(rng, n_out, n_src, 8)
    C = reg_dense(*oracle.reg(n_src, indptr, idx), n_out)
    S = [set(r) for r in rows]
    for i, j in itertools.product(range(n_out), repeat=2):
        want = 0 if i == j else len(S[i] & S[j])
        assert C[i, j] == want, (i, j)


@pytest.mark.parametrize("seed", range(4))
def test_reg_matches_scipy_product(seed):
    """REG == (B B^T) minus its diagonal, B the binary n_out x n_src matrix
    (library routine, test-only)."""
    rng = np.random.default_rng(100 + seed)
    n_out, n_src = 300, 500
    rows, indptr, idx = random_block(rng, n_out, n_src, 25)
    B = sp.csr_matrix((np.ones(len(idx)), idx, indptr), shape=(n_out, n_src))
    B.data[:] = 1.0
    Cs = (B @ B.T).tolil()
    Cs.setdiag(0)
    Cs = Cs.tocsr()
    Cs.eliminate_zeros()
    Cs.sort_indices()
    rp, col, w = oracle.reg(n_src, indptr, idx)
    np.testing.assert_array_equal(rp, Cs.indptr)
    np.testing.assert_array_equal(col, Cs.indices)
    np.testing.assert_array_equal(w, Cs.data.astype(np.int64))


def test_reg_multi_edges_collapse():
    """A is binary (Eq. 2: 'a binary value indicating if there is any
    connection'): duplicate (u,i) entries count once."""
    rng = np.random.default_rng(7)
    rows, indptr, idx = random_block(rng, 30, 10, 12, allow_dups=True)
    dd = [sorted(set(r)) for r in rows]
    ip2 = np.zeros(31, dtype=np.int64)
    for i, r in enumerate(dd):
        ip2[i + 1] = ip2[i] + len(r)
    idx2 = np.array([x for r in dd for x in r], dtype=np.int32)
    a = oracle.reg(10, indptr, idx)
    b = oracle.reg(10, ip2, idx2)
    for x, y in zip(a, b):
        np.testing.assert_array_equal(x, y)


def test_reg_closed_form_star():
    """One source shared by n outputs -> complete graph K_n, all weights 1."""
    n = 9
    indptr = np.arange(n + 1, dtype=np.int64)
    idx = np.zeros(n, dtype=np.int32)
    C = reg_dense(*oracle.reg(1, indptr, idx), n)
    np.testing.assert_array_equal(C, np.ones((n, n), dtype=np.int64) - np.eye(n, dtype=np.int64))


def test_reg_closed_form_complete_bipartite():
    """K_{m,n}: every output sees all m sources -> all off-diagonal weights m."""
    m, n = 6, 7
    indptr = np.arange(n + 1, dtype=np.int64) * m
    idx = np.tile(np.arange(m, dtype=np.int32), n)
    C = reg_dense(*oracle.reg(m, indptr, idx), n)
    np.testing.assert_array_equal(C, m * (np.ones((n, n), dtype=np.int64) - np.eye(n, dtype=np.int64)))


def test_reg_closed_form_disjoint_stars_and_identity():
    # disjoint stars: outputs 0..3 share source 0, outputs 4..6 share source 1 -> block diagonal
    indptr = np.arange(8, dtype=np.int64)
    idx = np.array([0, 0, 0, 0, 1, 1, 1], dtype=np.int32)
    C = reg_dense(*oracle.reg(2, indptr, idx), 7)
    want = np.zeros((7, 7), dtype=np.int64)
    want[:4, :4] = 1
    want[4:, 4:] = 1
    np.fill_diagonal(want, 0)
    np.testing.assert_array_equal(C, want)
    # identity block: no sharing -> empty REG with all rows present
    rp, col, w = oracle.reg(5, np.arange(6, dtype=np.int64), np.arange(5, dtype=np.int32))
    np.testing.assert_array_equal(rp, np.zeros(6, dtype=np.int64))
    assert len(col) == 0


def test_reg_empty_rows_and_empty_block():
    rp, col, w = oracle.reg(3, np.zeros(4, dtype=np.int64), np.zeros(0, dtype=np.int32))
    assert list(rp) == [0, 0, 0, 0] and len(col) == 0


def test_reg_golden_g1():
    g = load_golden("g1.json")
    import synth
    rows = [{int(k): v for k, v in g["rows"][str(l)].items()} for l in (0, 1)]
    full = synth.blocks_from_rows(g["seeds"], rows)
    rp, col, w = oracle.reg(full[1].n_src, full[1].indptr, full[1].nbr_pos)
    assert list(rp) == g["reg"]["indptr"] and list(col) == g["reg"]["col"] and list(w) == g["reg"]["w"]


@pytest.mark.parametrize("seed", [1, 2])
def test_reg_invariants_on_sampled_block(seed):
    """Invariants on a real sampled output block: symmetric, zero diagonal,
    row sums = sum_{u in S_i} (d_u - 1), total = sum_u d_u (d_u - 1),
    c_ij <= min(|S_i|, |S_j|)."""
    g, sd, blocks, feats, labels = tiny(n=400, pairs=1600, fanouts=(5, 6), n_out=80, seed=seed)
    b = blocks[-1]
    rp, col, w = oracle.reg(b.n_src, b.indptr, b.nbr_pos)
    n = b.n_dst
    C = reg_dense(rp, col, w, n)
    assert (C == C.T).all()
    assert (np.diag(C) == 0).all()
    assert (w >= 1).all()
    for i in range(n):
        assert (np.diff(col[rp[i]:rp[i + 1]]) > 0).all()
    d = np.bincount(b.nbr_pos, minlength=b.n_src)
    rowsum = np.array([sum(d[u] - 1 for u in b.nbr_pos[b.indptr[i]:b.indptr[i + 1]]) for i in range(n)])
    np.testing.assert_array_equal(C.sum(1), rowsum)
    assert C.sum() == int((d * (d - 1)).sum())
    sizes = np.diff(b.indptr)
    assert (C <= np.minimum.outer(sizes, sizes)).all()
