"""Pins of the oracle's SAGE forward/backward, loss and gradient accumulation:
dense-matrix forward (numpy), textbook reductions, central finite differences,
the two SAGEConv forms, bf16 rounding against torch, and Betty's defining
invariant sum_k g_k = g_full."""
import numpy as np
import pytest
import torch
from scipy.special import logsumexp

import oracle
import synth
from tests.helpers import assert_close, dense_P, split_params, tiny


def dense_forward(blocks, dims, aggr, params, feats, src_gid0):
    """Independent dense forward: per layer S = X_d Ws + A Wn + b with
    A = D^-1 P X (mean) or masked max of ReLU(X Wp + bp) (pool)."""
    W = split_params(params, dims, aggr)
    X = feats[src_gid0, :dims[0]].astype(np.float64)
    L = len(blocks)
    for l, b in enumerate(blocks):
        P = dense_P(b)
        nd = b.n_dst
        if aggr == "mean":
            deg = P.sum(1, keepdims=True)
            A = np.divide(P @ X, deg, out=np.zeros((nd, X.shape[1])), where=deg > 0)
        elif aggr == "sum":                      # Table 1 "Sum": no 1/D
            A = P @ X
        else:
            Z = np.maximum(X @ W[l]["Wp"] + W[l]["bp"], 0.0)
            A = np.zeros((nd, X.shape[1]))
            for v in range(nd):
                nb = np.nonzero(P[v])[0]
                if len(nb):
                    A[v] = Z[nb].max(0)
        S = X[:nd] @ W[l]["Ws"] + A @ W[l]["Wn"] + W[l]["b"]
        X = np.maximum(S, 0.0) if l < L - 1 else S
    return X


CASES = [
    dict(name="mean2", aggr="mean", fanouts=(3, 4), dims=[5, 7, 3]),
    dict(name="mean3-projfirst", aggr="mean", fanouts=(2, 3, 4), dims=[6, 8, 8, 3]),
    dict(name="mean2-projfirst", aggr="mean", fanouts=(3, 4), dims=[9, 4, 3]),
    dict(name="pool2", aggr="pool", fanouts=(3, 4), dims=[5, 6, 3]),
    dict(name="pool3", aggr="pool", fanouts=(2, 3, 3), dims=[4, 5, 5, 3]),
    dict(name="sum2", aggr="sum", fanouts=(3, 4), dims=[5, 7, 3]),
    dict(name="sum3-projfirst", aggr="sum", fanouts=(2, 3, 4), dims=[6, 8, 4, 3]),
]


def make_case(c, seed=1, n=120, pairs=400, n_out=14):
    g, sd, blocks, feats, _ = tiny(n=n, pairs=pairs, fanouts=c["fanouts"], n_out=n_out, F=c["dims"][0],
                                   C=c["dims"][-1], seed=seed)
    labels = (np.arange(n) * 5 % c["dims"][-1]).astype(np.int32)
    params = synth.init_params(c["dims"], c["aggr"], seed=seed).astype(np.float64)
    return g, sd, blocks, feats, labels, params


@pytest.mark.parametrize("c", CASES, ids=lambda c: c["name"])
def test_forward_matches_dense(c):
    g, sd, blocks, feats, labels, params = make_case(c)
    _, loss, logits = oracle.sage(c["dims"], c["aggr"], False, blocks, params, feats, labels, 1.0 / len(sd),
                                  want_logits=True)
    ref = dense_forward(blocks, c["dims"], c["aggr"], params, feats, blocks[0].src_gid)
    np.testing.assert_allclose(logits, ref, rtol=1e-12, atol=1e-12)
    # loss = mean softmax cross-entropy over the batch's outputs (reading #15)
    y = labels[blocks[-1].src_gid[:blocks[-1].n_dst]]
    want = np.mean(logsumexp(ref, axis=1) - ref[np.arange(len(y)), y])
    assert loss == pytest.approx(want, rel=1e-12)


def test_mean_all_equal_rows_and_pool_identity_reduction():
    """mean of identical neighbour rows = that row; pool with W_p = I, b_p = 0
    and H >= 0 is the column-wise max over neighbours (Table 1)."""
    c = dict(aggr="pool", fanouts=(4,), dims=[4, 4])
    g, sd, blocks, feats, labels, params = make_case(c, n_out=10)
    feats = np.abs(feats)
    W = split_params(params, c["dims"], "pool")
    P = params.copy()
    # layer params: Wp(16) bp(4) Ws(16) Wn(16) b(4)
    P[0:16] = np.eye(4).ravel(); P[16:20] = 0.0
    P[20:36] = 0.0; P[36:52] = np.eye(4).ravel(); P[52:56] = 0.0
    _, _, logits = oracle.sage(c["dims"], "pool", False, blocks, P, feats, labels, 1.0, want_logits=True)
    b = blocks[0]
    X = feats[b.src_gid, :4].astype(np.float64)
    for v in range(b.n_dst):
        nb = b.nbr_pos[b.indptr[v]:b.indptr[v + 1]]
        want = X[nb].max(0) if len(nb) else np.zeros(4)
        np.testing.assert_array_equal(logits[v], want)
    # mean over identical rows
    feats2 = np.tile(np.array([[1.5, -2.0, 0.25, 3.0]], np.float32), (len(feats), 1))
    Pm = np.zeros(4 * 4 * 2 + 4)
    Pm[16:32] = np.eye(4).ravel()                 # W_neigh = I, W_self = 0, b = 0
    _, _, lg = oracle.sage([4, 4], "mean", False, blocks, Pm, feats2, labels, 1.0, want_logits=True)
    deg = np.diff(b.indptr)
    np.testing.assert_array_equal(lg[deg > 0], np.tile(feats2[:1].astype(np.float64), ((deg > 0).sum(), 1)))
    assert (lg[deg == 0] == 0).all()


@pytest.mark.parametrize("c", [c for c in CASES if c["aggr"] != "pool"], ids=lambda c: c["name"])
def test_two_sageconv_forms_agree(c):
    g, sd, blocks, feats, labels, params = make_case(c)
    a = oracle.sage(c["dims"], c["aggr"], False, blocks, params, feats, labels, 0.1, force_form=0, want_logits=True)
    b = oracle.sage(c["dims"], c["aggr"], False, blocks, params, feats, labels, 0.1, force_form=1, want_logits=True)
    np.testing.assert_allclose(a[2], b[2], rtol=1e-12, atol=1e-13)
    np.testing.assert_allclose(a[0], b[0], rtol=1e-10, atol=1e-13)
    assert a[1] == pytest.approx(b[1], rel=1e-13)


@pytest.mark.parametrize("c", CASES, ids=lambda c: c["name"])
def test_backward_finite_differences(c):
    """Central differences of the loss (eps = 1e-6) against the closed-form
    gradient for a random sample of parameters."""
    g, sd, blocks, feats, labels, params = make_case(c, seed=3)
    scale = 1.0 / len(sd)
    grad, loss, _ = oracle.sage(c["dims"], c["aggr"], False, blocks, params, feats, labels, scale)
    rng = np.random.default_rng(0)
    idx = rng.choice(len(params), size=min(120, len(params)), replace=False)
    eps = 1e-6
    fd = np.empty(len(idx))
    for t, i in enumerate(idx):
        p1 = params.copy(); p1[i] += eps
        p2 = params.copy(); p2[i] -= eps
        l1 = oracle.sage(c["dims"], c["aggr"], False, blocks, p1, feats, labels, scale)[1]
        l2 = oracle.sage(c["dims"], c["aggr"], False, blocks, p2, feats, labels, scale)[1]
        fd[t] = (l1 - l2) / (2 * eps)
    assert np.abs(grad).max() > 0
    assert_close(grad[idx], fd, 1e-6, "grad vs FD")


@pytest.mark.parametrize("c", CASES, ids=lambda c: c["name"])
@pytest.mark.parametrize("K", [2, 3, 14])
def test_sum_of_micro_batch_gradients_equals_full_batch(c, K):
    """Betty's invariant: sum_k g_k == g_full (float64)."""
    g, sd, blocks, feats, labels, params = make_case(c, seed=5)
    scale = 1.0 / len(sd)
    g_full, l_full, _ = oracle.sage(c["dims"], c["aggr"], False, blocks, params, feats, labels, scale)
    part = synth.random_partition(len(sd), K, seed=K)
    acc = np.zeros_like(g_full)
    lacc = 0.0
    for k in range(K):
        mb = oracle.extract(blocks, part, K, k)
        if mb[-1].n_dst == 0:
            continue
        gk, lk, _ = oracle.sage(c["dims"], c["aggr"], False, mb, params, feats, labels, scale)
        acc += gk
        lacc += lk
    assert np.linalg.norm(acc - g_full) <= 1e-12 * np.linalg.norm(g_full)
    assert lacc == pytest.approx(l_full, rel=1e-12)
    # oracle_step does the same loop
    gs, ls = oracle.step(c["dims"], c["aggr"], False, blocks, part, K, list(range(K)), params, feats, labels, scale)
    np.testing.assert_allclose(gs, acc, rtol=1e-13, atol=1e-16)
    assert ls == pytest.approx(lacc, rel=1e-13)


def test_bf16_round_matches_torch():
    """The oracle's RNE bf16 rounding agrees with torch's float32->bfloat16
    conversion (a library routine), including exact ties."""
    rng = np.random.default_rng(0)
    x = np.concatenate([rng.standard_normal(2000).astype(np.float32),
                        (rng.standard_normal(200) * 1e-30).astype(np.float32),
                        (rng.standard_normal(200) * 1e30).astype(np.float32)])
    # exact ties: bf16 value + half an ulp
    base = torch.tensor(rng.standard_normal(300).astype(np.float32)).to(torch.bfloat16).float().numpy()
    ties = (base.view(np.uint32) | np.uint32(0x8000)).view(np.float32)
    x = np.concatenate([x, ties, np.float32([0.0, -0.0, 1.0, -3.0])])
    want = torch.tensor(x).to(torch.bfloat16).double().numpy()
    got = np.array([oracle.bf16_round(float(v)) for v in x])
    np.testing.assert_array_equal(got, want)


@pytest.mark.parametrize("c", CASES, ids=lambda c: c["name"])
def test_bf16_mode_is_close_to_fp32_mode(c):
    g, sd, blocks, feats, labels, params = make_case(c, seed=2)
    a = oracle.sage(c["dims"], c["aggr"], False, blocks, params, feats, labels, 0.1, want_logits=True)
    b = oracle.sage(c["dims"], c["aggr"], True, blocks, params, feats, labels, 0.1, want_logits=True)
    e_log = np.linalg.norm(a[2] - b[2]) / np.linalg.norm(a[2])
    e_grad = np.linalg.norm(a[0] - b[0]) / np.linalg.norm(a[0])
    assert 0 < e_log < 3e-2 and 0 < e_grad < 5e-2, (e_log, e_grad)


def test_sum_is_degree_times_mean():
    """Table 1: the sum aggregator equals D_v times the mean (one layer, W_self = 0, b = 0, W_neigh = I:
    the logits are the aggregated rows themselves)."""
    c = dict(aggr="sum", fanouts=(4,), dims=[4, 4])
    g, sd, blocks, feats, labels, params = make_case(c, n_out=12)
    P = np.zeros(4 * 4 * 2 + 4)
    P[16:32] = np.eye(4).ravel()                 # W_neigh = I, W_self = 0, b = 0
    _, _, ls = oracle.sage([4, 4], "sum", False, blocks, P, feats, labels, 1.0, want_logits=True)
    _, _, lm = oracle.sage([4, 4], "mean", False, blocks, P, feats, labels, 1.0, want_logits=True)
    deg = np.diff(blocks[0].indptr).astype(np.float64)[:, None]
    np.testing.assert_allclose(ls, deg * lm, rtol=1e-13, atol=1e-13)
    assert (deg > 1).any()
