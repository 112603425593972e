"""Pins of the oracle's ReLU-decision report (oracle.sage_ties, reading #24) and of the flip-aware
gradient comparison (tests/helpers.explain_relu_flips) used by the full-size fp32 parity tests.

A hidden ReLU decision at |S| <= tau * M (M = sum of the magnitudes of the terms of S) can be taken
either way by a finite-precision evaluation; both resulting gradients are correct.  The report is
checked against an independent dense re-derivation (S, M and the gated gradient g), and the
comparison is checked to explain a planted flip and to reject a gradient that no flip explains."""
import numpy as np
import pytest

import oracle
import synth
from tests.helpers import dense_P, explain_relu_flips, split_params, tiny

DIMS = [6, 9, 4]


def case(seed=1):
    g, sd, blocks, feats, _ = tiny(n=150, pairs=600, fanouts=(3, 4), n_out=16, F=DIMS[0], C=DIMS[-1], seed=seed)
    labels = (np.arange(150) * 5 % DIMS[-1]).astype(np.int32)
    params = synth.init_params(DIMS, "mean", seed=seed).astype(np.float64)
    return sd, blocks, feats, labels, params


def dense_internals(blocks, feats, labels, params, scale):
    """2-layer SAGE-mean (aggregate-first layer 0, project-first or not layer 1 is irrelevant for
    the values): S_1 (layer 0's pre-activation), M_1 (sum of the term magnitudes) and the gradient
    dX_1 of H_1 before the ReLU mask."""
    W = split_params(params, DIMS, "mean")
    b0, b1 = blocks
    X = feats[b0.src_gid, :DIMS[0]].astype(np.float64)
    P0 = dense_P(b0)
    d0 = P0.sum(1, keepdims=True)
    A0 = np.divide(P0 @ X, d0, out=np.zeros((b0.n_dst, DIMS[0])), where=d0 > 0)
    Xd = X[:b0.n_dst]
    S1 = Xd @ W[0]["Ws"] + A0 @ W[0]["Wn"] + W[0]["b"]
    M1 = np.abs(Xd) @ np.abs(W[0]["Ws"]) + np.abs(A0) @ np.abs(W[0]["Wn"]) + np.abs(W[0]["b"])
    H1 = np.maximum(S1, 0.0)
    P1 = dense_P(b1)
    d1 = P1.sum(1, keepdims=True)
    D1 = np.divide(1.0, d1, out=np.zeros_like(d1), where=d1 > 0)
    S2 = H1[:b1.n_dst] @ W[1]["Ws"] + (D1 * (P1 @ H1)) @ W[1]["Wn"] + W[1]["b"]
    y = labels[b1.src_gid[:b1.n_dst]]
    m = S2.max(1, keepdims=True)
    p = np.exp(S2 - m)
    p /= p.sum(1, keepdims=True)
    dS2 = p
    dS2[np.arange(len(y)), y] -= 1.0
    dS2 *= scale
    dX1 = np.zeros_like(H1)
    dX1[:b1.n_dst] += dS2 @ W[1]["Ws"].T
    dX1 += P1.T @ (D1 * (dS2 @ W[1]["Wn"].T))
    return S1, M1, dX1, A0, Xd


def test_tie_report_matches_dense():
    sd, blocks, feats, labels, params = case()
    scale = 1.0 / len(sd)
    grad, loss, t, found = oracle.sage_ties(DIMS, "mean", False, blocks, params, feats, labels, scale, tau=1.0)
    S1, M1, dX1, _, _ = dense_internals(blocks, feats, labels, params, scale)
    assert found == S1.size and (t["level"] == 1).all()          # tau = 1: every decision reported
    np.testing.assert_array_equal(t["v"] * DIMS[1] + t["j"], np.arange(S1.size))
    np.testing.assert_allclose(t["S"], S1.ravel(), rtol=1e-12, atol=1e-14)
    np.testing.assert_allclose(t["M"], M1.ravel(), rtol=1e-12, atol=1e-14)
    np.testing.assert_allclose(t["g"], dX1.ravel(), rtol=1e-10, atol=1e-16)
    # the report does not change the gradient
    g2, l2, _ = oracle.sage(DIMS, "mean", False, blocks, params, feats, labels, scale)
    np.testing.assert_array_equal(grad, g2)
    # a tight tau reports exactly the decisions within it
    tau = 0.05
    _, _, t2, f2 = oracle.sage_ties(DIMS, "mean", False, blocks, params, feats, labels, scale, tau=tau)
    assert f2 == int((np.abs(S1) <= tau * M1).sum())


def test_flip_explanation_accepts_a_planted_flip_and_rejects_noise():
    sd, blocks, feats, labels, params = case(2)
    scale = 1.0 / len(sd)
    ref, _, t, _ = oracle.sage_ties(DIMS, "mean", False, blocks, params, feats, labels, scale, tau=1.0)
    S1, M1, dX1, A0, Xd = dense_internals(blocks, feats, labels, params, scale)
    # plant one flip: a decision with S > 0 taken as 0 by "the other evaluation"
    cand = np.nonzero((t["S"] > 0) & (np.abs(t["g"]) > 1e-3 * np.abs(t["g"]).max()))[0]
    i = int(cand[0])
    v, j = int(t["v"][i]), int(t["j"][i])
    gpu = ref.copy()
    F, Fo = DIMS[0], DIMS[1]
    # flat layout of layer 0: Ws (F x Fo), Wn (F x Fo), b (Fo)
    gpu[0:F * Fo].reshape(F, Fo)[:, j] -= t["g"][i] * Xd[v]
    gpu[F * Fo:2 * F * Fo].reshape(F, Fo)[:, j] -= t["g"][i] * A0[v]
    gpu[2 * F * Fo + j] -= t["g"][i]
    ties = {k: a[[i] + [int(x) for x in cand[1:4]]] for k, a in t.items()}
    mb = blocks
    assert explain_relu_flips(gpu, ref, ties, mb, feats, DIMS, "mean", 1e-9) == 1
    # the same error with the decision missing from the candidate list is not explained
    ties_wo = {k: a[[int(x) for x in cand[1:4]]] for k, a in t.items()}
    with pytest.raises(AssertionError):
        explain_relu_flips(gpu, ref, ties_wo, mb, feats, DIMS, "mean", 1e-9)
    # nor is noise on W_self
    noisy = ref.copy()
    noisy[0:F * Fo] *= 1.0 + 1e-3
    with pytest.raises(AssertionError):
        explain_relu_flips(noisy, ref, ties, mb, feats, DIMS, "mean", 1e-6)
