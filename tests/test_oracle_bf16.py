"""Pins of the oracle's bf16-GEMM mode (DESIGN.md §3 reading #17) and of the
pool aggregator's tie rule (reading #14).

The reference here is an independent dense re-derivation in numpy float64: no
oracle code, its own layer loop over dense P matrices, and its own bfloat16
rounding (integer carry on the float64 bits, pinned to torch's conversion).  It applies
the bf16 casts at exactly the points reading #17 names:
  * the feature table (H_0) and every parameter tensor (W_s, W_n, b, W_p, b_p)
    are GEMM operands -> bf16;
  * every other GEMM operand: the aggregated neighbour features A
    (aggregate-first, pool), dS, dA's producer dS, dZ (project-first), dZp;
  * the hidden activations H_{l+1} = ReLU(S) are stored in bf16;
  * DGL SAGEConv's rule (reading #11): W_n before the aggregation when
    F_in > F_out (project-first), where Z = X W_n is NOT rounded (it is not a
    GEMM operand: it is aggregated and added to S in fp32).
The bias is folded into the GEMM as a ones column, so b (and, in the backward,
dS in 1^T dS) are rounded like every other operand.
"""
import numpy as np
import pytest
import torch

import oracle
import synth
from tests.helpers import dense_P, split_params, tiny


def idx_of(b):
    """Local neighbour ids of a block (micro-batch MBlock or full-batch synth.Block)."""
    return b.indices if hasattr(b, "indices") else b.nbr_pos


def q(x):
    """RNE of float64 values to bfloat16's 8 significant bits, by integer arithmetic on the float64 bit
    pattern (the carry trick: add 2^44 - 1 + lsb, clear the low 45 mantissa bits).  A single rounding
    from float64: going through float32 first (torch's double -> bfloat16 conversion does) double-rounds
    values with more than 24 significant bits, which the sum aggregator's exact sums produce.  The
    helper is itself pinned to torch's float32 -> bfloat16 conversion below."""
    x = np.ascontiguousarray(x, dtype=np.float64)
    b = x.view(np.uint64)
    lsb = (b >> np.uint64(45)) & np.uint64(1)
    r = ((b + np.uint64((1 << 44) - 1) + lsb) >> np.uint64(45)) << np.uint64(45)
    return np.where(np.isfinite(x) & (x != 0), r.view(np.float64), x)


def test_q_equals_torch_bfloat16_on_float32_inputs():
    rng = np.random.default_rng(5)
    x = rng.standard_normal(20000).astype(np.float32)
    base = torch.tensor(x[:3000]).to(torch.bfloat16).float().numpy()
    ties = (base.view(np.uint32) | np.uint32(0x8000)).view(np.float32)       # exact bf16 ties
    x = np.concatenate([x, ties, np.float32([0.0, -0.0, 1.0, -3.0, 65504.0])])
    want = torch.tensor(x).to(torch.bfloat16).double().numpy()
    np.testing.assert_array_equal(q(x.astype(np.float64)), want)


def dense_step(blocks, dims, aggr, params, feats, labels, scale, bf16=True, tie="first"):
    """Dense forward + softmax-CE + backward of one (micro-)batch.
    Returns (flat gradient float64, loss, logits)."""
    r = q if bf16 else (lambda x: np.asarray(x, dtype=np.float64))
    W = split_params(np.asarray(params, dtype=np.float64), dims, aggr)
    L = len(blocks)
    X = r(feats[blocks[0].src_gid, :dims[0]].astype(np.float64))
    Hs, As, Zps, args, forms = [X], [], [], [], []
    for l, b in enumerate(blocks):
        P = dense_P(b)
        nd, ns = b.n_dst, b.n_src
        fi, fo = dims[l], dims[l + 1]
        Ws, Wn, bb = r(W[l]["Ws"]), r(W[l]["Wn"]), r(W[l]["b"])
        deg = P.sum(1, keepdims=True)
        Dinv = np.divide(1.0, deg, out=np.zeros_like(deg), where=deg > 0)
        Xd = X[:nd]
        S = r(Xd) @ Ws + bb[None, :]
        if aggr in ("mean", "sum"):
            norm = Dinv if aggr == "mean" else (deg > 0).astype(np.float64)
            pf = fi > fo
            forms.append(pf)
            if not pf:
                A = norm * (P @ X)
                S = S + r(A) @ Wn
            else:
                A = norm * (P @ (r(X) @ Wn))      # Z = X W_n: fp32 in the kernel, not rounded
                S = S + A
            As.append(A)
            Zps.append(None)
            args.append(None)
        else:
            forms.append(False)
            Zp = r(X) @ r(W[l]["Wp"]) + r(W[l]["bp"])[None, :]
            Z = np.maximum(Zp, 0.0)
            A = np.zeros((nd, fi))
            arg = -np.ones((nd, fi), dtype=np.int64)
            for v in range(nd):
                nb = np.asarray(idx_of(b)[b.indptr[v]:b.indptr[v + 1]], dtype=np.int64)
                if len(nb) == 0:
                    continue
                Zr = Z[nb]                                      # rows in canonical row order
                A[v] = Zr.max(0)
                hit = Zr == A[v][None, :]
                pos = hit.argmax(0) if tie == "first" else len(nb) - 1 - hit[::-1].argmax(0)
                arg[v] = nb[pos]
            S = S + r(A) @ Wn
            As.append(A)
            Zps.append(Zp)
            args.append(arg)
        if l < L - 1:
            X = r(np.maximum(S, 0.0))
            Hs.append(X)
    logits = S
    out_gid = blocks[-1].src_gid[:blocks[-1].n_dst]
    y = labels[out_gid]
    m = logits.max(1, keepdims=True)
    lse = (m + np.log(np.exp(logits - m).sum(1, keepdims=True)))[:, 0]
    loss = scale * float(np.sum(lse - logits[np.arange(len(y)), y]))
    dS = np.exp(logits - lse[:, None])
    dS[np.arange(len(y)), y] -= 1.0
    dS *= scale
    grads = [dict() for _ in range(L)]
    for l in range(L - 1, -1, -1):
        b = blocks[l]
        P = dense_P(b)
        nd, ns = b.n_dst, b.n_src
        fi, fo = dims[l], dims[l + 1]
        X = Hs[l]
        Ws, Wn = r(W[l]["Ws"]), r(W[l]["Wn"])
        deg = P.sum(1, keepdims=True)
        Dinv = np.divide(1.0, deg, out=np.zeros_like(deg), where=deg > 0)
        g = grads[l]
        g["Ws"] = r(X[:nd]).T @ r(dS)
        g["b"] = r(dS).sum(0)
        dX = np.zeros((ns, fi))
        dX[:nd] += r(dS) @ Ws.T
        if aggr in ("mean", "sum"):
            norm = Dinv if aggr == "mean" else (deg > 0).astype(np.float64)
            if not forms[l]:
                g["Wn"] = r(As[l]).T @ r(dS)
                dA = r(dS) @ Wn.T
                dX += P.T @ (norm * dA)
            else:
                dZ = P.T @ (norm * dS)
                g["Wn"] = r(X).T @ r(dZ)
                dX += r(dZ) @ Wn.T
        else:
            g["Wn"] = r(As[l]).T @ r(dS)
            dA = r(dS) @ Wn.T
            dZ = np.zeros((ns, fi))
            arg = args[l]
            for v in range(nd):
                for f in range(fi):
                    if arg[v, f] >= 0:
                        dZ[arg[v, f], f] += dA[v, f]
            dZp = dZ * (Zps[l] > 0)
            g["Wp"] = r(X).T @ r(dZp)
            g["bp"] = r(dZp).sum(0)
            dX += r(dZp) @ r(W[l]["Wp"]).T
        dS = dX * (X > 0) if l > 0 else None
    flat = []
    for l in range(L):
        for name in (["Wp", "bp"] if aggr == "pool" else []) + ["Ws", "Wn", "b"]:
            flat.append(np.asarray(grads[l][name]).ravel())
    return np.concatenate(flat), loss, logits


CASES = [
    dict(name="mean2-aggfirst", aggr="mean", fanouts=(3, 4), dims=[5, 7, 3]),
    dict(name="mean2-projfirst", aggr="mean", fanouts=(3, 4), dims=[9, 4, 3]),
    dict(name="mean3-mixed", aggr="mean", fanouts=(2, 3, 4), dims=[6, 8, 8, 3]),
    dict(name="mean3-wide", aggr="mean", fanouts=(3, 3, 4), dims=[12, 20, 6, 5]),
    dict(name="pool2", aggr="pool", fanouts=(3, 4), dims=[5, 6, 3]),
    dict(name="pool3", aggr="pool", fanouts=(2, 3, 3), dims=[4, 5, 5, 3]),
    dict(name="sum2-aggfirst", aggr="sum", fanouts=(3, 4), dims=[5, 7, 3]),
    dict(name="sum2-projfirst", aggr="sum", fanouts=(3, 4), dims=[9, 4, 3]),
]


def make(c, seed):
    g, sd, blocks, feats, _ = tiny(n=150, pairs=500, fanouts=c["fanouts"], n_out=16, F=c["dims"][0],
                                   C=c["dims"][-1], seed=seed)
    labels = (np.arange(150) * 5 % c["dims"][-1]).astype(np.int32)
    params = synth.init_params(c["dims"], c["aggr"], seed=seed).astype(np.float64)
    return sd, blocks, feats, labels, params


@pytest.mark.parametrize("seed", [1, 2])
@pytest.mark.parametrize("c", CASES, ids=lambda c: c["name"])
def test_bf16_mode_equals_dense_bf16_reference(c, seed):
    """oracle.sage(bf16=True) == the dense bf16-cast reference, 1e-12: the
    rounding points of reading #17 are pinned (dropping the H_{l+1} rounding,
    the bias rounding, or inverting the project-first rule fails here)."""
    sd, blocks, feats, labels, params = make(c, seed)
    scale = 1.0 / len(sd)
    g, l, lg = oracle.sage(c["dims"], c["aggr"], True, blocks, params, feats, labels, scale, want_logits=True)
    rg, rl, rlg = dense_step(blocks, c["dims"], c["aggr"], params, feats, labels, scale, bf16=True)
    np.testing.assert_allclose(lg, rlg, rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(g, rg, rtol=1e-10, atol=1e-14)
    assert l == pytest.approx(rl, rel=1e-12)
    # the reference itself is not degenerate: bf16 mode really differs from fp32 mode
    g32, _, lg32 = oracle.sage(c["dims"], c["aggr"], False, blocks, params, feats, labels, scale, want_logits=True)
    assert np.abs(lg32 - rlg).max() > 1e-6


@pytest.mark.parametrize("c", CASES, ids=lambda c: c["name"])
def test_fp32_mode_equals_dense_reference(c):
    """The same dense reference without rounding is the fp32 (float64) mode."""
    sd, blocks, feats, labels, params = make(c, 3)
    scale = 1.0 / len(sd)
    g, l, lg = oracle.sage(c["dims"], c["aggr"], False, blocks, params, feats, labels, scale, want_logits=True)
    rg, rl, rlg = dense_step(blocks, c["dims"], c["aggr"], params, feats, labels, scale, bf16=False)
    np.testing.assert_allclose(lg, rlg, rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(g, rg, rtol=1e-10, atol=1e-14)


def tie_case(seed=0, n_out=24):
    """One pool layer on integer data: features in {0,1,2}, W_p in {-1,0,1},
    b_p = 0 -> Z = ReLU(X W_p) is integer-valued and ties in the max are the
    common case; which neighbour is the argmax decides dW_p."""
    g, sd, blocks, feats, _ = tiny(n=80, pairs=400, fanouts=(6,), n_out=n_out, F=4, C=3, seed=seed)
    rng = np.random.default_rng(seed)
    feats = rng.integers(0, 3, size=feats.shape).astype(np.float32)
    dims = [4, 3]
    params = synth.init_params(dims, "pool", seed=seed).astype(np.float64)
    params[0:16] = rng.integers(-1, 2, size=16)
    params[16:20] = 0.0
    labels = (np.arange(80) % 3).astype(np.int32)
    return sd, blocks, feats, labels, params, dims


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_pool_tie_first_max_in_row_order(seed):
    """Reading #14: on a tie the FIRST neighbour in canonical row order is the
    argmax and receives the gradient.  The first- and last-max rules give
    different dW_p on these inputs, and the oracle matches the first."""
    sd, blocks, feats, labels, params, dims = tie_case(seed)
    scale = 1.0 / len(sd)
    g, _, _ = oracle.sage(dims, "pool", False, blocks, params, feats, labels, scale)
    first, _, _ = dense_step(blocks, dims, "pool", params, feats, labels, scale, bf16=False, tie="first")
    last, _, _ = dense_step(blocks, dims, "pool", params, feats, labels, scale, bf16=False, tie="last")
    assert np.abs(first - last).max() > 1e-3          # the tie rule matters on this input
    np.testing.assert_allclose(g, first, rtol=1e-12, atol=1e-15)
