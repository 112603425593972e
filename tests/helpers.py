"""Shared test helpers: tiny seeded inputs and brute-force references.

Nothing here implements Betty's arithmetic in a way the oracle uses; the
brute-force functions are independent re-derivations (sets, dense matrices)
used to pin the oracle."""
from __future__ import annotations

import json
import os
from typing import Dict, List, Sequence

import numpy as np

import synth

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load_golden(name: str) -> dict:
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def tiny(n=60, pairs=150, fanouts=(3, 4), n_out=12, F=5, C=3, n_comm=3, mu=0.3, seed=1, ld=None):
    """A small seeded dataset with the same structure as the presets."""
    g = synth.graph(n, pairs, n_comm, mu, 0.4, seed)
    sd = synth.seeds(g.n, n_out, seed + 10)
    blocks = synth.sample(g, sd, fanouts, seed + 20)
    ld = ld or F
    feats = synth.features(g.comm, F, ld, 0, seed=seed + 30)
    labels = (np.arange(n) * 7 % C).astype(np.int32)
    return g, sd, blocks, feats, labels


def rows_by_gid(blocks) -> List[Dict[int, List[int]]]:
    """Per layer: dst gid -> list of neighbour gids (from full-batch blocks)."""
    out = []
    for l, b in enumerate(blocks):
        if l == len(blocks) - 1:
            dst_gid = b.src_gid[:b.n_dst]
        else:
            dst_gid = blocks[l].src_gid[:b.n_dst]
        rows = {}
        for i in range(b.n_dst):
            rows[int(dst_gid[i])] = [int(b.src_gid[p]) for p in b.nbr_pos[b.indptr[i]:b.indptr[i + 1]]]
        out.append(rows)
    return out


def closure(blocks, out_gids: Sequence[int]):
    """Brute force k-hop closure: per layer (dst set, src set, edge set) of
    the computation tree of out_gids, by set operations on gid rows."""
    rows = rows_by_gid(blocks)
    L = len(blocks)
    dst = set(int(x) for x in out_gids)
    res = [None] * L
    for l in range(L - 1, -1, -1):
        edges = {(u, v) for v in dst for u in rows[l][v]}
        src = dst | {u for (u, v) in edges}
        res[l] = (dst, src, edges)
        dst = src
    return res


def dense_P(b) -> np.ndarray:
    P = np.zeros((b.n_dst, b.n_src))
    idx = getattr(b, "indices", None)
    if idx is None:
        idx = b.nbr_pos
    for i in range(b.n_dst):
        for e in range(b.indptr[i], b.indptr[i + 1]):
            P[i, idx[e]] = 1.0
    return P


def split_params(params, dims, aggr):
    """Flat parameter vector -> per layer dict of float64 matrices."""
    out, o = [], 0
    for l in range(len(dims) - 1):
        fi, fo = dims[l], dims[l + 1]
        d = {}
        if aggr == "pool":
            d["Wp"] = params[o:o + fi * fi].reshape(fi, fi).astype(np.float64); o += fi * fi
            d["bp"] = params[o:o + fi].astype(np.float64); o += fi
        d["Ws"] = params[o:o + fi * fo].reshape(fi, fo).astype(np.float64); o += fi * fo
        d["Wn"] = params[o:o + fi * fo].reshape(fi, fo).astype(np.float64); o += fi * fo
        d["b"] = params[o:o + fo].astype(np.float64); o += fo
        out.append(d)
    assert o == len(params)
    return out


def rel_err(x, ref):
    x = np.asarray(x, dtype=np.float64).ravel()
    ref = np.asarray(ref, dtype=np.float64).ravel()
    nr = np.linalg.norm(ref)
    return np.linalg.norm(x - ref) / (nr if nr > 0 else 1.0)


def assert_close(x, ref, rtol, name=""):
    """DESIGN.md §3 reading #18: ||x-ref||/||ref|| <= rtol and
    max|x-ref| <= 10 rtol max|ref|."""
    x = np.asarray(x, dtype=np.float64).ravel()
    ref = np.asarray(ref, dtype=np.float64).ravel()
    assert x.shape == ref.shape, (name, x.shape, ref.shape)
    re = rel_err(x, ref)
    mx = float(np.max(np.abs(ref))) if ref.size else 0.0
    ma = float(np.max(np.abs(x - ref))) if ref.size else 0.0
    assert np.all(np.isfinite(x)), f"{name}: non-finite values"
    assert re <= rtol, f"{name}: rel l2 err {re:.3e} > {rtol:.1e}"
    assert ma <= 10 * rtol * mx + 1e-300, f"{name}: max abs err {ma:.3e} > 10*rtol*max|ref| = {10 * rtol * mx:.3e}"


def param_tensors(flat, dims, aggr):
    """Flat gradient -> [(name, array)] per layer and tensor (W_pool, b_pool,
    W_self, W_neigh, b), the flat layout of synth.init_params."""
    out = []
    for l, d in enumerate(split_params(np.asarray(flat, dtype=np.float64), dims, aggr)):
        for name, a in d.items():
            out.append((f"{name}{l}", a))
    return out


def assert_grad_close(x, ref, dims, aggr, rtol, name=""):
    """Reading #18 applied PER PARAMETER TENSOR (not to the flat vector, where
    a small tensor such as a bias could hide a large relative error)."""
    for (tn, a), (_, b) in zip(param_tensors(x, dims, aggr), param_tensors(ref, dims, aggr)):
        assert_close(a, b, rtol, f"{name} {tn}")


def explain_relu_flips(gpu, ref, ties, mb, feats, dims, aggr, rtol, name=""):
    """Reading #24: compare a gradient whose hidden ReLU decisions may legitimately differ.

    Where |S| <= tau * M (oracle.sage_ties), fp32 evaluation can take the ReLU decision either way:
    both gradients are correct.  A decision on H_1 (layer 0's output) at (v, j) gates dS_0[v, j] = g,
    and flipping it changes only layer 0's gradient, by d * g * (x_v (x) e_j, A_v (x) e_j, e_j) for
    (W_self, W_neigh, b) (d = +1 if the oracle's S <= 0, else -1; x_v the dst row's input, A_v its
    aggregated neighbours, the same rank-1 form for either SAGEConv form of mean/sum).  Per output
    column the flips are fitted by least squares and rounded to {0, 1}; the residual must then pass
    the per-tensor bound of reading #18 and every flip must be one of the oracle's candidates.
    Returns the number of flips explained."""
    assert aggr in ("mean", "sum")
    gpu = np.asarray(gpu, np.float64)
    ref = np.asarray(ref, np.float64)
    lev = ties["level"]
    assert (lev == 1).all() or len(lev) == 0 or len(dims) == 2, "flip explanation covers decisions on H_1"
    sel = lev == 1
    tv, tj, tS, tg = ties["v"][sel], ties["j"][sel], ties["S"][sel], ties["g"][sel]
    F, Fo = dims[0], dims[1]
    b0 = mb[0]
    X = feats[b0.src_gid, :F].astype(np.float64)
    delta = gpu - ref
    W = split_params(delta, dims, aggr)
    dWs, dWn, db = W[0]["Ws"].copy(), W[0]["Wn"].copy(), W[0]["b"].copy()
    flips = 0
    for j in np.unique(tj):
        idx = np.nonzero(tj == j)[0]
        cols = []
        for i in idx:
            v = int(tv[i])
            nb = (b0.indices if hasattr(b0, "indices") else b0.nbr_pos)[b0.indptr[v]:b0.indptr[v + 1]]
            Av = X[nb].sum(0) if len(nb) else np.zeros(F)
            if aggr == "mean" and len(nb):
                Av = Av / len(nb)
            d = 1.0 if tS[i] <= 0 else -1.0
            cols.append(d * tg[i] * np.concatenate([X[v], Av, [1.0]]))
        Amat = np.stack(cols, 1)
        rhs = np.concatenate([dWs[:, j], dWn[:, j], [db[j]]])
        c, *_ = np.linalg.lstsq(Amat, rhs, rcond=None)
        c = np.clip(np.rint(c), 0, 1)
        fix = Amat @ c
        dWs[:, j] -= fix[:F]
        dWn[:, j] -= fix[F:2 * F]
        db[j] -= fix[2 * F]
        flips += int(c.sum())
    R = split_params(ref, dims, aggr)
    for tn, d, r in (("Ws0", dWs, R[0]["Ws"]), ("Wn0", dWn, R[0]["Wn"]), ("b0", db, R[0]["b"])):
        assert_close(r + d, r, rtol, f"{name} {tn} (after {flips} explained ReLU flips)")
    for (tn, a), (_, b) in list(zip(param_tensors(gpu, dims, aggr), param_tensors(ref, dims, aggr)))[3:]:
        assert_close(a, b, rtol, f"{name} {tn}")
    return flips
