"""CPU oracle for Betty's micro-batch training hot path -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_asplos_yangzd023_b200``) never imports it and shares no code with
it; the only common dependency is the input generator ``synth`` (no method
arithmetic).

The arithmetic lives in ``oracle.c`` (plain C, float64); this module only
marshals numpy arrays through ctypes.  See the header of ``oracle.c`` for the
paper passages each function follows, and DESIGN.md §3 for the readings.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass
from typing import List, Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        # no -ffast-math: the oracle must keep IEEE float64 semantics
        subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


class OBlock(ctypes.Structure):
    _fields_ = [("n_dst", ctypes.c_int64), ("n_src", ctypes.c_int64), ("n_edges", ctypes.c_int64),
                ("indptr", ctypes.c_void_p), ("indices", ctypes.c_void_p), ("src_pos", ctypes.c_void_p),
                ("src_gid", ctypes.c_void_p), ("t_indptr", ctypes.c_void_p), ("t_indices", ctypes.c_void_p)]


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        P, i64, i32, dbl = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_double
        L.oracle_reg.restype = i64
        L.oracle_reg.argtypes = [i64, i64, P, P, ctypes.POINTER(P), ctypes.POINTER(P), ctypes.POINTER(P)]
        L.oracle_extract.restype = ctypes.c_int
        L.oracle_extract.argtypes = [ctypes.c_int, P, P, i64, i32, i32, P]
        L.oracle_sage.restype = ctypes.c_int
        L.oracle_sage.argtypes = [ctypes.c_int, P, ctypes.c_int, ctypes.c_int, ctypes.c_int, P, P, P, i64, P, dbl,
                                  P, ctypes.POINTER(dbl), P]
        L.oracle_step.restype = ctypes.c_int
        L.oracle_step.argtypes = [ctypes.c_int, P, ctypes.c_int, ctypes.c_int, P, P, i64, i32, P, i32, P, P, i64,
                                  P, dbl, P, ctypes.POINTER(dbl)]
        L.oracle_sage_ties.restype = i64
        L.oracle_sage_ties.argtypes = [ctypes.c_int, P, ctypes.c_int, ctypes.c_int, P, P, P, i64, P, dbl, P,
                                       ctypes.POINTER(dbl), dbl, i64, P, P, P, P, P, P]
        L.oracle_mem_estimate.restype = ctypes.c_int
        L.oracle_mem_estimate.argtypes = [ctypes.c_int, P, ctypes.c_int, P, P, P, P]
        L.oracle_bf16_round.restype = dbl
        L.oracle_bf16_round.argtypes = [dbl]
        L.oracle_free.restype = None
        L.oracle_free.argtypes = [P]
        L.oracle_block_free.restype = None
        L.oracle_block_free.argtypes = [P, ctypes.c_int]
        _lib = L
    return _lib


def _aggr(aggr: str) -> int:
    """aggregator code of oracle.c: 0 mean, 1 pool (Table 1)"""
    return {"mean": 0, "pool": 1, "sum": 2}[aggr]


def _p(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data


def _take(addr: int, n: int, dtype) -> np.ndarray:
    if n == 0 or not addr:
        out = np.zeros(n, dtype=dtype)
    else:
        buf = (ctypes.c_char * (n * np.dtype(dtype).itemsize)).from_address(addr)
        out = np.frombuffer(buf, dtype=dtype).copy()
    return out


@dataclass
class MBlock:
    """A micro-batch block as the oracle returns it (all numpy, host)."""
    n_dst: int
    n_src: int
    indptr: np.ndarray       # int64 [n_dst+1]
    indices: np.ndarray      # int32 [E] local src ids
    src_pos: np.ndarray      # int32 [n_src] full-batch src positions
    src_gid: np.ndarray      # int32 [n_src]
    t_indptr: np.ndarray     # int64 [n_src+1]
    t_indices: np.ndarray    # int32 [E]

    @property
    def n_edges(self) -> int:
        return int(self.indptr[-1])


def _oblocks(blocks) -> tuple:
    """Marshal full-batch (synth.Block) or micro-batch (MBlock) blocks."""
    L = len(blocks)
    arr = (OBlock * L)()
    keep = []
    for l, b in enumerate(blocks):
        ip = np.ascontiguousarray(b.indptr, dtype=np.int64)
        ix = np.ascontiguousarray(getattr(b, "indices", None) if hasattr(b, "indices") else b.nbr_pos,
                                  dtype=np.int32)
        sg = np.ascontiguousarray(b.src_gid, dtype=np.int32)
        keep += [ip, ix, sg]
        arr[l].n_dst, arr[l].n_src, arr[l].n_edges = b.n_dst, b.n_src, int(ip[-1])
        arr[l].indptr, arr[l].indices, arr[l].src_gid = _p(ip), _p(ix), _p(sg)
    return arr, keep


def bf16_round(x: float) -> float:
    return lib().oracle_bf16_round(float(x))


def reg(n_src: int, indptr: np.ndarray, idx: np.ndarray):
    """REG of the output block: (indptr int64 [n_out+1], col int32, w int32)."""
    indptr = np.ascontiguousarray(indptr, dtype=np.int64)
    idx = np.ascontiguousarray(idx, dtype=np.int32)
    n_out = len(indptr) - 1
    rp, col, w = ctypes.c_void_p(), ctypes.c_void_p(), ctypes.c_void_p()
    nnz = lib().oracle_reg(n_out, n_src, _p(indptr), _p(idx), ctypes.byref(rp), ctypes.byref(col), ctypes.byref(w))
    out = (_take(rp.value, n_out + 1, np.int64), _take(col.value, nnz, np.int32), _take(w.value, nnz, np.int32))
    for p in (rp, col, w):
        lib().oracle_free(p.value)
    return out


def extract(full: Sequence, part: np.ndarray, K: int, k: int) -> List[MBlock]:
    L = len(full)
    arr, keep = _oblocks(full)
    part = np.ascontiguousarray(part, dtype=np.int32)
    out = (OBlock * L)()
    rc = lib().oracle_extract(L, ctypes.addressof(arr), _p(part), full[L - 1].n_dst, K, k, ctypes.addressof(out))
    if rc != 0:
        raise ValueError("oracle_extract: invalid input")
    res = []
    for l in range(L):
        o = out[l]
        E = o.n_edges
        res.append(MBlock(o.n_dst, o.n_src, _take(o.indptr, o.n_dst + 1, np.int64), _take(o.indices, E, np.int32),
                          _take(o.src_pos, o.n_src, np.int32), _take(o.src_gid, o.n_src, np.int32),
                          _take(o.t_indptr, o.n_src + 1, np.int64), _take(o.t_indices, E, np.int32)))
    lib().oracle_block_free(ctypes.addressof(out), L)
    return res


def sage(dims: Sequence[int], aggr: str, bf16: bool, blocks: Sequence, params: np.ndarray, feats: np.ndarray,
         labels: np.ndarray, loss_scale: float, force_form: int = -1, want_logits: bool = False):
    """Forward + loss + backward of one micro-batch (or the full batch).
    Returns (grad float64 [P], loss float, logits float64 or None)."""
    L = len(blocks)
    arr, keep = _oblocks(blocks)
    d = np.ascontiguousarray(dims, dtype=np.int32)
    params = np.ascontiguousarray(params, dtype=np.float64)
    feats = np.ascontiguousarray(feats, dtype=np.float32)
    labels = np.ascontiguousarray(labels, dtype=np.int32)
    grad = np.zeros(len(params), dtype=np.float64)
    loss = ctypes.c_double(0.0)
    logits = np.zeros((blocks[-1].n_dst, dims[-1]), dtype=np.float64) if want_logits else None
    lib().oracle_sage(L, _p(d), _aggr(aggr), int(bf16), force_form, ctypes.addressof(arr),
                      _p(params), _p(feats), feats.shape[1], _p(labels), loss_scale, _p(grad), ctypes.byref(loss),
                      _p(logits))
    return grad, loss.value, logits


def sage_ties(dims: Sequence[int], aggr: str, bf16: bool, blocks: Sequence, params: np.ndarray, feats: np.ndarray,
              labels: np.ndarray, loss_scale: float, tau: float, cap: int = 1 << 20):
    """oracle_sage plus the hidden ReLU decisions finite precision may take either way (reading #24):
    every (level, v, j) with |S| <= tau * M (M = sum of the magnitudes of S's terms), with S, M and
    the gradient g the decision gates.  Returns (grad, loss, ties dict of arrays, found)."""
    L = len(blocks)
    arr, keep = _oblocks(blocks)
    d = np.ascontiguousarray(dims, dtype=np.int32)
    params = np.ascontiguousarray(params, dtype=np.float64)
    feats = np.ascontiguousarray(feats, dtype=np.float32)
    labels = np.ascontiguousarray(labels, dtype=np.int32)
    grad = np.zeros(len(params), dtype=np.float64)
    loss = ctypes.c_double(0.0)
    t = {"level": np.zeros(cap, np.int32), "v": np.zeros(cap, np.int64), "j": np.zeros(cap, np.int32),
         "S": np.zeros(cap), "M": np.zeros(cap), "g": np.zeros(cap)}
    found = lib().oracle_sage_ties(L, _p(d), _aggr(aggr), int(bf16), ctypes.addressof(arr),
                                   _p(params), _p(feats), feats.shape[1], _p(labels), loss_scale, _p(grad),
                                   ctypes.byref(loss), tau, cap, _p(t["level"]), _p(t["v"]), _p(t["j"]), _p(t["S"]),
                                   _p(t["M"]), _p(t["g"]))
    n = min(found, cap)
    return grad, loss.value, {k: a[:n] for k, a in t.items()}, found


def step(dims: Sequence[int], aggr: str, bf16: bool, full: Sequence, part: np.ndarray, K: int,
         ks: Sequence[int], params: np.ndarray, feats: np.ndarray, labels: np.ndarray, loss_scale: float):
    """One batch: micro-batches ks of the K-way partition; returns (grad, loss)."""
    L = len(full)
    arr, keep = _oblocks(full)
    d = np.ascontiguousarray(dims, dtype=np.int32)
    part = np.ascontiguousarray(part, dtype=np.int32)
    ks = np.ascontiguousarray(ks, dtype=np.int32)
    params = np.ascontiguousarray(params, dtype=np.float64)
    feats = np.ascontiguousarray(feats, dtype=np.float32)
    labels = np.ascontiguousarray(labels, dtype=np.int32)
    grad = np.zeros(len(params), dtype=np.float64)
    loss = ctypes.c_double(0.0)
    rc = lib().oracle_step(L, _p(d), _aggr(aggr), int(bf16), ctypes.addressof(arr), _p(part),
                           full[-1].n_dst, K, _p(ks), len(ks), _p(params), _p(feats), feats.shape[1], _p(labels),
                           loss_scale, _p(grad), ctypes.byref(loss))
    if rc != 0:
        raise ValueError("oracle_step: invalid input")
    return grad, loss.value


def mem_estimate(dims: Sequence[int], aggr: str, blocks: Sequence) -> np.ndarray:
    """Table 3 memory estimate of one (micro-)batch:
    int64 [9] = element counts of terms (1)..(8) and the peak.  See
    oracle_mem_estimate in oracle.c."""
    L = len(blocks)
    d = np.ascontiguousarray(dims, dtype=np.int32)
    nd = np.array([b.n_dst for b in blocks], dtype=np.int64)
    ns = np.array([b.n_src for b in blocks], dtype=np.int64)
    ne = np.array([int(b.indptr[-1]) for b in blocks], dtype=np.int64)
    t = np.zeros(9, dtype=np.int64)
    lib().oracle_mem_estimate(L, _p(d), _aggr(aggr), _p(nd), _p(ns), _p(ne), _p(t))
    return t


def memory_aware_k(full: Sequence, dims: Sequence[int], aggr: str, capacity_elems: int, partition_fn,
                   K0: int = 1, K_max: Optional[int] = None):
    """Memory-aware batch re-partitioning: partition the
    REG K ways (partition_fn(K) -> part, supplied by the caller: the partition
    is an input both sides share), estimate every micro-batch without running
    it; if the largest estimate exceeds the capacity try K+1.  Returns
    (K, part, peak) or (-1, None, smallest peak seen) when no K <= K_max
    (default n_out) fits."""
    n_out = full[-1].n_dst
    K_max = n_out if K_max is None else K_max
    best = None
    for K in range(max(1, K0), K_max + 1):
        part = np.asarray(partition_fn(K), dtype=np.int32)
        peak = max(int(mem_estimate(dims, aggr, extract(full, part, K, k))[8]) for k in range(K))
        best = peak if best is None else min(best, peak)
        if peak <= capacity_elems:
            return K, part, peak
    return -1, None, best
