"""Seeded synthetic inputs shared by the CUDA path and the CPU oracle.

This module holds none of Betty's arithmetic.  It generates power-law graphs
shaped like the paper's datasets (Table 4), features,
labels, training seeds, and the canonical full-batch sampled blocks
(DGL-style fanout sampling).  All of it
runs in ``gen.c`` (C + OpenMP), built on first use into ``libsynth.so``.

Presets C1..C5 follow SURVEY.md §8(d) / BASELINE.json ``configs``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field
from typing import List, Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gen.c")
_LIB_PATH = os.path.join(_HERE, "libsynth.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-march=x86-64-v2", "-fopenmp", "-shared", "-fPIC",
                               "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


class _CBlock(ctypes.Structure):
    _fields_ = [("n_dst", ctypes.c_int64), ("n_src", ctypes.c_int64), ("n_edges", ctypes.c_int64),
                ("indptr", ctypes.POINTER(ctypes.c_int64)), ("nbr_pos", ctypes.POINTER(ctypes.c_int32)),
                ("src_gid", ctypes.POINTER(ctypes.c_int32))]


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        P = ctypes.c_void_p
        i64, i32, u64, dbl = ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64, ctypes.c_double
        L.synth_graph.restype = i64
        L.synth_graph.argtypes = [i64, i64, i32, dbl, dbl, u64, ctypes.POINTER(P), ctypes.POINTER(P), P]
        L.synth_features.restype = None
        L.synth_features.argtypes = [i64, i32, i64, P, i32, dbl, dbl, u64, P]
        L.synth_features_ids.restype = None
        L.synth_features_ids.argtypes = [P, i64, i64, i32, i64, P, i32, dbl, dbl, u64, P]
        L.synth_seeds.restype = None
        L.synth_seeds.argtypes = [i64, i64, u64, P]
        L.synth_sample.restype = ctypes.c_int
        L.synth_sample.argtypes = [i64, P, P, i64, P, i32, P, u64, ctypes.POINTER(_CBlock)]
        L.synth_free.restype = None
        L.synth_free.argtypes = [P]
        L.synth_num_threads.restype = ctypes.c_int
        _lib = L
    return _lib


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


def _take(p, n: int, dtype) -> np.ndarray:
    """Copy a malloc'd C array into numpy and free it."""
    addr = p if isinstance(p, int) else ctypes.cast(p, ctypes.c_void_p).value
    if n == 0:
        out = np.zeros(0, dtype=dtype)
    else:
        buf = (ctypes.c_char * (n * np.dtype(dtype).itemsize)).from_address(addr)
        out = np.frombuffer(buf, dtype=dtype).copy()
    lib().synth_free(addr)
    return out


@dataclass
class Graph:
    indptr: np.ndarray      # int64 [N+1]
    indices: np.ndarray     # int32 [nnz], rows ascending, symmetric, no self loops
    comm: np.ndarray        # int32 [N]

    @property
    def n(self) -> int:
        return len(self.indptr) - 1


def graph(n: int, pairs: int, n_comm: int, mu: float, beta: float, seed: int) -> Graph:
    comm = np.empty(n, dtype=np.int32)
    ip, ix = ctypes.c_void_p(), ctypes.c_void_p()
    nnz = lib().synth_graph(n, pairs, n_comm, mu, beta, seed, ctypes.byref(ip), ctypes.byref(ix), _ptr(comm))
    if nnz < 0:
        raise MemoryError("synth_graph: allocation failed")
    return Graph(_take(ip.value, n + 1, np.int64), _take(ix.value, nnz, np.int32), comm)


def graph_from_edges(n: int, edges: Sequence) -> Graph:
    """Hand-built graph (tests): undirected pairs -> symmetric deduped CSR."""
    adj = [set() for _ in range(n)]
    for u, v in edges:
        if u != v:
            adj[u].add(v)
            adj[v].add(u)
    indptr = np.zeros(n + 1, dtype=np.int64)
    for i in range(n):
        indptr[i + 1] = indptr[i] + len(adj[i])
    indices = np.array([j for i in range(n) for j in sorted(adj[i])], dtype=np.int32)
    return Graph(indptr, indices, np.zeros(n, dtype=np.int32))


def features(comm: np.ndarray, F: int, ld: int, kind: int = 0, signal: float = 0.5, p: float = 0.0126,
             seed: int = 5) -> np.ndarray:
    n = len(comm)
    out = np.empty((n, ld), dtype=np.float32)
    lib().synth_features(n, F, ld, _ptr(np.ascontiguousarray(comm, dtype=np.int32)), kind, signal, p, seed,
                         _ptr(out))
    return out


def features_rows(comm: np.ndarray, F: int, ld: int, ids: Optional[np.ndarray] = None, row0: int = 0, n: int = 0,
                  kind: int = 0, signal: float = 0.5, p: float = 0.0126, seed: int = 5) -> np.ndarray:
    """Rows of `features(comm, ...)` for the nodes `ids` (or the range [row0, row0+n)) only: tables
    too large for host memory (C5) are generated in chunks, and a sample's rows on their own."""
    comm = np.ascontiguousarray(comm, dtype=np.int32)
    if ids is not None:
        ids = np.ascontiguousarray(ids, dtype=np.int32)
        n = len(ids)
    out = np.empty((n, ld), dtype=np.float32)
    lib().synth_features_ids(None if ids is None else _ptr(ids), row0, n, F, ld, _ptr(comm), kind, signal, p, seed,
                             _ptr(out))
    return out


def seeds(n: int, n_out: int, seed: int) -> np.ndarray:
    out = np.empty(n_out, dtype=np.int32)
    lib().synth_seeds(n, n_out, seed, _ptr(out))
    return out


@dataclass
class Block:
    """One full-batch bipartite layer, CSR by dst.  dst ids == src ids [0, n_dst)."""
    n_dst: int
    n_src: int
    indptr: np.ndarray      # int64 [n_dst+1]
    nbr_pos: np.ndarray     # int32 [E] full-batch src positions
    src_gid: np.ndarray     # int32 [n_src] global node ids

    @property
    def n_edges(self) -> int:
        return int(self.indptr[-1])


def sample(g: Graph, seed_nodes: np.ndarray, fanouts: Sequence[int], seed: int) -> List[Block]:
    """fanouts[l] bounds block l (l=0 input ... L-1 output); <0 = full neighbourhood."""
    L = len(fanouts)
    fan = np.ascontiguousarray(fanouts, dtype=np.int32)
    sd = np.ascontiguousarray(seed_nodes, dtype=np.int32)
    cb = (_CBlock * L)()
    rc = lib().synth_sample(g.n, _ptr(g.indptr), _ptr(g.indices), len(sd), _ptr(sd), L, _ptr(fan), seed, cb)
    if rc != 0:
        raise MemoryError("synth_sample failed")
    out = []
    for l in range(L):
        b = cb[l]
        out.append(Block(int(b.n_dst), int(b.n_src),
                         _take(ctypes.cast(b.indptr, ctypes.c_void_p).value, b.n_dst + 1, np.int64),
                         _take(ctypes.cast(b.nbr_pos, ctypes.c_void_p).value, b.n_edges, np.int32),
                         _take(ctypes.cast(b.src_gid, ctypes.c_void_p).value, b.n_src, np.int32)))
    return out


def blocks_from_rows(seed_nodes: Sequence[int], rows_per_layer: Sequence[dict]) -> List[Block]:
    """Hand-built full-batch blocks (tests / golden).  rows_per_layer[l] maps a
    dst global id to its (already sampled) neighbour global ids for block l.
    Applies the canonical C-1 layout: rows ascending gid, src = dst ++ new
    ascending gid, edges as src positions."""
    L = len(rows_per_layer)
    dst = [int(x) for x in seed_nodes]
    blocks: List[Optional[Block]] = [None] * L
    for l in range(L - 1, -1, -1):
        rows = rows_per_layer[l]
        nb = [sorted(rows.get(v, [])) for v in dst]
        in_dst = set(dst)
        new = sorted({u for r in nb for u in r if u not in in_dst})
        src = dst + new
        pos = {g: i for i, g in enumerate(src)}
        indptr = np.zeros(len(dst) + 1, dtype=np.int64)
        for i, r in enumerate(nb):
            indptr[i + 1] = indptr[i] + len(r)
        nbr = np.array([pos[u] for r in nb for u in r], dtype=np.int32)
        blocks[l] = Block(len(dst), len(src), indptr, nbr, np.array(src, dtype=np.int32))
        dst = src
    return blocks  # type: ignore[return-value]


@dataclass
class Config:
    name: str
    n: int
    pairs: int
    F: int
    C: int
    hidden: int
    L: int
    aggr: str                 # "mean" | "pool"
    fanouts: Sequence[int]    # block 0 (input) ... block L-1 (output)
    n_out: int
    Ks: Sequence[int]
    n_comm: int
    mu: float
    beta: float = 0.45
    feat_kind: int = 0
    oversample: float = 1.0   # candidate pairs drawn per target pair (dedupe loses some)
    seeds: dict = field(default_factory=lambda: dict(graph=1, sample=2, part=3, init=4, feat=5, train=6))

    @property
    def dims(self) -> List[int]:
        return [self.F] + [self.hidden] * (self.L - 1) + [self.C]

    @property
    def ld(self) -> int:
        return (self.F + 7) // 8 * 8


CONFIGS = {
    # configs[0]: Cora-shaped, 2-layer SAGE-mean, fanout (10,25), 140 outputs, K=2
    "C1": Config("cora", 2708, 5278, 1433, 7, 256, 2, "mean", (10, 25), 140, (2,), 7, 0.2, beta=0.35,
                 feat_kind=1),
    # configs[1]: ogbn-arxiv-shaped, 3-layer SAGE-mean, full neighbourhood, K 4..32
    "C2": Config("arxiv", 169343, 1166243, 128, 40, 256, 3, "mean", (-1, -1, -1), 90941, (4, 8, 16, 32), 400,
                 0.2),
    # configs[2]: ogbn-products-shaped, 2-layer SAGE-mean, fanout (10,25), K 8..64  (the metric's workload)
    "C3": Config("products", 2449029, 61859140, 100, 47, 256, 2, "mean", (10, 25), 196615, (8, 16, 32, 64),
                 4000, 0.1),
    # configs[3]: products-shaped, 5-layer SAGE-pool fanout 10 per layer
    "C4": Config("products-deep-pool", 2449029, 61859140, 100, 47, 256, 5, "pool", (10, 10, 10, 10, 10),
                 196615, (8,), 4000, 0.1, oversample=1.096),
    # configs[4]: ogbn-papers100M-shaped, 3-layer SAGE-mean, fanout (5, 10, 15) (SURVEY.md §8(d) proposal),
    # 1.2 M outputs, K 16..64; the 57 GB fp32 feature table is generated in chunks (features_rows)
    "C5": Config("papers100M", 111059956, 800000000, 128, 172, 256, 3, "mean", (5, 10, 15), 1207179, (16, 32, 64),
                 20000, 0.1),
}

# feature tables above this many bytes (fp32) are never materialised on the host
HOST_FEATURE_LIMIT = 8 << 30


def scaled(cfg: Config, frac: float, name: Optional[str] = None) -> Config:
    """A smaller graph of the same shape (same degree, communities scaled)."""
    import dataclasses
    return dataclasses.replace(cfg, name=name or f"{cfg.name}@{frac:g}", n=max(64, int(cfg.n * frac)),
                               pairs=max(64, int(cfg.pairs * frac)), n_out=max(4, int(cfg.n_out * frac)),
                               n_comm=max(2, int(cfg.n_comm * frac)))


@dataclass
class Dataset:
    cfg: Config
    graph: Graph
    feats: Optional[np.ndarray]   # float32 [N, ld]; None when generated in chunks (features_rows)
    labels: np.ndarray        # int32 [N]
    seeds: np.ndarray         # int32 [n_out] ascending
    blocks: List[Block]       # block 0 (input) ... L-1 (output)


def relabel_by_community(g: Graph) -> Graph:
    """(Study input) the same graph with node ids renumbered so that every community is a contiguous id
    range (stable within a community): an upper bound on what a locality-aware node order can do."""
    order = np.argsort(g.comm, kind="stable")
    inv = np.empty_like(order)
    inv[order] = np.arange(len(order))
    deg = np.diff(g.indptr)[order]
    indptr = np.concatenate([[0], np.cumsum(deg)]).astype(np.int64)
    starts = g.indptr[order]
    idx = np.repeat(starts - indptr[:-1], deg) + np.arange(indptr[-1])
    vals = inv[g.indices[idx]].astype(np.int64)
    rows = np.repeat(np.arange(len(order), dtype=np.int64), deg)
    vals = vals[np.lexsort((vals, rows))].astype(np.int32)
    return Graph(indptr, vals, g.comm[order])


def make(cfg: Config, with_features: Optional[bool] = True, community_order: bool = False) -> Dataset:
    s = cfg.seeds
    g = graph(cfg.n, int(cfg.pairs * cfg.oversample), cfg.n_comm, cfg.mu, cfg.beta, s["graph"])
    if community_order:
        g = relabel_by_community(g)
    sd = seeds(g.n, cfg.n_out, s["train"])
    blocks = sample(g, sd, cfg.fanouts, s["sample"])
    if with_features is None:
        with_features = cfg.n * cfg.ld * 4 <= HOST_FEATURE_LIMIT
    feats = features(g.comm, cfg.F, cfg.ld, cfg.feat_kind, seed=s["feat"]) if with_features else None
    labels = (g.comm % cfg.C).astype(np.int32)
    return Dataset(cfg, g, feats, labels, sd, blocks)


def features_device(cfg: Config, ds: "Dataset", bf16: bool, align: int, device, chunk_rows: int = 1 << 22):
    """The feature table as a torch tensor in HBM (bf16 or fp32), rows padded with zeros to a multiple
    of `align` bytes (0: cfg.ld).  Tables too large for host memory (C5: 111 M x 128 fp32 = 57 GB)
    are generated in chunks of rows (features_rows) and converted on the device; the others are
    copied from ds.feats."""
    import torch
    dt = torch.bfloat16 if bf16 else torch.float32
    esz = 2 if bf16 else 4
    per = max(1, align // esz) if align > 0 else 1
    ld = (cfg.ld + per - 1) // per * per
    out = torch.zeros((cfg.n, ld), dtype=dt, device=device)
    if ds.feats is not None:
        out[:, :cfg.ld] = torch.as_tensor(ds.feats).to(device).to(dt)
        return out
    for r0 in range(0, cfg.n, chunk_rows):
        n = min(chunk_rows, cfg.n - r0)
        h = features_rows(ds.graph.comm, cfg.F, cfg.ld, row0=r0, n=n, kind=cfg.feat_kind, seed=cfg.seeds["feat"])
        out[r0:r0 + n, :cfg.ld] = torch.from_numpy(h).to(device).to(dt)
    return out


def features_fill_rows(cfg: Config, ds: "Dataset", out, row0: int, chunk_rows: int = 1 << 22):
    """Fill a device tensor out[n, ld] (n <= rows left from row0) with feature rows row0 .. row0+n-1
    (columns [0, cfg.ld), the rest zero): one shard of a row-sharded table."""
    import torch
    n = min(out.shape[0], cfg.n - row0)
    out.zero_()
    for r0 in range(row0, row0 + n, chunk_rows):
        m = min(chunk_rows, row0 + n - r0)
        if ds.feats is not None:
            h = ds.feats[r0:r0 + m]
        else:
            h = features_rows(ds.graph.comm, cfg.F, cfg.ld, row0=r0, n=m, kind=cfg.feat_kind, seed=cfg.seeds["feat"])
        out[r0 - row0:r0 - row0 + m, :cfg.ld] = torch.from_numpy(np.ascontiguousarray(h)).to(out.device).to(out.dtype)
    return out


def init_params(dims: Sequence[int], aggr: str, seed: int = 4) -> np.ndarray:
    """Xavier-uniform weights, zero... small uniform biases; flat fp32 in the
    layout of include/betty.h (per layer: [W_pool, b_pool] (pool only),
    W_self [F_l x F_l+1], W_neigh [F_l x F_l+1], b [F_l+1])."""
    rng = np.random.default_rng(seed)
    parts = []
    for l in range(len(dims) - 1):
        fi, fo = dims[l], dims[l + 1]
        if aggr == "pool":
            a = np.sqrt(6.0 / (fi + fi))
            parts += [rng.uniform(-a, a, fi * fi), rng.uniform(-0.1, 0.1, fi)]
        a = np.sqrt(6.0 / (fi + fo))
        parts += [rng.uniform(-a, a, fi * fo), rng.uniform(-a, a, fi * fo), rng.uniform(-0.1, 0.1, fo)]
    return np.concatenate(parts).astype(np.float32)


def n_params(dims: Sequence[int], aggr: str) -> int:
    n = 0
    for l in range(len(dims) - 1):
        fi, fo = dims[l], dims[l + 1]
        if aggr == "pool":
            n += fi * fi + fi
        n += 2 * fi * fo + fo
    return n


def range_partition(n_out: int, K: int) -> np.ndarray:
    """Contiguous output positions per part (the paper's 'range' baseline,
    PAPER.md:1222-1230).  Host-side, outside the hot path."""
    return (np.arange(n_out, dtype=np.int64) * K // max(n_out, 1)).astype(np.int32)


def random_partition(n_out: int, K: int, seed: int = 3) -> np.ndarray:
    rng = np.random.default_rng(seed)
    return rng.integers(0, K, n_out).astype(np.int32)
