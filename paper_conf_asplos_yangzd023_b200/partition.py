"""Host-side partition baselines (outside the hot path, like the REG partitioner itself).

The paper compares Betty's REG partition with three redundancy-unaware partitions of the output
nodes (§6.1 "Comparison with other graph partition algorithms"; redundancy at
K = 64 in §6.5): range, random (synth.range_partition / random_partition) and
METIS.  Reading P2: "Metis" partitions the output nodes by the structure of the RAW
input graph -- the subgraph it induces on the outputs, unit weights -- with the same multilevel
partitioner the REG uses (betty_reg_partition_ex, the METIS scheme), so the two differ only in the
graph they cut: raw adjacency (redundancy-unaware) vs REG weights (shared input neighbours).
"""
from __future__ import annotations

import numpy as np


def induced_subgraph(indptr: np.ndarray, indices: np.ndarray, nodes: np.ndarray):
    """CSR over positions 0..len(nodes)-1 of the subgraph the graph (CSR, global ids) induces on
    `nodes` (global ids): row i lists the positions j of i's neighbours that are in `nodes`,
    ascending.  Returns (indptr int64, col int32)."""
    indptr = np.asarray(indptr, dtype=np.int64)
    indices = np.asarray(indices, dtype=np.int64)
    nodes = np.asarray(nodes, dtype=np.int64)
    pos = np.full(len(indptr) - 1, -1, dtype=np.int64)
    pos[nodes] = np.arange(len(nodes))
    starts, ends = indptr[nodes], indptr[nodes + 1]
    deg = ends - starts
    rows = np.repeat(np.arange(len(nodes)), deg)
    flat = np.concatenate([indices[s:e] for s, e in zip(starts, ends)]) if len(nodes) else np.zeros(0, np.int64)
    tgt = pos[flat]
    keep = tgt >= 0
    rows, tgt = rows[keep], tgt[keep]
    order = np.lexsort((tgt, rows))
    rows, tgt = rows[order], tgt[order]
    ip = np.zeros(len(nodes) + 1, dtype=np.int64)
    np.add.at(ip, rows + 1, 1)
    return np.cumsum(ip), tgt.astype(np.int32)


def raw_graph_partition(indptr: np.ndarray, indices: np.ndarray, seeds: np.ndarray, K: int) -> np.ndarray:
    """The paper's "Metis" baseline: K-way multilevel partition of the outputs (seeds, in output order)
    by the raw graph's induced subgraph, unit weights.  int32 part[n_out]."""
    from . import betty_reg_partition
    ip, col = induced_subgraph(indptr, indices, seeds)
    return betty_reg_partition(ip, col, np.ones(len(col), dtype=np.int32), K, method="multilevel")
