"""Multi-GPU glue (host side): one process per GPU, micro-batches sharded
across ranks, ONE all-reduce of the accumulated gradient per step.

Betty itself is single-GPU (multi-GPU is future work);
here the K micro-batches of a batch are independent units (they share only
the read-only full-batch blocks, features and parameters), so each rank takes
a subset, accumulates its micro-batches' gradients locally (fused into the
dW GEMMs), and the ranks sum them with one NCCL all-reduce over NVLink before
the identical Adam update.
"""
from __future__ import annotations

import heapq
from typing import List, Sequence

import numpy as np


def micro_batch_costs(part: np.ndarray, K: int, out_indptr: np.ndarray) -> np.ndarray:
    """Scheduling cost proxy per micro-batch: sampled output-block edges of its
    outputs (host, O(n_out); not part of the hot path)."""
    deg = np.diff(np.asarray(out_indptr, dtype=np.int64))
    return np.bincount(np.asarray(part, dtype=np.int64), weights=deg + 1, minlength=K).astype(np.float64)


def plan_costs(sizes: np.ndarray, dims: Sequence[int], gamma: float = 0.008) -> np.ndarray:
    """Scheduling cost per micro-batch from its per-layer sizes (betty_mb_sizes: [K, L, 3] = n_dst,
    n_src, n_edges of every layer, a GPU count-only extraction): SURVEY.md §8(e)'s
    cost_k = sum_l (E_{k,l} F_l + gamma n_dst,k,l F_l F_{l+1}) -- the aggregation's gathered elements
    plus the dense layer's flops converted to element-equivalents (gamma = 2 / ridge, ridge ~ 250 flop
    per byte).  Host arithmetic, outside the hot path."""
    sizes = np.asarray(sizes, dtype=np.float64)
    F = np.asarray(dims, dtype=np.float64)
    nd, E = sizes[:, :, 0], sizes[:, :, 2]
    return (E * F[None, :-1] + gamma * nd * F[None, :-1] * F[None, 1:]).sum(1)


def lpt_assign(costs: Sequence[float], world: int) -> List[List[int]]:
    """Longest-processing-time-first: micro-batches in decreasing cost go to
    the least loaded rank.  Deterministic (ties by index).  Returns, per rank,
    its micro-batch ids in ascending order."""
    order = sorted(range(len(costs)), key=lambda k: (-float(costs[k]), k))
    heap = [(0.0, r) for r in range(world)]
    out: List[List[int]] = [[] for _ in range(world)]
    for k in order:
        load, r = heapq.heappop(heap)
        out[r].append(k)
        heapq.heappush(heap, (load + float(costs[k]), r))
    return [sorted(x) for x in out]


def reg_rows(n_out: int, rank: int, world: int):
    """This rank's share [row0, row1) of the REG rows: the in-step REG rebuild is sharded by output
    rows instead of repeated on every rank (contiguous, sizes differ by at most one)."""
    return n_out * rank // world, n_out * (rank + 1) // world


def allreduce_grad(grad, group=None):
    """The one exchange step of a training step: sum of the ranks' gradients."""
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized() and dist.get_world_size() > 1:
        dist.all_reduce(grad, op=dist.ReduceOp.SUM, group=group)
    return grad
