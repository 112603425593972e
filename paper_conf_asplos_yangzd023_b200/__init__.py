"""Betty on B200: the data-parallel hot path of batch-level partitioned GNN
training (Yang et al., ASPLOS '23), as hand-written sm_100a CUDA behind the C
ABI of include/betty.h.

This module is the thin Python binding: the functions carry the ABI's names
and only marshal torch tensors (device memory, streams) into plain pointers.
Every step of the path runs in libbetty.so; if the library is missing, every
call raises -- there is no CPU or PyTorch fallback.
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass, field
from typing import List, Optional, Sequence

import numpy as np
import torch

from . import _lib as L
from ._lib import LIB_PATH  # noqa: F401

AGGR = {"mean": 0, "pool": 1, "sum": 2}
GEMM = {"fp32": 0, "bf16": 1}
PLAN_GRAPH, PLAN_REG, PLAN_FRESH = 1, 2, 4


class BettyError(RuntimeError):
    pass


def _stream(stream: Optional[torch.cuda.Stream] = None) -> ctypes.c_void_p:
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def _p(t: Optional[torch.Tensor]):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


class Context:
    """betty_ctx: one per device / rank."""

    def __init__(self, device: int = 0):
        self.device = device
        self.h = ctypes.c_void_p()
        st = L.lib().betty_ctx_create(device, None, None, None, ctypes.byref(self.h))
        if st != 0:
            raise BettyError(f"betty_ctx_create: {L.STATUS.get(st, st)}")

    def check(self, st: int, what: str):
        if st != 0:
            msg = L.lib().betty_last_error(self.h).decode()
            raise BettyError(f"{what}: {L.STATUS.get(st, st)}: {msg}")

    def close(self):
        if self.h:
            L.lib().betty_ctx_destroy(self.h)
            self.h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def betty_version() -> str:
    return L.lib().betty_version().decode()


def betty_ctx_create(device: int = 0) -> Context:
    return Context(device)


class _CAI:
    """__cuda_array_interface__ view of a library-owned device array."""

    def __init__(self, ptr: int, n: int, typestr: str):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False), "version": 2,
                                         "strides": None}


def _copy_out(ptr, n: int, dtype: torch.dtype, device: int) -> torch.Tensor:
    if n == 0 or not ptr:
        return torch.zeros(n, dtype=dtype, device=f"cuda:{device}")
    ts = {torch.int32: "<i4", torch.int64: "<i8", torch.float32: "<f4"}[dtype]
    return torch.as_tensor(_CAI(int(ptr), n, ts), device=f"cuda:{device}").clone()


@dataclass
class Block:
    """One bipartite layer on the device (betty_block); tensors own the memory."""
    n_dst: int
    n_src: int
    indptr: torch.Tensor                 # int64 [n_dst+1]
    indices: torch.Tensor                # int32 [E]
    src_gid: torch.Tensor                # int32 [n_src]
    src_pos: Optional[torch.Tensor] = None
    t_indptr: Optional[torch.Tensor] = None
    t_indices: Optional[torch.Tensor] = None

    @property
    def n_edges(self) -> int:
        return int(self.indices.numel())

    def struct(self) -> L.betty_block:
        return L.betty_block(self.n_dst, self.n_src, self.n_edges, _p(self.indptr), _p(self.indices),
                             _p(self.src_pos), _p(self.src_gid), _p(self.t_indptr), _p(self.t_indices))


def _blocks_struct(blocks: Sequence[Block]):
    arr = (L.betty_block * len(blocks))()
    for i, b in enumerate(blocks):
        arr[i] = b.struct()
    return arr


def blocks_to_device(blocks, device: int = 0) -> List[Block]:
    """Full-batch blocks from the input generator (numpy) -> device tensors."""
    dev = f"cuda:{device}"
    out = []
    for b in blocks:
        out.append(Block(int(b.n_dst), int(b.n_src), torch.as_tensor(b.indptr, dtype=torch.int64).to(dev),
                         torch.as_tensor(b.nbr_pos, dtype=torch.int32).to(dev),
                         torch.as_tensor(b.src_gid, dtype=torch.int32).to(dev)))
    return out


def betty_reg_build(ctx: Context, out_block: Block, stream=None):
    """a1: REG of the full-batch output block -> (indptr int64, col int32, w int32) device tensors."""
    ob = out_block.struct()
    csr = L.betty_csr()
    ctx.check(L.lib().betty_reg_build(ctx.h, ctypes.byref(ob), ctypes.byref(csr), _stream(stream)), "betty_reg_build")
    try:
        return (_copy_out(csr.indptr, out_block.n_dst + 1, torch.int64, ctx.device),
                _copy_out(csr.col, csr.nnz, torch.int32, ctx.device),
                _copy_out(csr.w, csr.nnz, torch.int32, ctx.device))
    finally:
        L.lib().betty_csr_free(ctx.h, ctypes.byref(csr))


def betty_reg_build_rows(ctx: Context, out_block: Block, row0: int, row1: int, stream=None):
    """a1 for output rows [row0, row1) only (one rank's share): (indptr rebased, col global, w)."""
    ob = out_block.struct()
    csr = L.betty_csr()
    ctx.check(L.lib().betty_reg_build_rows(ctx.h, ctypes.byref(ob), row0, row1, ctypes.byref(csr), _stream(stream)),
              "betty_reg_build_rows")
    try:
        return (_copy_out(csr.indptr, csr.n + 1, torch.int64, ctx.device),
                _copy_out(csr.col, csr.nnz, torch.int32, ctx.device),
                _copy_out(csr.w, csr.nnz, torch.int32, ctx.device))
    finally:
        L.lib().betty_csr_free(ctx.h, ctypes.byref(csr))


def betty_extract_blocks(ctx: Context, full: Sequence[Block], part: torch.Tensor, K: int, k: int,
                         stream=None) -> List[Block]:
    """a2: micro-batch k of the K-way partition `part` (int32 cuda [n_out])."""
    nL = len(full)
    fa = _blocks_struct(full)
    out = (L.betty_block * nL)()
    ctx.check(L.lib().betty_extract_blocks(ctx.h, fa, nL, _p(part), full[-1].n_dst, K, k, out, _stream(stream)),
              "betty_extract_blocks")
    try:
        res = []
        for o in out:
            d = ctx.device
            res.append(Block(o.n_dst, o.n_src, _copy_out(o.indptr, o.n_dst + 1, torch.int64, d),
                             _copy_out(o.indices, o.n_edges, torch.int32, d),
                             _copy_out(o.src_gid, o.n_src, torch.int32, d),
                             _copy_out(o.src_pos, o.n_src, torch.int32, d),
                             _copy_out(o.t_indptr, o.n_src + 1, torch.int64, d),
                             _copy_out(o.t_indices, o.n_edges, torch.int32, d)))
        return res
    finally:
        L.lib().betty_block_free(ctx.h, out, nL)


@dataclass
class Model:
    dims: Sequence[int]
    aggr: str = "mean"
    gemm: str = "fp32"
    feat_dtype: str = "fp32"
    _dims: object = field(default=None, repr=False)

    def struct(self) -> L.betty_model:
        self._dims = (ctypes.c_int32 * len(self.dims))(*self.dims)
        return L.betty_model(len(self.dims) - 1, AGGR[self.aggr], GEMM[self.gemm],
                             0 if self.feat_dtype == "fp32" else 1, self._dims)


def betty_num_params(model: Model) -> int:
    m = model.struct()
    return int(L.lib().betty_num_params(ctypes.byref(m)))


class Saved:
    def __init__(self, ctx: Context, h: ctypes.c_void_p):
        self.ctx, self.h = ctx, h

    def free(self):
        if self.h:
            L.lib().betty_saved_free(self.ctx.h, self.h)
            self.h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def betty_sage_fwd(ctx: Context, model: Model, params: torch.Tensor, mb: Sequence[Block], feats: torch.Tensor,
                   stream=None):
    """a3: forward of one micro-batch -> (Saved, logits fp32 [n_out_mb, C])."""
    m = model.struct()
    ma = _blocks_struct(mb)
    logits = torch.empty((mb[-1].n_dst, model.dims[-1]), dtype=torch.float32, device=params.device)
    h = ctypes.c_void_p()
    ctx.check(L.lib().betty_sage_fwd(ctx.h, ctypes.byref(m), _p(params), ma, _p(feats), feats.stride(0),
                                     ctypes.byref(h), _p(logits), _stream(stream)), "betty_sage_fwd")
    return Saved(ctx, h), logits


def betty_sage_bwd(ctx: Context, model: Model, params: torch.Tensor, mb: Sequence[Block], saved: Saved,
                   labels: torch.Tensor, loss_scale: float, grad_accum: torch.Tensor, loss_accum: torch.Tensor,
                   stream=None):
    """a4-a6: loss + backward of one micro-batch, ADDING into grad_accum / loss_accum."""
    m = model.struct()
    ma = _blocks_struct(mb)
    ctx.check(L.lib().betty_sage_bwd(ctx.h, ctypes.byref(m), _p(params), ma, saved.h, _p(labels), loss_scale,
                                     _p(grad_accum), _p(loss_accum), _stream(stream)), "betty_sage_bwd")


class Plan:
    def __init__(self, ctx: Context, h: ctypes.c_void_p, keep):
        self.ctx, self.h, self._keep = ctx, h, keep

    def info(self) -> dict:
        i = L.betty_plan_info()
        self.ctx.check(L.lib().betty_plan_info_get(self.h, ctypes.byref(i)), "betty_plan_info_get")
        n = i.L
        return {"n_groups": i.n_groups, "edges": list(i.edges[:n]), "n_src": list(i.n_src[:n]),
                "n_dst": list(i.n_dst[:n]), "max_group_edges": list(i.max_group_edges[:n]), "reg_nnz": i.reg_nnz,
                "arena_bytes": i.arena_bytes, "kernels_per_step": i.kernels_per_step}

    def group_blocks(self, g: int) -> List[Block]:
        """Extraction of launch group g (group-concatenated), copied out (tests)."""
        out = (L.betty_block * len(self._keep[0]))()
        self.ctx.check(L.lib().betty_plan_group_blocks(self.ctx.h, self.h, g, out, _stream(None)),
                       "betty_plan_group_blocks")
        d = self.ctx.device
        res = []
        for o in out:
            res.append(Block(o.n_dst, o.n_src, _copy_out(o.indptr, o.n_dst + 1, torch.int64, d),
                             _copy_out(o.indices, o.n_edges, torch.int32, d),
                             _copy_out(o.src_gid, o.n_src, torch.int32, d),
                             _copy_out(o.src_pos, o.n_src, torch.int32, d),
                             _copy_out(o.t_indptr, o.n_src + 1, torch.int64, d) if o.t_indptr else None,
                             _copy_out(o.t_indices, o.n_edges, torch.int32, d) if o.t_indptr else None))
        return res

    def set_reg_rows(self, row0: int, row1: int, stream=None):
        """Shard the in-step REG rebuild: this plan computes output rows [row0, row1) only."""
        self.ctx.check(L.lib().betty_plan_set_reg_rows(self.ctx.h, self.h, row0, row1, _stream(stream)),
                       "betty_plan_set_reg_rows")

    def set_feature_shards(self, bases: Sequence[int], rows_per_shard: int):
        """Layer-0 features sharded by rows: row g in bases[g // rows_per_shard] (device pointers, peer
        mappings included); [] = one contiguous table (the feats argument of betty_step)."""
        arr = (ctypes.c_void_p * max(1, len(bases)))(*[int(b) for b in bases])
        self.ctx.check(L.lib().betty_plan_set_feature_shards(self.ctx.h, self.h, len(bases), arr, int(rows_per_shard)),
                       "betty_plan_set_feature_shards")

    def probe(self, site: int):
        """Bracket the launches of one kernel site with CUDA events (see betty.h)."""
        self.ctx.check(L.lib().betty_plan_probe(self.h, site), "betty_plan_probe")

    def probe_read(self):
        ms, n = ctypes.c_float(), ctypes.c_int32()
        self.ctx.check(L.lib().betty_plan_probe_read(self.h, ctypes.byref(ms), ctypes.byref(n)),
                       "betty_plan_probe_read")
        return ms.value, n.value

    def free(self):
        if self.h:
            L.lib().betty_plan_destroy(self.ctx.h, self.h)
            self.h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def betty_plan_create(ctx: Context, model: Model, full: Sequence[Block], part: torch.Tensor, K: int,
                      my_k: Sequence[int], group: int = 0, flags: int = PLAN_GRAPH, stream=None) -> Plan:
    m = model.struct()
    fa = _blocks_struct(full)
    ks = (ctypes.c_int32 * max(1, len(my_k)))(*my_k)
    h = ctypes.c_void_p()
    ctx.check(L.lib().betty_plan_create(ctx.h, ctypes.byref(m), fa, len(full), _p(part), full[-1].n_dst, K, ks,
                                        len(my_k), group, flags, ctypes.byref(h), _stream(stream)),
              "betty_plan_create")
    # the plan keeps pointers to the full blocks and part: keep them alive
    return Plan(ctx, h, (full, part, m))


def betty_step(ctx: Context, plan: Plan, params: torch.Tensor, feats: torch.Tensor, labels: torch.Tensor,
               loss_scale: float, grad_accum: torch.Tensor, loss_accum: torch.Tensor, stream=None):
    """One step on this rank: extraction + forward + loss + backward of all
    the plan's micro-batches, gradients ADDED into grad_accum."""
    ctx.check(L.lib().betty_step(ctx.h, plan.h, _p(params), _p(feats), feats.stride(0), _p(labels), loss_scale,
                                 _p(grad_accum), _p(loss_accum), _stream(stream)), "betty_step")


def betty_adam(ctx: Context, params: torch.Tensor, grad: torch.Tensor, m: torch.Tensor, v: torch.Tensor, t: int,
               lr: float = 1e-3, b1: float = 0.9, b2: float = 0.999, eps: float = 1e-8, zero_grad: bool = False,
               stream=None):
    ctx.check(L.lib().betty_adam(ctx.h, _p(params), _p(grad), _p(m), _p(v), params.numel(), t, lr, b1, b2, eps,
                                 int(zero_grad), _stream(stream)), "betty_adam")


def betty_test_gemm(ctx: Context, kind: int, A: torch.Tensor, B: torch.Tensor, K: int, N: int, use_tc: bool = True,
                    M: Optional[int] = None, stream=None) -> torch.Tensor:
    """Test hook of the dense kernels.  kind 0: A[M,K] @ B[N,K]^T; kind 1: A[M,K]^T @ B[M,N].  fp32
    operands (A.dtype float32) select FP32 mode (3xTF32 on tcgen05 when use_tc, else SIMT)."""
    M = A.shape[0] if M is None else M
    if A.dtype == torch.float32:
        kind |= 2
    if kind & 1 == 0:
        # rows up to A.shape[0] (the capacity) may be written; row stride padded to 16 bytes
        ldc = (N + 3) // 4 * 4
        Cfull = torch.zeros((A.shape[0], ldc), dtype=torch.float32, device=A.device)
        ctx.check(L.lib().betty_test_gemm(ctx.h, kind, _p(A), A.stride(0), _p(B), B.stride(0), M, A.shape[0], K, N,
                                          _p(Cfull), ldc, int(use_tc), _stream(stream)), "betty_test_gemm")
        return Cfull[:M, :N]
    else:
        C = torch.zeros((K, N), dtype=torch.float32, device=A.device)
        ldc = N
    ctx.check(L.lib().betty_test_gemm(ctx.h, kind, _p(A), A.stride(0), _p(B), B.stride(0), M, A.shape[0], K, N,
                                      _p(C), ldc, int(use_tc), _stream(stream)), "betty_test_gemm")
    return C


def betty_sync_check(ctx: Context, stream=None):
    ctx.check(L.lib().betty_sync_check(ctx.h, _stream(stream)), "betty_sync_check")


PART_METHODS = {"greedy": 0, "multilevel": 1}


def betty_reg_partition(indptr, col, w, K: int, method: str = "greedy", imbalance: float = 0.03):
    """Host K-way partition of a REG (numpy int64/int32 arrays) -> int32 part[n].
    method 'greedy' (exactly balanced) or 'multilevel' (METIS scheme, parts <=
    (1 + imbalance) n / K)."""
    import numpy as np
    if method != "greedy":
        indptr = np.ascontiguousarray(indptr, dtype=np.int64)
        col = np.ascontiguousarray(col, dtype=np.int32)
        w = None if w is None else np.ascontiguousarray(w, dtype=np.int32)
        n = len(indptr) - 1
        part = np.empty(max(n, 1), dtype=np.int32)
        st = L.lib().betty_reg_partition_ex(indptr.ctypes.data, col.ctypes.data,
                                            None if w is None else w.ctypes.data, n, K, PART_METHODS[method],
                                            float(imbalance), part.ctypes.data)
        if st != 0:
            raise BettyError(f"betty_reg_partition_ex: {L.STATUS.get(st, st)}")
        return part[:n]
    indptr = np.ascontiguousarray(indptr, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int32)
    w = None if w is None else np.ascontiguousarray(w, dtype=np.int32)
    n = len(indptr) - 1
    part = np.empty(max(n, 1), dtype=np.int32)
    st = L.lib().betty_reg_partition(indptr.ctypes.data, col.ctypes.data, None if w is None else w.ctypes.data, n,
                                     K, part.ctypes.data)
    if st != 0:
        raise BettyError(f"betty_reg_partition: {L.STATUS.get(st, st)}")
    return part[:n]


# ------------------------------------------------- §4.4 memory-aware micro-batch count
def betty_mb_sizes(ctx: Context, full: Sequence[Block], part: torch.Tensor, K: int, stream=None):
    """Count-only extraction: int64 numpy [K, L, 3] = (n_dst, n_src, n_edges)
    of every layer of every micro-batch of the K-way partition (cuda int32)."""
    import numpy as np
    nL = len(full)
    out = np.zeros((K, nL, 3), dtype=np.int64)
    ctx.check(L.lib().betty_mb_sizes(ctx.h, _blocks_struct(full), nL, _p(part), full[-1].n_dst, K,
                                     out.ctypes.data, _stream(stream)), "betty_mb_sizes")
    return out


def betty_mem_estimate(model: Model, sizes):
    """Table 3 estimate of one micro-batch from its
    [L, 3] sizes: int64 numpy [9] = element counts of terms (1)..(8), peak."""
    import numpy as np
    sz = np.ascontiguousarray(sizes, dtype=np.int64).reshape(-1)
    t = np.zeros(9, dtype=np.int64)
    m = model.struct()
    st = L.lib().betty_mem_estimate(ctypes.byref(m), sz.ctypes.data, t.ctypes.data)
    if st != 0:
        raise BettyError(f"betty_mem_estimate: {L.STATUS.get(st, st)}")
    return t


def betty_memory_aware_k(ctx: Context, model: Model, full: Sequence[Block], reg, capacity_bytes: int, K0: int = 1,
                         K_max: int = 0, method: str = "multilevel", stream=None):
    """Memory-aware re-partitioning: the first K >= K0
    whose largest micro-batch estimate fits capacity_bytes.  reg = host
    (indptr, col, w) numpy arrays.  Returns (K, part int32 numpy, peak_bytes);
    K = -1 (part None) when no K <= K_max fits."""
    import numpy as np
    ip, col, w = (np.ascontiguousarray(reg[0], dtype=np.int64), np.ascontiguousarray(reg[1], dtype=np.int32),
                  np.ascontiguousarray(reg[2], dtype=np.int32))
    n_out = full[-1].n_dst
    part = np.zeros(max(1, n_out), dtype=np.int32)
    k_out, peak = ctypes.c_int32(0), ctypes.c_int64(0)
    m = model.struct()
    ctx.check(L.lib().betty_memory_aware_k(ctx.h, ctypes.byref(m), _blocks_struct(full), len(full), ip.ctypes.data,
                                           col.ctypes.data, w.ctypes.data, n_out, int(capacity_bytes), K0, K_max,
                                           PART_METHODS[method], part.ctypes.data, ctypes.byref(k_out), ctypes.byref(peak),
                                           _stream(stream)), "betty_memory_aware_k")
    return k_out.value, (part[:n_out] if k_out.value > 0 else None), peak.value


# ------------------------------------------------------------------ CUDA IPC buffers (sharded features)
class DevBuffer:
    """A cudaMalloc'd device buffer other processes can map (betty_dev_alloc); .tensor(dtype, shape)
    views it as a torch tensor (no copy)."""

    def __init__(self, ctx: Context, nbytes: int, ptr: Optional[int] = None, owned: bool = True):
        self.ctx, self.nbytes, self.owned = ctx, int(nbytes), owned
        if ptr is None:
            p = ctypes.c_void_p()
            ctx.check(L.lib().betty_dev_alloc(ctx.h, self.nbytes, ctypes.byref(p)), "betty_dev_alloc")
            ptr = p.value
        self.ptr = int(ptr)

    def tensor(self, dtype: torch.dtype, shape) -> torch.Tensor:
        ts = {torch.float32: "<f4", torch.bfloat16: "<V2", torch.int32: "<i4"}[dtype]
        n = int(np.prod(shape))
        cai = _CAI(self.ptr, n, ts if dtype != torch.bfloat16 else "<i2")
        t = torch.as_tensor(cai, device=f"cuda:{self.ctx.device}")
        if dtype == torch.bfloat16:
            t = t.view(torch.bfloat16)
        return t.view(*shape)

    def ipc_handle(self) -> bytes:
        buf = ctypes.create_string_buffer(64)
        self.ctx.check(L.lib().betty_ipc_handle(self.ctx.h, ctypes.c_void_p(self.ptr), buf), "betty_ipc_handle")
        return buf.raw

    @staticmethod
    def open(ctx: Context, handle: bytes, nbytes: int) -> "DevBuffer":
        p = ctypes.c_void_p()
        ctx.check(L.lib().betty_ipc_open(ctx.h, ctypes.create_string_buffer(handle, 64), ctypes.byref(p)),
                  "betty_ipc_open")
        return DevBuffer(ctx, nbytes, p.value, owned=False)

    def free(self):
        if self.ptr:
            if self.owned:
                L.lib().betty_dev_free(self.ctx.h, ctypes.c_void_p(self.ptr))
            else:
                L.lib().betty_ipc_close(self.ctx.h, ctypes.c_void_p(self.ptr))
            self.ptr = 0
