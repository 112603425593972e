"""Layer-0 features sharded by rows (BASELINE.json configs[4]): the plan's gathers
read row g from shard g // rows_per_shard.  One process with R virtual shards (separate device
buffers on cuda:0), and two processes on cuda:0 that map each other's shard through CUDA IPC (the
multi-GPU mechanism: peer pointers, no collective), against the unsharded step and the oracle."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import oracle
import synth
from tests.helpers import assert_grad_close, tiny

pytestmark = pytest.mark.gpu

DIMS = [24, 48, 5]
K = 5


def _case():
    g, sd, blocks, feats, _ = tiny(n=1000, pairs=5000, fanouts=(4, 6), n_out=80, F=DIMS[0], C=DIMS[-1], seed=31,
                                   ld=24)
    labels = (np.arange(1000) * 3 % DIMS[-1]).astype(np.int32)
    part = synth.random_partition(len(sd), K, 2)
    params = synth.init_params(DIMS, "mean", seed=7)
    return sd, blocks, feats, labels, part, params


def _shard(B, ctx, feats, mode, r, rps):
    """DevBuffer holding rows [r rps, (r+1) rps) of the table (padded with zero rows)."""
    dt = torch.bfloat16 if mode == "bf16" else torch.float32
    ld = feats.shape[1]
    buf = B.DevBuffer(ctx, rps * ld * (2 if mode == "bf16" else 4))
    t = buf.tensor(dt, (rps, ld))
    t.zero_()
    rows = torch.as_tensor(feats[r * rps:(r + 1) * rps]).cuda().to(dt)
    t[:rows.shape[0]].copy_(rows)
    return buf


def _step(B, ctx, plan, P, X, Y, n_out):
    grad = torch.zeros_like(P)
    loss = torch.zeros(1, device="cuda")
    B.betty_step(ctx, plan, P, X, Y, 1.0 / n_out, grad, loss)
    B.betty_sync_check(ctx)
    return grad.cpu().numpy().astype(np.float64), loss.item()


@pytest.mark.parametrize("mode,rtol", [("fp32", 1e-5), ("bf16", 2e-2)])
@pytest.mark.parametrize("R", [1, 3, 8])
def test_virtual_shards_one_gpu(mode, rtol, R):
    import paper_conf_asplos_yangzd023_b200 as B
    sd, blocks, feats, labels, part, params = _case()
    ctx = B.betty_ctx_create(0)
    dev = B.blocks_to_device(blocks)
    model = B.Model(DIMS, "mean", mode, mode)
    plan = B.betty_plan_create(ctx, model, dev, torch.as_tensor(part).cuda(), K, list(range(K)), group=2,
                               flags=B.PLAN_GRAPH)
    P = torch.as_tensor(params).cuda()
    X = torch.as_tensor(feats).cuda()
    if mode == "bf16":
        X = X.to(torch.bfloat16).contiguous()
    Y = torch.as_tensor(labels).cuda()
    g_full, l_full = _step(B, ctx, plan, P, X, Y, len(sd))
    rps = (len(feats) + R - 1) // R
    bufs = [_shard(B, ctx, feats, mode, r, rps) for r in range(R)]
    plan.set_feature_shards([b.ptr for b in bufs], rps)
    for rep in range(2):
        stub = torch.zeros((1, X.shape[1]), dtype=X.dtype, device="cuda")     # only its row stride is used
        g, l = _step(B, ctx, plan, P, stub, Y, len(sd))
        np.testing.assert_allclose(g, g_full, rtol=1e-6, atol=1e-12)
        assert l == pytest.approx(l_full, rel=1e-6)
    og, ol = oracle.step(DIMS, "mean", mode == "bf16", blocks, part, K, list(range(K)), params, feats, labels,
                         1.0 / len(sd))
    assert_grad_close(g, og, DIMS, "mean", rtol, f"{R} shards {mode}")
    plan.set_feature_shards([], 0)                     # back to the contiguous table
    g2, _ = _step(B, ctx, plan, P, X, Y, len(sd))
    np.testing.assert_array_equal(g2, g_full)
    plan.free()
    for b in bufs:
        b.free()


def test_shards_rejected_for_project_first_layer0():
    import paper_conf_asplos_yangzd023_b200 as B
    g, sd, blocks, feats, labels = tiny(n=300, pairs=1000, fanouts=(3, 4), n_out=20, F=40, C=4, seed=3, ld=40)
    ctx = B.betty_ctx_create(0)
    dev = B.blocks_to_device(blocks)
    plan = B.betty_plan_create(ctx, B.Model([40, 16, 4], "mean", "fp32", "fp32"), dev,
                               torch.as_tensor(synth.random_partition(20, 2, 1)).cuda(), 2, [0, 1], group=0, flags=0)
    buf = B.DevBuffer(ctx, 1024)
    with pytest.raises(B.BettyError, match="EUNSUPPORTED"):
        plan.set_feature_shards([buf.ptr], 300)
    plan.free()
    buf.free()


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _ipc_worker(rank, world, port, q):
    import torch.distributed as dist
    import paper_conf_asplos_yangzd023_b200 as B
    from paper_conf_asplos_yangzd023_b200.dist import allreduce_grad, lpt_assign, plan_costs
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    sd, blocks, feats, labels, part, params = _case()
    ctx = B.betty_ctx_create(0)
    rps = (len(feats) + world - 1) // world
    mine = _shard(B, ctx, feats, "fp32", rank, rps)            # this rank owns rows [rank rps, ...)
    handles = [None] * world
    dist.all_gather_object(handles, mine.ipc_handle())
    bases, opened = [], []
    for r in range(world):
        if r == rank:
            bases.append(mine.ptr)
        else:
            o = B.DevBuffer.open(ctx, handles[r], rps * feats.shape[1] * 4)
            opened.append(o)
            bases.append(o.ptr)
    dev = B.blocks_to_device(blocks)
    dpart = torch.as_tensor(part).cuda()
    ks = lpt_assign(plan_costs(B.betty_mb_sizes(ctx, dev, dpart, K), DIMS), world)[rank]
    plan = B.betty_plan_create(ctx, B.Model(DIMS, "mean", "fp32", "fp32"), dev, dpart, K, ks, group=0,
                               flags=B.PLAN_GRAPH)
    plan.set_feature_shards(bases, rps)
    grad = torch.zeros(len(params), device="cuda")
    loss = torch.zeros(1, device="cuda")
    B.betty_step(ctx, plan, torch.as_tensor(params).cuda(), torch.zeros((1, feats.shape[1]), device="cuda"),
                 torch.as_tensor(labels).cuda(), 1.0 / len(sd), grad, loss)
    B.betty_sync_check(ctx)
    t = torch.cat([grad, loss]).double()
    allreduce_grad(t)
    dist.barrier()                                             # peers done reading before unmapping
    plan.free()
    for o in opened:
        o.free()
    dist.barrier()
    mine.free()
    if rank == 0:
        q.put(t.cpu().numpy())
    dist.destroy_process_group()


def test_two_ranks_ipc_shards():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_ipc_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    t = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    sd, blocks, feats, labels, part, params = _case()
    og, ol = oracle.step(DIMS, "mean", False, blocks, part, K, list(range(K)), params, feats, labels, 1.0 / len(sd))
    assert_grad_close(t[:-1], og, DIMS, "mean", 1e-5, "2 ranks, IPC-mapped shards")
    assert t[-1] == pytest.approx(ol, rel=1e-5)
