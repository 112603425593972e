"""The multi-rank CUDA path on one GPU: two processes on cuda:0, gloo for the
collective, each running libbetty's fused step (plan + betty_step, CUDA graph, in-step REG on its
row share) over its LPT share of the K micro-batches; the all-reduced gradient and loss must equal
the oracle's step over ALL K micro-batches (Betty's invariant across ranks), per
parameter tensor (reading #18): 1e-5 in fp32 (3xTF32 GEMMs), 2e-2 in bf16."""
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
K = 7


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _case():
    g, sd, blocks, feats, _ = tiny(n=900, pairs=4000, fanouts=(4, 6), n_out=90, F=DIMS[0], C=DIMS[-1], seed=21,
                                   ld=24)
    labels = (np.arange(900) * 3 % DIMS[-1]).astype(np.int32)
    part = synth.random_partition(len(sd), K, 4)
    params = synth.init_params(DIMS, "mean", seed=6)
    return sd, blocks, feats, labels, part, params


def _worker(rank, world, port, mode, q):
    import torch.distributed as dist
    import paper_conf_asplos_yangzd023_b200 as B
    from paper_conf_asplos_yangzd023_b200.dist import allreduce_grad, lpt_assign, plan_costs, reg_rows
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    sd, blocks, feats, labels, part, params = _case()
    ctx = B.betty_ctx_create(0)
    dev = B.blocks_to_device(blocks)
    dpart = torch.as_tensor(part).cuda()
    mine = lpt_assign(plan_costs(B.betty_mb_sizes(ctx, dev, dpart, K), DIMS), world)[rank]
    model = B.Model(DIMS, "mean", mode, mode)
    plan = B.betty_plan_create(ctx, model, dev, dpart, K, mine, group=0, flags=B.PLAN_GRAPH | B.PLAN_REG)
    plan.set_reg_rows(*reg_rows(len(sd), rank, world))
    P = torch.as_tensor(params).cuda()
    X = torch.as_tensor(feats).cuda()
    if mode == "bf16":
        X = X.to(torch.bfloat16).contiguous()
    Y = torch.as_tensor(labels).cuda()
    out = []
    for rep in range(2):                    # graph capture, then replay
        grad = torch.zeros_like(P)
        loss = torch.zeros(1, device="cuda")
        B.betty_step(ctx, plan, P, X, Y, 1.0 / len(sd), grad, loss)
        B.betty_sync_check(ctx)
        t = torch.cat([grad, loss]).double()
        allreduce_grad(t)
        out.append(t.cpu().numpy())
    shares = [None] * world
    dist.all_gather_object(shares, mine)
    plan.free()
    if rank == 0:
        q.put((out, shares))
    dist.destroy_process_group()


@pytest.mark.parametrize("mode,rtol", [("fp32", 1e-5), ("bf16", 2e-2)])
def test_two_ranks_all_reduce_equals_oracle_over_all_micro_batches(mode, rtol):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, mode, q)) for r in range(2)]
    for p in procs:
        p.start()
    out, shares = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert sorted(k for s in shares for k in s) == list(range(K)) and all(len(s) > 0 for s in shares)
    sd, blocks, feats, labels, part, params = _case()
    og, ol = oracle.step(DIMS, "mean", mode == "bf16", blocks, part, K, list(range(K)), params, feats, labels,
                         1.0 / len(sd))
    for rep, t in enumerate(out):
        assert_grad_close(t[:-1], og, DIMS, "mean", rtol, f"2 ranks {mode} rep {rep}")
        assert t[-1] == pytest.approx(ol, rel=rtol)
