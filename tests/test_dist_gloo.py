"""Multi-rank host logic on CPU (gloo, world_size 2): LPT assignment of
micro-batches to ranks + one all-reduce of the accumulated gradient gives the
full-batch gradient (the oracle computes each rank's share)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_asplos_yangzd023_b200.dist import allreduce_grad, lpt_assign, micro_batch_costs, reg_rows
from tests.helpers import tiny

DIMS = [6, 10, 4]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g, sd, blocks, feats, labels = tiny(n=300, pairs=1000, fanouts=(3, 4), n_out=40, F=6, C=4, seed=9)
    K = 7
    part = synth.random_partition(len(sd), K, 5)
    mine = lpt_assign(micro_batch_costs(part, K, blocks[-1].indptr), world)[rank]
    params = synth.init_params(DIMS, "mean", seed=1).astype(np.float64)
    grad, loss = oracle.step(DIMS, "mean", False, blocks, part, K, mine, params, feats, labels, 1.0 / len(sd))
    t = torch.tensor(np.concatenate([grad, [loss]]))
    allreduce_grad(t)
    # row-sharded REG: each rank's share of the rows, gathered, is the whole REG
    rp, rc, rw = oracle.reg(blocks[-1].n_src, blocks[-1].indptr, blocks[-1].nbr_pos)
    r0, r1 = reg_rows(len(sd), rank, world)
    shares = [None] * world
    dist.all_gather_object(shares, (r0, r1, rp[r0:r1 + 1] - rp[r0], rc[rp[r0]:rp[r1]], rw[rp[r0]:rp[r1]]))
    if rank == 0:
        full, lfull, _ = oracle.sage(DIMS, "mean", False, blocks, params, feats, labels, 1.0 / len(sd))
        assert [s_[0] for s_ in shares] == [0, shares[0][1]] and shares[-1][1] == len(sd)
        ip = np.concatenate([[0]] + [s_[2][1:] + off for s_, off in
                                     zip(shares, np.cumsum([0] + [s_[2][-1] for s_ in shares[:-1]]))])
        np.testing.assert_array_equal(ip, rp)
        np.testing.assert_array_equal(np.concatenate([s_[3] for s_ in shares]), rc)
        np.testing.assert_array_equal(np.concatenate([s_[4] for s_ in shares]), rw)
        q.put((t.numpy(), full, lfull, mine))
    dist.destroy_process_group()


def test_lpt_assign_properties():
    costs = [5, 1, 9, 3, 3, 7, 2]
    a = lpt_assign(costs, 3)
    assert sorted(k for r in a for k in r) == list(range(7))
    loads = [sum(costs[k] for k in r) for r in a]
    assert max(loads) - min(loads) <= max(costs)
    assert lpt_assign(costs, 3) == a                       # deterministic
    assert lpt_assign(costs, 1) == [list(range(7))]


def test_reg_rows_cover_every_row_once():
    for n in (0, 1, 7, 120, 196615):
        for world in (1, 2, 3, 8):
            shares = [reg_rows(n, r, world) for r in range(world)]
            assert shares[0][0] == 0 and shares[-1][1] == n
            assert all(a[1] == b[0] for a, b in zip(shares, shares[1:]))
            assert max(b - a for a, b in shares) - min(b - a for a, b in shares) <= 1


def test_two_rank_allreduce_equals_full_batch():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    red, full, lfull, mine = q.get(timeout=120)
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert np.linalg.norm(red[:-1] - full) <= 1e-12 * np.linalg.norm(full)
    assert abs(red[-1] - lfull) <= 1e-12 * abs(lfull)


def test_plan_costs_closed_form():
    """cost_k = sum_l (E_{k,l} F_l + gamma n_dst,k,l F_l F_{l+1})."""
    from paper_conf_asplos_yangzd023_b200.dist import plan_costs
    sizes = np.array([[[10, 20, 100], [2, 10, 30]], [[5, 9, 40], [1, 5, 8]]])
    dims = [24, 48, 5]
    g = 0.5
    want = [100 * 24 + g * 10 * 24 * 48 + 30 * 48 + g * 2 * 48 * 5, 40 * 24 + g * 5 * 24 * 48 + 8 * 48 + g * 1 * 48 * 5]
    np.testing.assert_allclose(plan_costs(sizes, dims, gamma=g), want)
