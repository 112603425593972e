"""Run-to-run determinism of the fused step: the row GEMMs claim their tiles from a
global counter (which CTA computes which rows changes from run to run, and with the REG rebuild on the
side stream holding SMs), the aggregation and extraction claim rows dynamically, the scans exchange
chunk aggregates through flags -- yet every output element is produced by one thread in a fixed
arithmetic order and every reduction (dW partials, loss partials, CSC gathers) sums in a fixed order,
so repeated steps on the same inputs must give bit-identical gradients and losses.  A C3-shaped graph
at 1/20 scale: its layer-0 GEMMs have hundreds of 128-row tiles over the 148 CTAs."""
import numpy as np
import pytest
import torch

import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def B():
    import paper_conf_asplos_yangzd023_b200 as B
    assert torch.cuda.is_available()
    return B


@pytest.fixture(scope="module")
def ctx(B):
    return B.betty_ctx_create(0)


@pytest.fixture(scope="module")
def case():
    cfg = synth.scaled(synth.CONFIGS["C3"], 0.05)
    ds = synth.make(cfg)
    return cfg, ds


@pytest.mark.parametrize("mode", ["bf16", "fp32"])
def test_fused_step_is_bitwise_repeatable(B, ctx, case, mode):
    cfg, ds = case
    K = 8
    dev = B.blocks_to_device(ds.blocks)
    part = torch.as_tensor(synth.random_partition(cfg.n_out, K, 5)).cuda()
    model = B.Model(cfg.dims, cfg.aggr, mode, mode)
    P = torch.as_tensor(synth.init_params(cfg.dims, cfg.aggr)).cuda()
    X = torch.as_tensor(ds.feats).cuda()
    if mode == "bf16":
        X = X.to(torch.bfloat16).contiguous()
    Y = torch.as_tensor(ds.labels).cuda()
    plan = B.betty_plan_create(ctx, model, dev, part, K, list(range(K)), group=0,
                               flags=B.PLAN_GRAPH | B.PLAN_REG)
    assert plan.info()["n_dst"][0] > 64 * 128        # many row tiles per GEMM CTA
    grads, losses = [], []
    for _ in range(4):
        grad = torch.zeros_like(P)
        loss = torch.zeros(1, device="cuda")
        B.betty_step(ctx, plan, P, X, Y, 1.0 / cfg.n_out, grad, loss)
        B.betty_sync_check(ctx)
        grads.append(grad.cpu().numpy())
        losses.append(loss.item())
    plan.free()
    assert np.isfinite(grads[0]).all() and np.abs(grads[0]).max() > 0
    for r in range(1, 4):
        np.testing.assert_array_equal(grads[r], grads[0], err_msg=f"{mode} run {r}")
        assert losses[r] == losses[0]
