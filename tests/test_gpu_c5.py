"""C5: the ogbn-papers100M-shaped configuration (BASELINE.json configs[4]):
3-layer SAGE-mean [128, 256, 256, 172], fanout (5, 10, 15), 1.2 M outputs, K = 32, on a 111 M-node /
1.6 B-entry graph whose feature table (57 GB fp32) is generated in row chunks straight into HBM.

* Scaled C5 (same shape, 1/500 of the nodes, pairs, outputs and communities): the fused step over
  launch groups smaller than K (ragged last group) against the float64 oracle, and Betty's
  invariant (the K = 8 step equals the K = 1 step) on the GPU.
* Full size (opt-in: BETTY_C5_FULL=1, ~4 min of generation and ~150 GB of HBM): in the bench's
  launch configuration (multilevel REG partition, K = 32, the launch group create_plan picks),
  every micro-batch of the first launch group bit-exact against the oracle's extraction, and a
  sampled micro-batch through the fused step against the oracle on its own feature rows.
"""
import os

import numpy as np
import pytest
import torch

import oracle
import synth
from tests.helpers import assert_close, assert_grad_close

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
def c5s(B, ctx):
    cfg = synth.scaled(synth.CONFIGS["C5"], 0.002)
    ds = synth.make(cfg)
    dev = B.blocks_to_device(ds.blocks)
    K = 8
    ip, col, w = B.betty_reg_build(ctx, dev[-1])
    part = B.betty_reg_partition(ip.cpu().numpy(), col.cpu().numpy(), w.cpu().numpy(), K, method="multilevel")
    params = synth.init_params(cfg.dims, cfg.aggr, seed=cfg.seeds["init"])
    want = oracle.step(cfg.dims, cfg.aggr, True, ds.blocks, part, K, list(range(K)), params, ds.feats, ds.labels,
                       1.0 / cfg.n_out)
    return cfg, ds, dev, part, K, params, want


def _step(B, ctx, plan, cfg, P, X, Y):
    grad = torch.zeros_like(P)
    loss = torch.zeros(1, device="cuda")
    B.betty_step(ctx, plan, P, X, Y, 1.0 / cfg.n_out, grad, loss)
    B.betty_sync_check(ctx)
    return grad.cpu().numpy().astype(np.float64), loss.item()


@pytest.mark.parametrize("group", [3, 0])
def test_c5_scaled_step_vs_oracle(B, ctx, c5s, group):
    """All 8 micro-batches in launch groups of 3 (3 + 3 + 2) or one group, bf16 GEMM mode, against
    oracle_step (reading #17: bf16-rounded GEMM operands) within 2e-2; the feature table goes
    through the chunked device path (chunks of 100 k rows, 256-byte rows)."""
    cfg, ds, dev, part, K, params, (og, ol) = c5s
    assert ds.feats is not None
    no_host = synth.Dataset(cfg, ds.graph, None, ds.labels, ds.seeds, ds.blocks)
    X = synth.features_device(cfg, no_host, True, 256, "cuda", chunk_rows=100_000)
    assert X.shape == (cfg.n, 128) and X.dtype == torch.bfloat16
    np.testing.assert_array_equal(X.float().cpu().numpy(),
                                  torch.as_tensor(ds.feats).to(torch.bfloat16).float().numpy())
    model = B.Model(cfg.dims, cfg.aggr, "bf16", "bf16")
    plan = B.betty_plan_create(ctx, model, dev, torch.as_tensor(part).cuda(), K, list(range(K)), group=group,
                               flags=B.PLAN_GRAPH | B.PLAN_REG)
    assert plan.info()["n_groups"] == (3 if group == 3 else 1)
    P = torch.as_tensor(params).cuda()
    Y = torch.as_tensor(ds.labels).cuda()
    for rep in range(2):          # graph replay: the second step re-extracts into the same arenas
        g, l = _step(B, ctx, plan, cfg, P, X, Y)
        assert_grad_close(g, og, cfg.dims, cfg.aggr, 2e-2, f"grad rep {rep}")
        assert l == pytest.approx(ol, rel=2e-2)
    plan.free()


def test_c5_scaled_invariant(B, ctx, c5s):
    """Sum of the K = 8 micro-batch gradients == the full-batch gradient (fp32, 1e-5), on the GPU."""
    cfg, ds, dev, part, K, params, _ = c5s
    P = torch.as_tensor(params).cuda()
    X = torch.as_tensor(ds.feats).cuda()
    Y = torch.as_tensor(ds.labels).cuda()
    model = B.Model(cfg.dims, cfg.aggr, "fp32", "fp32")
    res = []
    for k, p, grp in ((K, part, 3), (1, np.zeros(cfg.n_out, np.int32), 0)):
        plan = B.betty_plan_create(ctx, model, dev, torch.as_tensor(p).cuda(), k, list(range(k)), group=grp,
                                   flags=B.PLAN_GRAPH)
        res.append(_step(B, ctx, plan, cfg, P, X, Y))
        plan.free()
    assert_grad_close(res[0][0], res[1][0], cfg.dims, cfg.aggr, 1e-5, "sum of micro-batch gradients vs full batch")
    assert res[0][1] == pytest.approx(res[1][1], rel=1e-5)


# ----------------------------------------------- C5 at 1/50: the feature table exceeds L2
@pytest.fixture(scope="module")
def c5m(B, ctx):
    """C5's shape at 1/50 (2.2 M nodes, 16 M pairs, 24 k outputs): the bf16 table (570 MB) and the
    fp32 table (1.1 GB) are several times the 126 MB L2, so the layer-0 gathers stream from HBM as
    in the full-size run."""
    cfg = synth.scaled(synth.CONFIGS["C5"], 0.02)
    ds = synth.make(cfg)
    dev = B.blocks_to_device(ds.blocks)
    ip, col, w = B.betty_reg_build(ctx, dev[-1])
    part = B.betty_reg_partition(ip.cpu().numpy(), col.cpu().numpy(), w.cpu().numpy(), 8, method="multilevel")
    return cfg, ds, dev, part


@pytest.mark.parametrize("mode,rtol", [("bf16", 2e-2), ("fp32", 1e-5)])
def test_c5_beyond_l2_sampled_micro_batch(B, ctx, c5m, mode, rtol):
    """24 outputs of micro-batch 0 as their own micro-batch through the fused step, on the whole
    > L2 feature table, against the float64 oracle (per tensor, reading #18)."""
    cfg, ds, dev, part = c5m
    assert ds.feats.nbytes > 4 * 126 * 2 ** 20
    idx = np.nonzero(part == 0)[0][:24]
    p2 = np.ones(cfg.n_out, np.int32)
    p2[idx] = 0
    params = synth.init_params(cfg.dims, cfg.aggr, seed=cfg.seeds["init"])
    og, ol = oracle.step(cfg.dims, cfg.aggr, mode == "bf16", ds.blocks, p2, 2, [0], params, ds.feats, ds.labels,
                         1.0 / cfg.n_out)
    model = B.Model(cfg.dims, cfg.aggr, mode, mode)
    plan = B.betty_plan_create(ctx, model, dev, torch.as_tensor(p2).cuda(), 2, [0], group=0,
                               flags=B.PLAN_GRAPH | B.PLAN_REG)
    X = torch.as_tensor(ds.feats).cuda()
    if mode == "bf16":
        X = X.to(torch.bfloat16).contiguous()
    P = torch.as_tensor(params).cuda()
    Y = torch.as_tensor(ds.labels).cuda()
    g, l = _step(B, ctx, plan, cfg, P, X, Y)
    assert_grad_close(g, og, cfg.dims, cfg.aggr, rtol, f"{mode} grad")
    assert l == pytest.approx(ol, rel=rtol)
    plan.free()


def test_c5_beyond_l2_invariant(B, ctx, c5m):
    """Betty's invariant on the > L2 table: the K = 8 step (launch groups of 3) equals the K = 1 step
    (fp32, 1e-5 per tensor)."""
    cfg, ds, dev, part = c5m
    params = synth.init_params(cfg.dims, cfg.aggr, seed=cfg.seeds["init"])
    P = torch.as_tensor(params).cuda()
    X = torch.as_tensor(ds.feats).cuda()
    Y = torch.as_tensor(ds.labels).cuda()
    model = B.Model(cfg.dims, cfg.aggr, "fp32", "fp32")
    res = []
    for k, p, grp in ((8, part, 3), (1, np.zeros(cfg.n_out, np.int32), 0)):
        plan = B.betty_plan_create(ctx, model, dev, torch.as_tensor(p).cuda(), k, list(range(k)), group=grp,
                                   flags=B.PLAN_GRAPH)
        res.append(_step(B, ctx, plan, cfg, P, X, Y))
        plan.free()
    assert_grad_close(res[0][0], res[1][0], cfg.dims, cfg.aggr, 1e-5, "K=8 vs K=1")
    assert res[0][1] == pytest.approx(res[1][1], rel=1e-5)


# ------------------------------------------------------------------ full size (opt-in)
full = pytest.mark.skipif(os.environ.get("BETTY_C5_FULL", "0") != "1",
                          reason="full-size C5 (~4 min, ~150 GB HBM): set BETTY_C5_FULL=1")
K_FULL = 32


@pytest.fixture(scope="module")
def c5(B, ctx):
    cfg = synth.CONFIGS["C5"]
    ds = synth.make(cfg, with_features=None)
    assert ds.feats is None
    dev = B.blocks_to_device(ds.blocks)
    ip, col, w = B.betty_reg_build(ctx, dev[-1])
    part = B.betty_reg_partition(ip.cpu().numpy(), col.cpu().numpy(), w.cpu().numpy(), K_FULL, method="multilevel")
    return cfg, ds, dev, part


@full
def test_c5_full_extraction(B, ctx, c5):
    """The first launch group of the bench's configuration: every micro-batch bit-exact (CSR, src_pos,
    src_gid of all 3 layers) against oracle_extract, in the group layout (DESIGN.md §3 row G)."""
    import bench
    cfg, ds, dev, part = c5
    model = B.Model(cfg.dims, cfg.aggr, "bf16", "bf16")
    X = synth.features_device(cfg, ds, True, 256, "cuda")     # the bench's memory picture
    plan, group = bench.create_plan(B, ctx, model, dev, torch.as_tensor(part).cuda(), K_FULL, list(range(K_FULL)),
                                    0, B.PLAN_GRAPH | B.PLAN_REG)
    ks = list(range(K_FULL if group == 0 else group))
    got = [{k: (v.cpu().numpy() if isinstance(v, torch.Tensor) else v) for k, v in vars(b).items()}
           for b in plan.group_blocks(0)]
    plan.free()
    del X
    L = cfg.L
    mbs = [oracle.extract(ds.blocks, part, K_FULL, k) for k in ks]
    n_out = [mb[L - 1].n_dst for mb in mbs]
    out_off = np.concatenate([[0], np.cumsum(n_out)])
    dst_map = [out_off[j] + np.arange(n_out[j]) for j in range(len(ks))]
    for l in range(L - 1, -1, -1):
        g = got[l]
        n_dst_g = sum(len(m) for m in dst_map)
        new = [mbs[j][l].n_src - mbs[j][l].n_dst for j in range(len(ks))]
        new_off = n_dst_g + np.concatenate([[0], np.cumsum(new)])
        src_map = [np.concatenate([dst_map[j], new_off[j] + np.arange(new[j])]).astype(np.int64)
                   for j in range(len(ks))]
        assert g["n_dst"] == n_dst_g and g["n_src"] == new_off[-1], l
        for j in range(len(ks)):
            m = mbs[j][l]
            rows = dst_map[j]
            b, e = g["indptr"][rows], g["indptr"][rows + 1]
            np.testing.assert_array_equal(e - b, np.diff(m.indptr), err_msg=f"layer {l} mb {j} degrees")
            lens = e - b
            gi = np.repeat(b - np.concatenate([[0], np.cumsum(lens)[:-1]]), lens) + np.arange(lens.sum())
            np.testing.assert_array_equal(g["indices"][gi], src_map[j][m.indices], err_msg=f"layer {l} mb {j} idx")
            np.testing.assert_array_equal(g["src_pos"][src_map[j]], m.src_pos, err_msg=f"layer {l} mb {j} src_pos")
            np.testing.assert_array_equal(g["src_gid"][src_map[j]], m.src_gid, err_msg=f"layer {l} mb {j} src_gid")
        dst_map = src_map


@full
def test_c5_full_sampled_micro_batch(B, ctx, c5):
    """16 outputs of micro-batch 0 as their own micro-batch through the fused step on the full-size
    graph and the full 111 M-row bf16 table in HBM, against the float64 oracle fed only the feature
    rows that micro-batch reads (synth.features_rows)."""
    import bench
    cfg, ds, dev, part = c5
    idx = np.nonzero(part == 0)[0][:16]
    p2 = np.ones(cfg.n_out, np.int32)
    p2[idx] = 0
    oblocks, ofeats = bench.oracle_inputs(cfg, ds, p2)
    params = synth.init_params(cfg.dims, cfg.aggr, seed=cfg.seeds["init"])
    og, ol = oracle.step(cfg.dims, cfg.aggr, True, oblocks, p2, 2, [0], params, ofeats, ds.labels, 1.0 / cfg.n_out)
    model = B.Model(cfg.dims, cfg.aggr, "bf16", "bf16")
    plan = B.betty_plan_create(ctx, model, dev, torch.as_tensor(p2).cuda(), 2, [0], group=0,
                               flags=B.PLAN_GRAPH | B.PLAN_REG)
    X = synth.features_device(cfg, ds, True, 256, "cuda")
    P = torch.as_tensor(params).cuda()
    Y = torch.as_tensor(ds.labels).cuda()
    g, l = _step(B, ctx, plan, cfg, P, X, Y)
    assert_grad_close(g, og, cfg.dims, cfg.aggr, 2e-2, "grad")
    assert l == pytest.approx(ol, rel=2e-2)
    plan.free()
