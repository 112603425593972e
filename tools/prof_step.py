"""One bench step under a profiler window (cudaProfilerStart/Stop), for
`ncu --profile-from-start off`.  Same workload and plan as bench.py (C3,
K=32, REG partition, bf16 mode, all micro-batches in one group), without the
CUDA graph so every kernel is a separate launch ncu can replay.

    ncu --profile-from-start off --set full ... python tools/prof_step.py [--config C3] [--K 32]
"""
import argparse
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402
import paper_conf_asplos_yangzd023_b200 as B  # noqa: E402


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--config", default="C3")
    p.add_argument("--K", type=int, default=32)
    p.add_argument("--mode", default="bf16")
    p.add_argument("--graph", action="store_true")
    p.add_argument("--steps", type=int, default=1)
    p.add_argument("--scale", type=float, default=1.0)
    p.add_argument("--group", type=int, default=0)
    p.add_argument("--feat-align", type=int, default=256)
    p.add_argument("--sim-world", type=int, default=1, help="rank 0's share of an N-rank job")
    p.add_argument("--fresh", action="store_true", help="BETTY_PLAN_FRESH plan (the e2e path's step)")
    a = p.parse_args()
    cfg = synth.CONFIGS[a.config]
    if a.scale != 1.0:
        cfg = synth.scaled(cfg, a.scale)
    ds = synth.make(cfg, with_features=None)
    ctx = B.betty_ctx_create(0)
    dev = B.blocks_to_device(ds.blocks)
    ip, col, w = B.betty_reg_build(ctx, dev[-1])
    part = B.betty_reg_partition(ip.cpu().numpy(), col.cpu().numpy(), w.cpu().numpy(), a.K, method="multilevel")
    dpart = torch.as_tensor(part).cuda()
    feats = synth.features_device(cfg, ds, a.mode == "bf16", a.feat_align, "cuda")
    labels = torch.as_tensor(ds.labels).cuda()
    model = B.Model(cfg.dims, cfg.aggr, a.mode, a.mode)
    params = torch.as_tensor(synth.init_params(cfg.dims, cfg.aggr, seed=cfg.seeds["init"])).cuda()
    grad = torch.zeros_like(params)
    loss = torch.zeros(1, device="cuda")
    flags = B.PLAN_REG | (B.PLAN_GRAPH if a.graph else 0) | (B.PLAN_FRESH if a.fresh else 0)
    from paper_conf_asplos_yangzd023_b200.dist import lpt_assign, micro_batch_costs, reg_rows
    my_k = lpt_assign(micro_batch_costs(part, a.K, ds.blocks[-1].indptr), a.sim_world)[0]
    plan = B.betty_plan_create(ctx, model, dev, dpart, a.K, my_k, group=a.group, flags=flags)
    if a.sim_world > 1:
        plan.set_reg_rows(*reg_rows(cfg.n_out, 0, a.sim_world))
    B.betty_step(ctx, plan, params, feats, labels, 1.0 / cfg.n_out, grad, loss)
    B.betty_sync_check(ctx)
    torch.cuda.synchronize()
    torch.cuda.profiler.start()
    for _ in range(a.steps):
        B.betty_step(ctx, plan, params, feats, labels, 1.0 / cfg.n_out, grad, loss)
    torch.cuda.synchronize()
    torch.cuda.profiler.stop()
    B.betty_sync_check(ctx)
    info = plan.info()
    print("prof_step ok", info["kernels_per_step"], "kernels/step; edges", info["edges"], "n_src", info["n_src"],
          "n_dst", info["n_dst"])
    plan.free()


if __name__ == "__main__":
    main()
