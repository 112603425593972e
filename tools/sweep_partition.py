"""Partition quality and Betty's memory mode on one B200, one process (C3 generated once).

Part 1 (PAPER.md:1222-1239 / 1733-1743, Fig. 16): for the REG partition (multilevel)
and the paper's redundancy-unaware baselines (Metis on the raw graph, random, range) at K = 8..64:
epoch time of the fused step (bf16, all micro-batches in one launch group, CUDA graph, REG in the
step), the sum over micro-batches of layer-0 inputs (redundancy vs the full batch) and of edges.
Part 2 (Table 6 memory column): the REG partition at K = 32 with launch groups of
c = 1 (the paper's sequential micro-batches), 4, 8 and all 32: epoch time and the plan's device arena.

    python tools/sweep_partition.py [--steps 20] > profiles/r02_sweep_partition.txt
"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
import paper_conf_asplos_yangzd023_b200 as B
from paper_conf_asplos_yangzd023_b200.partition import raw_graph_partition


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--Ks", default="8,16,32,64")
    ap.add_argument("--mode", default="bf16")
    a = ap.parse_args()
    cfg = synth.CONFIGS["C3"]
    t0 = time.time()
    ds = synth.make(cfg, with_features=None)
    ctx = B.betty_ctx_create(0)
    dev = B.blocks_to_device(ds.blocks)
    feats = synth.features_device(cfg, ds, a.mode == "bf16", 256, "cuda")
    labels = torch.as_tensor(ds.labels).cuda()
    params = torch.as_tensor(synth.init_params(cfg.dims, cfg.aggr, seed=cfg.seeds["init"])).cuda()
    model = B.Model(cfg.dims, cfg.aggr, a.mode, a.mode)
    ip, col, w = B.betty_reg_build(ctx, dev[-1])
    reg = (ip.cpu().numpy(), col.cpu().numpy(), w.cpu().numpy())
    full_src0, full_e = ds.blocks[0].n_src, sum(b.n_edges for b in ds.blocks)
    print(f"# C3 products-shaped ({cfg.n} nodes, {cfg.n_out} outputs), {a.mode}, generated in {time.time() - t0:.0f} s")
    print(f"# full batch: layer-0 inputs {full_src0}, edges {full_e}")

    def run(part, K, group):
        plan = B.betty_plan_create(ctx, model, dev, torch.as_tensor(part).cuda(), K, list(range(K)), group=group,
                                   flags=B.PLAN_GRAPH | B.PLAN_REG)
        grad = torch.zeros_like(params)
        loss = torch.zeros(1, device="cuda")
        for _ in range(3):
            B.betty_step(ctx, plan, params, feats, labels, 1.0 / cfg.n_out, grad, loss)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(a.steps):
            B.betty_step(ctx, plan, params, feats, labels, 1.0 / cfg.n_out, grad, loss)
        e1.record()
        torch.cuda.synchronize()
        B.betty_sync_check(ctx)
        info = plan.info()
        plan.free()
        return e0.elapsed_time(e1) / a.steps, info

    print("\n## partition quality (launch group = all micro-batches)")
    print(f"{'partition':>10} {'K':>3} {'ms/step':>8} {'sum L0 inputs':>14} {'redund.':>8} {'sum edges':>11} {'x full':>7} "
          f"{'G edges/s':>9}")
    for K in [int(x) for x in a.Ks.split(",")]:
        parts = {"reg": B.betty_reg_partition(*reg, K, method="multilevel"),
                 "metis-raw": raw_graph_partition(ds.graph.indptr, ds.graph.indices, ds.seeds, K),
                 "random": synth.random_partition(cfg.n_out, K, cfg.seeds["part"]),
                 "range": synth.range_partition(cfg.n_out, K)}
        for name, part in parts.items():
            ms, info = run(part, K, 0)
            e = sum(info["edges"])
            print(f"{name:>10} {K:>3} {ms:8.3f} {info['n_src'][0]:>14} {info['n_src'][0] / full_src0:8.2f} {e:>11} "
                  f"{e / full_e:7.2f} {e / ms / 1e6:9.2f}", flush=True)

    print("\n## Betty's memory mode: REG partition, K = 32, launch group c (c = 1: one micro-batch at a time)")
    print(f"{'c':>3} {'ms/step':>8} {'plan arena GB':>14}")
    part = B.betty_reg_partition(*reg, 32, method="multilevel")
    for c in (1, 4, 8, 32):
        ms, info = run(part, 32, c)
        print(f"{c:>3} {ms:8.3f} {info['arena_bytes'] / 2 ** 30:14.2f}", flush=True)


if __name__ == "__main__":
    main()
