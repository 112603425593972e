"""Per-tensor error of one whole C3 micro-batch (K=32 REG partition, micro-batch 0) against the
oracle, fp32 and bf16, through betty_step; prints one line per tensor.  Diagnostic (GPU box)."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import oracle, synth
import paper_conf_asplos_yangzd023_b200 as B
from tests.helpers import param_tensors, rel_err

cfg = synth.CONFIGS[os.environ.get("CFG", "C3")]
ds = synth.make(cfg)
ctx = B.betty_ctx_create(0)
dev = B.blocks_to_device(ds.blocks)
ip, col, w = B.betty_reg_build(ctx, dev[-1])
K = 32
part = B.betty_reg_partition(ip.cpu().numpy(), col.cpu().numpy(), w.cpu().numpy(), K, method="multilevel")
params = synth.init_params(cfg.dims, cfg.aggr, seed=cfg.seeds["init"])
modes = sys.argv[1:] or ["fp32", "bf16"]
for mode in modes:
    t = time.time()
    og, ol = oracle.step(cfg.dims, cfg.aggr, mode == "bf16", ds.blocks, part, K, [0], params, ds.feats, ds.labels,
                         1.0 / cfg.n_out)
    print(f"oracle {mode} {time.time() - t:.1f}s", flush=True)
    model = B.Model(cfg.dims, cfg.aggr, mode, mode)
    plan = B.betty_plan_create(ctx, model, dev, torch.as_tensor(part).cuda(), K, [0], group=0,
                               flags=B.PLAN_GRAPH | B.PLAN_REG)
    P = torch.as_tensor(params).cuda()
    X = torch.as_tensor(ds.feats).cuda()
    if mode == "bf16":
        X = X.to(torch.bfloat16).contiguous()
    Y = torch.as_tensor(ds.labels).cuda()
    grad = torch.zeros_like(P)
    loss = torch.zeros(1, device="cuda")
    B.betty_step(ctx, plan, P, X, Y, 1.0 / cfg.n_out, grad, loss)
    B.betty_sync_check(ctx)
    g = grad.cpu().numpy()
    print(f"{mode} info {plan.info()['n_dst']} {plan.info()['edges']} loss rel {abs(loss.item() - ol) / abs(ol):.2e}")
    for (n, a), (_, b) in zip(param_tensors(g, cfg.dims, cfg.aggr), param_tensors(og, cfg.dims, cfg.aggr)):
        d = np.abs(a - b)
        i = np.unravel_index(np.argmax(d), d.shape)
        print(f"  {mode} {n}: rel l2 {rel_err(a, b):.3e}  max {d.max() / np.abs(b).max():.3e} at {i} "
              f"(gpu {a[i]:.6e} ref {b[i]:.6e})", flush=True)
    plan.free()
