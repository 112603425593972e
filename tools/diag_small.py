"""Per-tensor gradient errors of small fused steps against the oracle (diagnostic, GPU box).
Usage: python tools/diag_small.py [mode] ; env BETTY_FP32_SIMT=1 for the SIMT fp32 path."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import oracle, synth
import paper_conf_asplos_yangzd023_b200 as B
from tests.helpers import param_tensors, rel_err, tiny

mode = sys.argv[1] if len(sys.argv) > 1 else "fp32"
ctx = B.betty_ctx_create(0)
for name, aggr, fan, dims in [("mean2", "mean", (3, 4), [20, 32, 5]), ("wide", "mean", (5, 8), [100, 256, 47]),
                              ("mean3", "mean", (3, 3, 4), [24, 40, 40, 6]), ("pool2", "pool", (3, 4), [16, 24, 5])]:
    F = dims[0]
    ld = (F + 7) // 8 * 8
    g, sd, blocks, feats, _ = tiny(n=600, pairs=2400, fanouts=fan, n_out=60, F=F, C=dims[-1], seed=2, ld=ld)
    labels = (np.arange(600) * 5 % dims[-1]).astype(np.int32)
    params = synth.init_params(dims, aggr, seed=2)
    K = 3
    part = synth.random_partition(len(sd), K, 11)
    dev = B.blocks_to_device(blocks)
    model = B.Model(dims, aggr, mode, mode)
    plan = B.betty_plan_create(ctx, model, dev, torch.as_tensor(part).cuda(), K, [0, 1, 2], group=0, flags=0)
    P = torch.as_tensor(params).cuda()
    X = torch.as_tensor(feats).cuda()
    if mode == "bf16":
        X = X.to(torch.bfloat16).contiguous()
    grad = torch.zeros_like(P)
    loss = torch.zeros(1, device="cuda")
    B.betty_step(ctx, plan, P, X, torch.as_tensor(labels).cuda(), 1.0 / len(sd), grad, loss)
    B.betty_sync_check(ctx)
    og, ol = oracle.step(dims, aggr, mode == "bf16", blocks, part, K, [0, 1, 2], params, feats, labels, 1.0 / len(sd))
    print(name, "loss", loss.item(), ol)
    for (n, a), (_, b) in zip(param_tensors(grad.cpu().numpy(), dims, aggr), param_tensors(og, dims, aggr)):
        print(f"   {n}: rel {rel_err(a, b):.3e} |gpu| {np.linalg.norm(a):.3e} |ref| {np.linalg.norm(b):.3e}")
    plan.free()
