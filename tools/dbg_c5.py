"""Debug the C5 plan memory (run under gpurun): generate (or load a /tmp cache of) C5, then plan with
group 1 and report memory / errors at each stage."""
import os, sys, time, pickle
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth
import paper_conf_asplos_yangzd023_b200 as B

cfg = synth.CONFIGS["C5"]
cache = "/tmp/c5_ds.pkl"
t0 = time.time()
if os.path.exists(cache):
    with open(cache, "rb") as f:
        ds = pickle.load(f)
else:
    ds = synth.make(cfg, with_features=None)
    ds.graph.indptr = None; ds.graph.indices = None
    with open(cache, "wb") as f:
        pickle.dump(ds, f, protocol=4)
print("data", time.time() - t0, [(b.n_dst, b.n_src, b.n_edges) for b in ds.blocks], flush=True)
ctx = B.betty_ctx_create(0)
dev = B.blocks_to_device(ds.blocks)
print("blocks on device; free GB", torch.cuda.mem_get_info()[0] / 2**30, flush=True)
K = int(os.environ.get("K", "32"))
part = synth.range_partition(cfg.n_out, K)
dpart = torch.as_tensor(part).cuda()
sz = B.betty_mb_sizes(ctx, dev, dpart, K)
print("mb sizes k=0", sz[0].tolist(), "sum E", sz[:, :, 2].sum(), flush=True)
model = B.Model(cfg.dims, cfg.aggr, "bf16", "bf16")
for g in [int(x) for x in os.environ.get("GRP", "1").split(",")]:
    try:
        p = B.betty_plan_create(ctx, model, dev, dpart, K, list(range(K)), group=g,
                                flags=B.PLAN_GRAPH | B.PLAN_REG)
        print("group", g, "ok arena GB", p.info()["arena_bytes"] / 2**30, "free GB", torch.cuda.mem_get_info()[0] / 2**30, flush=True)
        p.free()
    except Exception as e:
        print("group", g, "failed:", e, "free GB", torch.cuda.mem_get_info()[0] / 2**30, flush=True)
    torch.cuda.synchronize(); torch.cuda.empty_cache()
