#!/usr/bin/env python
"""bench.py -- Betty's micro-batch GNN training step on B200 (the metric of
BASELINE.json: epoch time & aggregated edges/s, SAGE, products-shape).

One step (= one epoch of the paper, Table 6 "training time per epoch",
PAPER.md:1668-1679) is the whole hot path over one batch: the REG rebuild
(a1), extraction of every micro-batch (a2), SAGE forward (a3), loss (a4),
backward (a5) with fused gradient accumulation (a6), the all-reduce across
ranks and the Adam update (a7).  Sampling and the host partitioner are
outside (the paper also excludes "data preparing").

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

For N > 1 it runs under torchrun, one rank per GPU over NCCL; micro-batches
are LPT-assigned to ranks and K (micro-batches per batch) is fixed across N
(the total work is the same batch), so the scaling is STRONG.
Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=50)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--config", default="C3")
    p.add_argument("--K", type=int, default=None,
                   help="micro-batches per batch (fixed across GPU counts); 0 = memory-aware (PAPER.md:1122-1134); "
                        "default: 32 for C3, memory-aware for C4, 8 for C2, 2 for C1")
    p.add_argument("--capacity-gb", type=float, default=24.0,
                   help="memory-aware K: per-micro-batch capacity of the Table 3 estimate (24 GB = the paper's "
                        "RTX 6000)")
    p.add_argument("--mode", default="bf16", choices=["fp32", "bf16"], help="GEMM operand precision")
    p.add_argument("--group", type=int, default=None,
                   help="micro-batches per launch group (0 = all of a rank's; default all, 1 for C4)")
    p.add_argument("--partition", default="reg", choices=["reg", "reg-greedy", "range", "random", "metis-raw"],
                   help="reg = REG + multilevel (METIS scheme, Alg. 1); reg-greedy = REG + greedy growing; "
                        "range / random / metis-raw = the paper's redundancy-unaware baselines (PAPER.md:1222-1230; "
                        "metis-raw: the multilevel partitioner on the raw graph induced on the outputs)")
    p.add_argument("--no-graph", action="store_true")
    p.add_argument("--no-reg", action="store_true", help="exclude the REG rebuild (a1) from the step")
    p.add_argument("--probe", default="auto")
    p.add_argument("--e2e-steps", type=int, default=20)
    p.add_argument("--no-fp32", action="store_true",
                   help="skip the nested paper-precision (fp32, 3xTF32 GEMMs) measurement of a bf16 run")
    p.add_argument("--cpu-threads", type=int, default=0, help="cpu_baseline / reference threads (0: all cores)")
    p.add_argument("--feat-shards", type=int, default=-1,
                   help="layer-0 feature table sharded by rows over R buffers: with N > 1 ranks R = N means one "
                        "shard per GPU, mapped by every rank through CUDA IPC (reads cross NVLink); at N = 1, R "
                        "virtual shards on the one GPU.  -1 (default): N for C5 (BASELINE configs[4]), else 0")
    p.add_argument("--cpu-sample-outputs", type=int, default=4096, help="cpu_baseline sample (~10 s)")
    p.add_argument("--ref-sample-outputs", type=int, default=512, help="--impl reference per-step sample (per core)")
    p.add_argument("--scale", type=float, default=1.0, help="shrink the graph (debug only)")
    p.add_argument("--json-out", default=None)
    p.add_argument("--sim-world", type=int, default=0, help="(study) run rank 0's share of an N-rank job on one GPU")
    p.add_argument("--feat-align", type=int, default=256, help="feature-table row alignment in bytes (0: 16)")
    p.add_argument("--input-order", default="random", choices=["random", "community"],
                   help="(study) node ids as generated (communities scattered) or community-contiguous")
    p.add_argument("--feat-layout", default="gid", choices=["gid", "owner", "l2"],
                   help="feature-table row order: gid (as generated) or owner (rows grouped by the micro-batch "
                        "that reads them most, experimental)")
    return p.parse_args()


# ------------------------------------------------------------------ helpers
def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled DURING the timed region."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device: int):
        self.device = device
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-lms", "50", "-i", str(self.device)], stdout=subprocess.PIPE,
                                         stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx = float(f[2])
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d, "measured (MEASURED_PEAKS.json)"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}, \
        "fallback (B200_PROFILING.md)"


def load_traffic(kernel: str, key: str):
    """ncu dram bytes per launch from a committed capture (profiles/), or None."""
    p = os.path.join(ROOT, "profiles", "traffic.json")
    if not os.path.exists(p):
        return None
    with open(p) as f:
        d = json.load(f)
    return d.get(key, {}).get(kernel)


# -------------------------------------------------------------- the workload
def build_inputs(args, rank, ws, device):
    """Rank 0 generates the synthetic products-shaped batch (C + OpenMP) and
    broadcasts it; every rank ends with the same host arrays."""
    import torch
    import torch.distributed as dist
    import synth
    cfg = synth.CONFIGS[args.config]
    if args.scale != 1.0:
        cfg = synth.scaled(cfg, args.scale)
    t0 = time.time()
    if rank == 0:
        ds = synth.make(cfg, with_features=None,      # None: C5's table is generated in chunks on the device
                        community_order=args.input_order == "community")
        arrays = [ds.graph.comm, ds.labels, ds.seeds]
        for b in ds.blocks:
            arrays += [b.indptr, b.nbr_pos, b.src_gid]
    else:
        ds, arrays = None, None
    if ws > 1:
        meta = [None]
        if rank == 0:
            meta = [[(a.shape, str(a.dtype)) for a in arrays]]
        dist.broadcast_object_list(meta, src=0)
        out = []
        for i, (shape, dt) in enumerate(meta[0]):
            t = torch.from_numpy(arrays[i]).to(device) if rank == 0 else \
                torch.empty(shape, dtype=getattr(torch, dt), device=device)
            dist.broadcast(t, src=0)
            out.append(t.cpu().numpy())
        arrays = out
        if rank != 0:
            blocks = []
            for l in range(cfg.L):
                ip, nb, sg = arrays[3 + 3 * l: 6 + 3 * l]
                blocks.append(synth.Block(len(ip) - 1, len(sg), ip, nb, sg))
            feats = synth.features(arrays[0], cfg.F, cfg.ld, cfg.feat_kind, seed=cfg.seeds["feat"]) \
                if cfg.n * cfg.ld * 4 <= synth.HOST_FEATURE_LIMIT else None
            ds = synth.Dataset(cfg, synth.Graph(None, None, arrays[0]), feats, arrays[1], arrays[2], blocks)
    return cfg, ds, time.time() - t0


def oracle_inputs(cfg, ds, part):
    """Full-batch blocks and a feature array for the oracle's micro-batch 0 of `part`: the host table
    itself, or (C5) only the rows micro-batch 0 reads, with layer-0 ids remapped onto them."""
    import synth
    import oracle
    if ds.feats is not None:
        return ds.blocks, ds.feats
    mb = oracle.extract(ds.blocks, part, 2, 0)
    gids = np.unique(mb[0].src_gid)
    feats = synth.features_rows(ds.graph.comm, cfg.F, cfg.ld, ids=gids, kind=cfg.feat_kind, seed=cfg.seeds["feat"])
    b0 = ds.blocks[0]
    j = np.minimum(np.searchsorted(gids, b0.src_gid), len(gids) - 1)
    remap = np.where(gids[j] == b0.src_gid, j, 0).astype(np.int32)
    blocks = [synth.Block(b0.n_dst, b0.n_src, b0.indptr, b0.nbr_pos, remap)] + list(ds.blocks[1:])
    return blocks, feats


def memory_aware(args, B, ctx, cfg, dev_blocks, rank, ws, device):
    """Choose K by the memory-aware loop on rank 0 (REG
    partition, Table 3 estimate under --capacity-gb) and share it; sets args.K."""
    import torch
    import torch.distributed as dist
    res = [None]
    if rank == 0:
        t0 = time.time()
        ip, col, w = B.betty_reg_build(ctx, dev_blocks[-1])
        reg = (ip.cpu().numpy(), col.cpu().numpy(), w.cpu().numpy())
        model = B.Model(cfg.dims, cfg.aggr, args.mode, args.mode)
        K, part, peak = B.betty_memory_aware_k(ctx, model, dev_blocks, reg, int(args.capacity_gb * 2 ** 30))
        res = [{"K": K, "capacity_gb": args.capacity_gb, "peak_estimate_gb": peak / 2 ** 30,
                "search_s": time.time() - t0}]
    if ws > 1:                     # every rank learns the outcome (a failure marker included) before exiting
        dist.broadcast_object_list(res, src=0)
    if res[0]["K"] < 0:
        raise SystemExit(f"memory-aware K: no K fits {args.capacity_gb} GB "
                         f"(smallest peak {res[0]['peak_estimate_gb']:.2f} GB)")
    args.K = res[0]["K"]
    return res[0]


def make_partition(args, B, ctx, cfg, ds, dev_blocks, rank, ws, device):
    import torch
    import torch.distributed as dist
    import synth
    if args.partition == "range":
        part = synth.range_partition(cfg.n_out, args.K)
    elif args.partition == "random":
        part = synth.random_partition(cfg.n_out, args.K, cfg.seeds["part"])
    elif args.partition == "metis-raw":
        from paper_conf_asplos_yangzd023_b200.partition import raw_graph_partition
        part = None
        if rank == 0:
            part = raw_graph_partition(ds.graph.indptr, ds.graph.indices, ds.seeds, args.K)
        if ws > 1:
            t = torch.as_tensor(part if rank == 0 else np.zeros(cfg.n_out, np.int32)).to(device)
            dist.broadcast(t, src=0)
            part = t.cpu().numpy()
    else:
        part = None
        if rank == 0:
            ip, col, w = B.betty_reg_build(ctx, dev_blocks[-1])
            part = B.betty_reg_partition(ip.cpu().numpy(), col.cpu().numpy(), w.cpu().numpy(), args.K,
                                         method="greedy" if args.partition == "reg-greedy" else "multilevel")
        if ws > 1:
            t = torch.as_tensor(part if rank == 0 else np.zeros(cfg.n_out, np.int32)).to(device)
            dist.broadcast(t, src=0)
            part = t.cpu().numpy()
    return np.ascontiguousarray(part, dtype=np.int32)


def alg_bytes(site: str, info: dict, cfg, mode: str, n_groups: int):
    """Algorithmic (compulsory) bytes of ONE launch of a kernel site, from the
    plan's per-layer totals.  Totals / n_groups = per launch.
    agg_l0 is SURVEY.md §8(d)'s AGG-MEAN formula with the gather stream replaced by each
    micro-batch's distinct source rows: 4E + 8(n_dst+1) + s F n_src + s F n_dst (index stream,
    indptr, every needed feature row once, the aggregated rows written) -- the kernel's extra
    self-row copy into XA and the ones column are not algorithmic."""
    s_feat = 2 if mode == "bf16" else 4
    s_act = 2 if mode == "bf16" else 4
    E, ns, nd = info["edges"], info["n_src"], info["n_dst"]
    F = cfg.F
    Fp = (F + 7) // 8 * 8
    ld_xa = (2 * Fp + 1 + 7) // 8 * 8
    if site == "agg_l0":
        b = 4 * E[0] + 8 * (nd[0] + 1) + s_feat * F * ns[0] + s_act * F * nd[0]
    elif site == "gemm_fwd_l0":
        H = cfg.hidden
        b = s_act * ld_xa * nd[0] + s_act * (2 * Fp + 1) * H + s_act * ((H + 1 + 7) // 8 * 8) * nd[0]
    elif site == "agg_l0_stream":        # the same formula with every edge's row gathered (no reuse)
        b = 4 * E[0] + 8 * (nd[0] + 1) + s_feat * F * E[0] + s_act * F * nd[0]
    else:
        return None
    return b / max(n_groups, 1)


METRIC = ("aggregated edges/s (SAGE, products-shape; edges of every micro-batch, redundant ones included, "
          "SURVEY §8(d)); epoch time = ms_per_step")


def workload_config(args, cfg, ws):
    """The `config` object both arms print (same workload, same K and partition)."""
    return {"workload": f"{args.config}: {cfg.name}-shaped DC-SBM ({cfg.n} nodes, {cfg.n}x{cfg.F} feats), "
                        f"{cfg.L}-layer SAGE-{cfg.aggr} {cfg.dims}, fanout {tuple(cfg.fanouts)}, {cfg.n_out} outputs",
            "K": args.K, "partition": args.partition, "group": args.group or "all",
            "step": ("REG + " if not args.no_reg else "") + "extract + fwd + loss + bwd + allreduce + adam",
            "graph": not args.no_graph, "parallelism": f"dp{ws} over micro-batches"}


# ------------------------------------------------------------ reference arm
def run_reference(args, ws, rank):
    """The CPU oracle, as it stands, on a bounded sample of the same workload: per step, one sample per
    host core in parallel (the first S outputs of micro-batch t of a range split, t = 0..cores-1)."""
    if rank != 0:
        return
    import synth
    import oracle
    from concurrent.futures import ThreadPoolExecutor
    cfg = synth.CONFIGS[args.config]
    if args.scale != 1.0:
        cfg = synth.scaled(cfg, args.scale)
    ds = synth.make(cfg, with_features=None)
    args.K = args.K or 8
    nt = cpu_threads(args)
    jobs = []
    for t in range(nt):
        part, sample_desc, edges = reference_sample(args, cfg, ds, args.ref_sample_outputs, mb=t % args.K)
        oblocks, ofeats = oracle_inputs(cfg, ds, part)
        jobs.append((part, oblocks, ofeats, edges))
    params = synth.init_params(cfg.dims, cfg.aggr, seed=cfg.seeds["init"])
    edges = sum(j[3] for j in jobs)

    def run(j):
        part, oblocks, ofeats, _ = j
        oracle.step(cfg.dims, cfg.aggr, args.mode == "bf16", oblocks, part, 2, [0], params, ofeats, ds.labels,
                    1.0 / cfg.n_out)
    times = []
    with ThreadPoolExecutor(nt) as ex:
        for it in range(args.warmup + args.steps):
            t0 = time.perf_counter()
            list(ex.map(run, jobs))
            if it >= args.warmup:
                times.append(time.perf_counter() - t0)
    t = float(np.mean(times))
    val = edges / t
    desc = (f"{nt} samples in parallel per step, each {args.ref_sample_outputs} outputs of one micro-batch "
            f"(K={args.K} range split) through {cfg.L} layers, extraction+fwd+bwd in float64; {edges} edges")
    line = {"impl": "reference", "metric": METRIC, "value": val,
            "unit": "edges/s", "higher_is_better": True, "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": t * 1e3, "dtype": "f64", "data": "synthetic",
            "config": dict(workload_config(args, cfg, ws), sample=desc),
            "cpu_baseline": {"value": val, "unit": "edges/s", "cores": nt, "kind": "oracle", "sample": desc},
            "e2e": {"value": val, "unit": "edges/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def reference_sample(args, cfg, ds, n_outputs, mb=0):
    """Outputs: the first S outputs (ascending) of micro-batch mb of a range
    partition into K parts -> a 2-way partition {sample, rest}."""
    import synth
    import oracle
    base = synth.range_partition(cfg.n_out, max(args.K, 1))
    idx = np.nonzero(base == mb)[0][:n_outputs]
    part = np.ones(cfg.n_out, dtype=np.int32)
    part[idx] = 0
    mb = oracle.extract(ds.blocks, part, 2, 0)
    edges = sum(b.n_edges for b in mb)
    desc = (f"{len(idx)} outputs (first of micro-batch {mb}, K={args.K}); {edges} edges through "
            f"{cfg.L} layers; extraction+fwd+bwd in float64, 1 thread")
    return part, desc, edges


# -------------------------------------------------------------------- main
def main():
    args = parse()
    if args.K is None:
        args.K = {"C1": 2, "C2": 8, "C3": 32, "C4": 0, "C5": 32}.get(args.config, 32)
    if args.group is None:
        args.group = 1 if args.config == "C4" else 0
    if args.config == "C5":      # 3 hops over a 111 M-node graph: ~20 s of oracle per 1k outputs
        args.cpu_sample_outputs = min(args.cpu_sample_outputs, 1024)
        args.ref_sample_outputs = min(args.ref_sample_outputs, 256)
    if args.config == "C4":      # a 5-hop closure reaches most of the graph: keep the oracle samples bounded
        args.cpu_sample_outputs = min(args.cpu_sample_outputs, 2)
        args.ref_sample_outputs = min(args.ref_sample_outputs, 1)
    ws, rank, local = dist_env()
    if args.impl == "reference":
        run_reference(args, ws, rank)
        return
    import torch
    import torch.distributed as dist
    import paper_conf_asplos_yangzd023_b200 as B
    from paper_conf_asplos_yangzd023_b200.dist import allreduce_grad, lpt_assign, plan_costs, reg_rows

    # BETTY_BENCH_ONE_GPU=1 (testing the multi-rank path on a one-GPU box): every rank on cuda:0 and
    # gloo for the collectives -- timings of such a run are not bench values
    one_gpu = os.environ.get("BETTY_BENCH_ONE_GPU", "0") == "1"
    if one_gpu:
        local = 0
    torch.cuda.set_device(local)
    device = torch.device("cuda", local)
    if ws > 1:
        if one_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=device)
    cfg, ds, t_gen = build_inputs(args, rank, ws, device)
    ctx = B.betty_ctx_create(local)
    dev_blocks = B.blocks_to_device(ds.blocks, local)
    mem_aware = None
    if args.K == 0:
        mem_aware = memory_aware(args, B, ctx, cfg, dev_blocks, rank, ws, device)
    part = make_partition(args, B, ctx, cfg, ds, dev_blocks, rank, ws, device)
    dpart = torch.as_tensor(part).to(device)
    # LPT cost per micro-batch from its per-layer sizes (GPU count-only extraction)
    costs = plan_costs(B.betty_mb_sizes(ctx, dev_blocks, dpart, args.K), cfg.dims)
    # --sim-world N (one GPU): run rank 0's share of an N-rank job -- its micro-batches and REG rows --
    # to study per-rank step time; the line is then per-rank, not a bench value
    wv, rv = (args.sim_world, 0) if args.sim_world > 1 else (ws, rank)
    my_k = lpt_assign(costs, wv)[rv]

    import synth
    if args.feat_shards < 0:
        args.feat_shards = ws if (args.config == "C5" and ws > 1) else 0
    shard = None
    if args.feat_shards > 0:       # rows sharded over R buffers (per GPU with IPC at N > 1)
        shard = make_shards(args, B, ctx, cfg, ds, rank, ws, device)
        feats = shard["stub"]
        args.no_fp32 = True
    else:
        feats = synth.features_device(cfg, ds, args.mode == "bf16", args.feat_align, device)   # bf16: reading #17
    host_gid0 = ds.blocks[0].src_gid
    if args.feat_layout == "l2":       # (study only) every layer-0 row read hits 64 Ki rows = 16 MB: L2-resident
        b0 = dev_blocks[0]
        b0.src_gid.copy_(torch.remainder(b0.src_gid, 65536))
        host_gid0 = b0.src_gid.cpu().numpy()
    if args.feat_layout == "owner":
        t_l = time.time()
        perm = owner_layout(ds.blocks, part, args.K)
        n_all = feats.shape[0]
        full_perm = np.empty(n_all, np.int64)
        miss = perm < 0
        full_perm[:len(perm)] = perm
        extra = np.nonzero(np.concatenate([miss, np.ones(n_all - len(perm), bool)]))[0]
        full_perm[extra] = len(perm) - miss.sum() + np.arange(len(extra))
        dperm = torch.as_tensor(full_perm).to(device)
        fp = torch.empty_like(feats)
        fp[dperm] = feats
        feats = fp
        b0 = dev_blocks[0]
        b0.src_gid.copy_(dperm[b0.src_gid.long()].to(torch.int32))
        del dperm, fp
        host_gid0 = b0.src_gid.cpu().numpy()
        print(f"feature layout: owner ({time.time() - t_l:.1f} s)", file=sys.stderr)
    labels = torch.as_tensor(ds.labels).to(device)
    model = B.Model(cfg.dims, cfg.aggr, args.mode, args.mode)
    params = torch.as_tensor(synth_params(cfg)).to(device)
    grad = torch.zeros_like(params)
    m = torch.zeros_like(params)
    v = torch.zeros_like(params)
    loss = torch.zeros(1, device=device)
    flags = (0 if args.no_graph else B.PLAN_GRAPH) | (0 if args.no_reg else B.PLAN_REG)
    t0 = time.time()
    plan, args.group = create_plan(B, ctx, model, dev_blocks, dpart, args.K, my_k, args.group, flags)
    if shard:
        plan.set_feature_shards(shard["bases"], shard["rps"])
    t_plan = time.time() - t0
    if wv > 1 and not args.no_reg:
        plan.set_reg_rows(*reg_rows(cfg.n_out, rv, wv))        # REG rows sharded across ranks
    info = plan.info()
    scale = 1.0 / cfg.n_out
    stream = torch.cuda.current_stream()
    t_opt = [0]

    def step(pl=None):
        loss.zero_()
        B.betty_step(ctx, pl or plan, params, feats, labels, scale, grad, loss)
        allreduce_grad(grad)
        t_opt[0] += 1
        B.betty_adam(ctx, params, grad, m, v, t_opt[0], zero_grad=True)

    for _ in range(args.warmup):
        step()
    B.betty_sync_check(ctx)

    # ------------------------------------------------------ timed region
    clocks = ClockSampler(local)
    clocks.start()
    ms = timed_ms(step, args.steps, ws, stream)
    clk = clocks.stop()
    t = torch.tensor([ms, float(sum(info["edges"])), float(info["kernels_per_step"])], device=device,
                     dtype=torch.float64)
    if ws > 1:
        tmax = t.clone()
        dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
        tsum = t.clone()
        dist.all_reduce(tsum, op=dist.ReduceOp.SUM)
        ms_step, edges_all = float(tmax[0]), float(tsum[1])
    else:
        ms_step, edges_all = ms, float(t[1])
    value = edges_all / (ms_step * 1e-3)
    launches = args.steps * (info["kernels_per_step"] + 1)
    full_edges = int(sum(b.n_edges for b in ds.blocks))
    peaks, peak_src = measured_peaks()
    tkey = lambda mode: f"{args.config}:K{args.K}:{mode}:n{ws}"     # noqa: E731 (profiles/traffic.json key)
    roof = roofline(plan, step, info, cfg, args.mode, ms, peaks, peak_src, tkey(args.mode))

    # ---------------------- paper precision (fp32) beside a bf16 headline
    paper = None
    if args.config == "C5" and args.mode == "bf16" and not args.no_fp32:
        args.no_fp32 = True           # a 57 GB fp32 table next to the bf16 plan's arenas does not fit one GPU
        paper = {"skipped": "C5: the fp32 feature table (57 GB) and fp32 arenas do not fit beside the bf16 run"}
    if args.mode == "bf16" and not args.no_fp32:
        feats32 = synth.features_device(cfg, ds, False, args.feat_align, device)
        if args.feat_layout != "gid":
            feats32 = None                       # (study layouts permute the bf16 table only)
        if feats32 is not None:
            model32 = B.Model(cfg.dims, cfg.aggr, "fp32", "fp32")
            plan32, g32 = create_plan(B, ctx, model32, dev_blocks, dpart, args.K, my_k, args.group, flags)
            if wv > 1 and not args.no_reg:
                plan32.set_reg_rows(*reg_rows(cfg.n_out, rv, wv))

            def step32():
                loss.zero_()
                B.betty_step(ctx, plan32, params, feats32, labels, scale, grad, loss)
                allreduce_grad(grad)
                t_opt[0] += 1
                B.betty_adam(ctx, params, grad, m, v, t_opt[0], zero_grad=True)
            for _ in range(args.warmup):
                step32()
            ms32 = timed_ms(step32, args.steps, ws, stream)
            info32 = plan32.info()
            t32 = torch.tensor([ms32], device=device, dtype=torch.float64)
            if ws > 1:
                dist.all_reduce(t32, op=dist.ReduceOp.MAX)
            ms32 = float(t32[0])
            paper = {"dtype": "fp32 (GEMMs as 3xTF32 on tcgen05: hi*hi + lo*hi + hi*lo, fp32 accumulation)",
                     "value": edges_all / (ms32 * 1e-3), "unit": "edges/s", "ms_per_step": ms32,
                     "full_batch_edges_per_s": full_edges / (ms32 * 1e-3), "group": g32 or "all",
                     "arena_gb": info32["arena_bytes"] / 2 ** 30,
                     "roofline": roofline(plan32, step32, info32, cfg, "fp32", ms32, peaks, peak_src,
                                          tkey("fp32"))}
            plan32.free()
            del feats32
            torch.cuda.synchronize()
            torch.cuda.empty_cache()

    # ------------------------------------- e2e: host buffers through the ABI
    # Every step copies its own inputs (the full-batch blocks and the partition) from pinned host
    # memory and reads its loss back.  The e2e plans are BETTY_PLAN_FRESH: each step derives everything
    # from the copied buffers (the full-batch CSCs and the REG's CSC are rebuilt inside the step), so a
    # step would consume a resampled batch of the same sizes.  Double-buffered when two plans fit in HBM
    # (the inputs of step i+1 are copied on a copy stream into the other buffer set while step i
    # computes; a plan binds its blocks' device pointers, so each buffer set has its own plan); else
    # serial.
    host = []
    for l, b in enumerate(ds.blocks):
        host += [torch.from_numpy(b.indptr).pin_memory(), torch.from_numpy(b.nbr_pos).pin_memory(),
                 torch.from_numpy(host_gid0 if l == 0 else b.src_gid).pin_memory()]
    host.append(torch.from_numpy(part).pin_memory())

    def dev_list(dbs, dp):
        out = []
        for db in dbs:
            out += [db.indptr, db.indices, db.src_gid]
        return out + [dp]
    fresh = flags | B.PLAN_FRESH
    plans, bufs = [], []
    for _ in range(2):
        try:
            dbs = B.blocks_to_device(ds.blocks, local)
            dbs[0].src_gid.copy_(dev_blocks[0].src_gid)
            dp = dpart.clone()
            pe, ge = create_plan(B, ctx, model, dbs, dp, args.K, my_k, args.group or 0, fresh)
            if ge != (args.group or 0):            # only the same launch grouping is the same step
                pe.free()
                raise RuntimeError("e2e plan would need a smaller launch group")
            if wv > 1 and not args.no_reg:
                pe.set_reg_rows(*reg_rows(cfg.n_out, rv, wv))
            if shard:
                pe.set_feature_shards(shard["bases"], shard["rps"])
            plans.append(pe)
            bufs.append(dev_list(dbs, dp))
            step(pe)                               # capture its graph outside the timed region
            torch.cuda.synchronize()
        except (B.BettyError, SystemExit, RuntimeError) as e:
            print(f"e2e: {len(plans)} buffer set(s) ({e})", file=sys.stderr)
            torch.cuda.synchronize()
            torch.cuda.empty_cache()
            break
    if not plans:                                  # no room for a FRESH plan: re-copy into the timed plan
        plans, bufs = [plan], [dev_list(dev_blocks, dpart)]
    h2d = sum(x.numel() * x.element_size() for x in host)
    # every step's loss is read on the host inside the timed region, one step behind the device (the
    # host waits for step i-1's loss while step i runs, so no step waits on a host round trip)
    loss_host = [torch.zeros(1).pin_memory() for _ in range(2)]
    ev_loss = [torch.cuda.Event() for _ in range(2)]
    losses = []
    cs = torch.cuda.Stream(device=device)
    ev_copied = [torch.cuda.Event() for _ in bufs]
    ev_used = [torch.cuda.Event() for _ in bufs]
    nb = len(bufs)

    def copy_in(b):
        with torch.cuda.stream(cs):
            for hsrc, ddst in zip(host, bufs[b]):
                ddst.copy_(hsrc, non_blocking=True)
            ev_copied[b].record(cs)
    e2e_steps = max(1, args.e2e_steps)
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()
    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    f0.record(stream)
    cs.wait_stream(stream)
    copy_in(0)
    for i in range(e2e_steps):
        b = i % nb
        stream.wait_event(ev_copied[b])
        if nb > 1 and i + 1 < e2e_steps:          # next step's inputs, once the step that used them is done
            if i >= 1:
                cs.wait_event(ev_used[1 - b])
            copy_in(1 - b)
        step(plans[b])
        ev_used[b].record(stream)
        loss_host[i % 2].copy_(loss, non_blocking=True)
        ev_loss[i % 2].record(stream)
        if nb == 1 and i + 1 < e2e_steps:
            cs.wait_stream(stream)
            copy_in(0)
        if i >= 1:                                  # step i-1's loss on the host
            ev_loss[(i - 1) % 2].synchronize()
            losses.append(float(loss_host[(i - 1) % 2][0]))
    ev_loss[(e2e_steps - 1) % 2].synchronize()
    losses.append(float(loss_host[(e2e_steps - 1) % 2][0]))
    f1.record(stream)
    torch.cuda.synchronize()
    e2e_ms = f0.elapsed_time(f1) / e2e_steps
    if ws > 1:
        te = torch.tensor([e2e_ms], device=device, dtype=torch.float64)
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
        e2e_ms = float(te[0])
    for pl in plans:
        if pl is not plan:
            pl.free()
    B.betty_sync_check(ctx)                        # FRESH steps validate the copied inputs on the device

    # ------------------------------------------------------- cpu baseline
    table_bytes = cfg.n * feats.shape[1] * feats.element_size() if shard else feats.numel() * feats.element_size()
    cpu = None
    if rank == 0 and ws == 1 and args.cpu_sample_outputs > 0:
        cpu = cpu_baseline(args, cfg, ds, scale)

    if rank == 0:
        line = {
            "metric": METRIC,
            "value": value, "unit": "edges/s", "n_gpus": ws, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": ms_step, "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "bf16-gemm/fp32-accum" if args.mode == "bf16" else "fp32",
            "data": "synthetic",
            "config": dict(workload_config(args, cfg, ws), micro_batches_per_rank=len(my_k),
                           l2="inputs > L2 (feature table %.2f GB + blocks)" % (table_bytes / 1e9)),
            "edges_per_step": edges_all,
            "full_batch_edges": full_edges,
            "full_batch_edges_per_s": full_edges / (ms_step * 1e-3),
            "plan": {k: info[k] for k in ("n_groups", "edges", "n_src", "n_dst", "reg_nnz", "arena_bytes",
                                          "kernels_per_step")},
            "memory": {"group": args.group or "all", "plan_arena_gb": info["arena_bytes"] / 2 ** 30,
                       "feature_table_gb": table_bytes / 2 ** 30,
                       "peak_allocated_gb": torch.cuda.max_memory_allocated(device) / 2 ** 30},
            "paper_precision": paper,
            "feature_shards": None if not shard else {
                "R": shard["R"], "rows_per_shard": shard["rps"], "mapping": shard["mapping"],
                "remote_row_fraction": shard["remote_fraction"],
                "layer0_gather_remote_GBps": (shard["remote_fraction"] * info["edges"][0] * shard["row_bytes"] /
                                              (roof["avg_launch_ms"] * roof["launches_per_step"] * 1e-3) / 1e9)
                if roof else None},
            "e2e": {"value": edges_all / (e2e_ms * 1e-3), "unit": "edges/s", "ms_per_step": e2e_ms,
                    "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": 4,
                    "input_buffers": nb, "fresh_inputs": plans[0] is not plan, "loss_reads": len(losses),
                    "loss_read": "every step's loss copied to pinned host memory and read on the host, one "
                                 "step behind the device"},
            "gpu_launches": launches,
            "clocks": clk,
            "roofline": roof,
            "cpu_baseline": cpu,
            "paper_context": "Table 6 (RTX 6000, real ogbn-products, fp32): 0.85 s/epoch at K=8, 2.55 s at K=64",
            "setup_s": {"generate": t_gen, "plan": t_plan},
            "memory_aware": mem_aware,
        }
        if args.sim_world > 1:
            line["note"] = (f"--sim-world {args.sim_world}: rank 0's share only (its micro-batches and REG rows), "
                            "per-rank step time, not a bench value")
        if one_gpu and ws > 1:
            line["note"] = "BETTY_BENCH_ONE_GPU: all ranks share cuda:0 over gloo (path test, not a bench value)"
        s = json.dumps(line)
        print(s, flush=True)
        if args.json_out:
            with open(args.json_out, "w") as f:
                f.write(s + "\n")
    plan.free()
    if shard:
        if ws > 1:
            dist.barrier()                         # no rank still reads a peer's shard
        for b in shard["buffers"]:
            b.free()
    if ws > 1:
        dist.destroy_process_group()


def make_shards(args, B, ctx, cfg, ds, rank, ws, device):
    """The layer-0 feature table split by rows into R shards.  N > 1 with R == N: rank r owns rows
    [r rps, (r+1) rps) in a cudaMalloc'd buffer and maps every other rank's buffer through CUDA IPC
    (handles exchanged with one all_gather_object; no collective in the step: the layer-0 gathers
    read remote rows over NVLink).  N = 1: R buffers on the one GPU (virtual shards)."""
    import torch
    import torch.distributed as dist
    import synth
    bf16 = args.mode == "bf16"
    dt = torch.bfloat16 if bf16 else torch.float32
    esz = 2 if bf16 else 4
    per = max(1, args.feat_align // esz) if args.feat_align > 0 else 1
    ld = (cfg.ld + per - 1) // per * per
    R = args.feat_shards
    rps = (cfg.n + R - 1) // R
    own = []
    if ws > 1:
        if R != ws:
            raise SystemExit("--feat-shards with N > 1 ranks must be N (one shard per GPU)")
        mine = B.DevBuffer(ctx, rps * ld * esz)
        synth.features_fill_rows(cfg, ds, mine.tensor(dt, (rps, ld)), rank * rps)
        torch.cuda.synchronize()
        handles = [None] * ws
        dist.all_gather_object(handles, mine.ipc_handle())
        bases = []
        for r in range(ws):
            if r == rank:
                bases.append(mine.ptr)
            else:
                o = B.DevBuffer.open(ctx, handles[r], rps * ld * esz)
                own.append(o)
                bases.append(o.ptr)
        own.append(mine)
        mapping = f"one shard per GPU, peers mapped with CUDA IPC ({ws} GPUs)"
    else:
        bases = []
        for r in range(R):
            b = B.DevBuffer(ctx, rps * ld * esz)
            synth.features_fill_rows(cfg, ds, b.tensor(dt, (rps, ld)), r * rps)
            own.append(b)
            bases.append(b.ptr)
        mapping = f"{R} virtual shards on one GPU"
    torch.cuda.synchronize()
    return {"R": R, "rps": rps, "bases": bases, "buffers": own, "mapping": mapping, "row_bytes": cfg.F * esz,
            "remote_fraction": (R - 1) / R if ws > 1 else 0.0,
            "stub": torch.zeros((1, ld), dtype=dt, device=device)}


def timed_ms(step, steps, ws, stream):
    """K steps between a barrier + synchronize on both sides, timed with CUDA events on the launching
    stream; ms per step of THIS rank (the caller takes the max over ranks)."""
    import torch
    import torch.distributed as dist
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(steps):
        step()
    e1.record(stream)
    torch.cuda.synchronize()
    if ws > 1:
        dist.barrier()
    return e0.elapsed_time(e1) / steps


SITES = {"agg_l0": 1, "gemm_fwd_l0": 2, "gemm_red_l0": 3, "extract": 4, "reg": 5}


def roofline(plan, step, info, cfg, mode, ms, peaks, peak_src, key):
    """Roofline of the dominant kernel (the layer-0 mean aggregation): its launches bracketed by CUDA
    events on the step's stream (betty_plan_probe) over 3 steps; the other sites alongside."""
    probe_ms = {}
    for name, sid in SITES.items():
        plan.probe(sid)
        tot, n = 0.0, 0
        for _ in range(3):
            step()
            ms_k, nl = plan.probe_read()
            tot += ms_k
            n += nl
        probe_ms[name] = (tot / max(n, 1), n / 3)
    plan.probe(0)
    dom = "agg_l0"
    per_launch_ms, launches_per_step = probe_ms[dom]
    ab = alg_bytes(dom, info, cfg, mode, info["n_groups"]) if cfg.aggr == "mean" else None
    if ab is None:
        return None
    achieved = ab / (per_launch_ms * 1e-3) / 1e9
    sb = alg_bytes("agg_l0_stream", info, cfg, mode, info["n_groups"])
    rows = (info["edges"][0] + info["n_dst"][0]) / max(info["n_groups"], 1)   # neighbour + self rows fetched
    return {"kernel": "k_agg_mean_g4 (layer-0 mean aggregation)", "bound": "hbm", "achieved": achieved,
            "peak": peaks["hbm_gbs"], "unit": "GB/s", "frac": achieved / peaks["hbm_gbs"],
            "traffic": load_traffic(dom, key), "alg_bytes_per_launch": ab,
            "alg_bytes_formula": "4E + 8(n_dst+1) + s*F*n_src + s*F*n_dst (SURVEY §8(d), distinct sources)",
            "avg_launch_ms": per_launch_ms, "launches_per_step": launches_per_step, "peak_source": peak_src,
            "share_of_step": per_launch_ms * launches_per_step / ms,
            # context (frac above is the official, compulsory-bytes figure): SURVEY §8(d)'s stream form
            # of the same formula, s*F*E gathered, and the row-fetch rate against the measured random-row
            # ceiling of a table larger than L2 (profiles/r03_gather_l2.txt, r03_agg_bound.txt)
            "stream": {"alg_bytes_per_launch": sb,
                       "achieved": sb / (per_launch_ms * 1e-3) / 1e9,
                       "frac": sb / (per_launch_ms * 1e-3) / 1e9 / peaks["hbm_gbs"],
                       "formula": "4E + 8(n_dst+1) + s*F*E + s*F*n_dst (SURVEY §8(d) AGG-MEAN fwd)"},
            "row_fetches_per_ns": rows / (per_launch_ms * 1e6),
            "row_fetch_ceiling_per_ns": {"value": 24.9, "what": "random 208-byte rows from a 0.52 GB table, "
                                         "LDG at full occupancy (tools/micro/gather_l2.cu); TMA gather4 22.9"}
            if mode == "bf16" and cfg.F == 100 else None,
            "other_sites_ms_per_step": {k: v[0] * v[1] for k, v in probe_ms.items()}}


def cpu_threads(args):
    n = args.cpu_threads or len(os.sched_getaffinity(0))
    return max(1, n)


def cpu_baseline(args, cfg, ds, scale):
    """The float64 oracle as it stands on the host cores: one bounded sample per thread (the first S
    outputs of micro-batch t of a range split of the outputs), threads in parallel (ctypes releases the
    GIL for the C call); value = the samples' edges / wall time."""
    import oracle
    from concurrent.futures import ThreadPoolExecutor
    nt = cpu_threads(args)
    jobs = []
    for t in range(nt):
        rpart, desc, redges = reference_sample(args, cfg, ds, args.cpu_sample_outputs, mb=t % max(args.K, 1))
        oblocks, ofeats = oracle_inputs(cfg, ds, rpart)
        jobs.append((rpart, oblocks, ofeats, redges))
    pr = synth_params(cfg).astype(np.float64)

    def run(j):
        rpart, oblocks, ofeats, _ = j
        oracle.step(cfg.dims, cfg.aggr, args.mode == "bf16", oblocks, rpart, 2, [0], pr, ofeats, ds.labels, scale)
    tc = time.perf_counter()
    with ThreadPoolExecutor(nt) as ex:
        list(ex.map(run, jobs))
    dt = time.perf_counter() - tc
    edges = sum(j[3] for j in jobs)
    return {"value": edges / dt, "unit": "edges/s", "cores": nt, "kind": "oracle",
            "sample": f"{nt} samples in parallel, each {args.cpu_sample_outputs} outputs of one micro-batch "
                      f"(K={args.K} range split) through {cfg.L} layers, extraction+fwd+bwd in float64; "
                      f"{edges} edges", "seconds": dt}


def create_plan(B, ctx, model, dev_blocks, dpart, K, my_k, group, flags):
    """The plan with the requested launch group (0 = all of the rank's micro-batches).  When its arenas
    do not fit in HBM (C5: ~10^9 micro-batch edges), a one-micro-batch plan measures the arena of the
    largest micro-batch and the group becomes what fits in 85 % of the free HBM (halved further on
    failure).  Returns (plan, group actually used; 0 = all)."""
    import torch

    def oom(e):
        return "ENOMEM" in str(e) or "out of memory" in str(e)

    def attempt(g):
        try:
            return B.betty_plan_create(ctx, model, dev_blocks, dpart, K, my_k, group=g, flags=flags)
        except B.BettyError as e:
            if not oom(e):
                raise
            torch.cuda.synchronize()
            torch.cuda.empty_cache()
            return None

    n = max(1, len(my_k))
    g = group if group > 0 else n
    plan = attempt(g)
    if plan is not None:
        return plan, (0 if group == 0 else g)
    one = attempt(1)
    if one is None:
        raise SystemExit("plan: one micro-batch does not fit in HBM")
    a1 = one.info()["arena_bytes"]
    one.free()
    torch.cuda.synchronize()
    torch.cuda.empty_cache()
    free = torch.cuda.mem_get_info()[0]
    g = max(1, min(g // 2, int(0.85 * free / max(a1, 1))))
    while True:
        print(f"plan: arenas of the full group do not fit; largest micro-batch {a1 / 2**30:.2f} GB, "
              f"free {free / 2**30:.1f} GB -> launch group {g}", file=sys.stderr)
        plan = attempt(g)
        if plan is not None:
            return plan, g
        if g == 1:
            raise SystemExit("plan: no launch group fits in HBM")
        g = max(1, g // 2)


def owner_layout(blocks, part, K):
    """Row order of the feature table grouped by owner micro-batch (majority vote of the micro-batches
    whose layer-0 sources contain the node, propagated down the full-batch blocks).  Returns perm with
    perm[gid] = new row.  Host preprocessing, outside the step (like the partition)."""
    def votes(n_items, idx, who):
        key = idx.astype(np.int64) * (K + 1) + who.astype(np.int64)
        u, c = np.unique(key, return_counts=True)
        item, own = u // (K + 1), u % (K + 1)
        o = np.lexsort((own, -c, item))
        item, own = item[o], own[o]
        first = np.ones(len(item), bool)
        first[1:] = item[1:] != item[:-1]
        out = np.full(n_items, K, np.int64)
        out[item[first]] = own[first]
        return out
    own_dst = np.asarray(part, dtype=np.int64)
    for b in reversed(blocks):
        deg = np.diff(b.indptr)
        idx = np.concatenate([b.nbr_pos.astype(np.int64), np.arange(b.n_dst)])
        who = np.concatenate([np.repeat(own_dst, deg), own_dst])
        own_dst = votes(b.n_src, idx, who)
    b0 = blocks[0]
    n = int(max(b0.src_gid.max() + 1, 1))
    order = np.lexsort((b0.src_gid, own_dst))
    perm = np.full(n, -1, np.int64)
    perm[b0.src_gid[order]] = np.arange(b0.n_src)
    return perm


def synth_params(cfg):
    import synth
    return synth.init_params(cfg.dims, cfg.aggr, seed=cfg.seeds["init"])


if __name__ == "__main__":
    main()
