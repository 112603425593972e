"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the
same seeded inputs.  Integer results (REG, blocks) bit-exact; floating point
within DESIGN.md §3 reading #18 (rtol 1e-5 fp32 / 2e-2 bf16-GEMM mode)."""
import numpy as np
import pytest
import torch

import oracle
import synth
from tests.helpers import assert_close, assert_grad_close, load_golden, tiny

pytestmark = pytest.mark.gpu

RTOL = {"fp32": 1e-5, "bf16": 2e-2}


@pytest.fixture(scope="module")
def B():
    import paper_conf_asplos_yangzd023_b200 as B
    assert torch.cuda.is_available()
    return B


@pytest.fixture(scope="module")
def ctx(B):
    return B.betty_ctx_create(0)


def golden_full():
    g = load_golden("g1.json")
    rows = [{int(k): v for k, v in g["rows"][str(l)].items()} for l in (0, 1)]
    return g, synth.blocks_from_rows(g["seeds"], rows)


def reg_equal(B, ctx, blk_dev, blk_host):
    ip, col, w = B.betty_reg_build(ctx, blk_dev)
    rp, rc, rw = oracle.reg(blk_host.n_src, blk_host.indptr, blk_host.nbr_pos)
    np.testing.assert_array_equal(ip.cpu().numpy(), rp)
    np.testing.assert_array_equal(col.cpu().numpy(), rc)
    np.testing.assert_array_equal(w.cpu().numpy(), rw)
    return len(rc)


def blocks_equal(gpu, ora):
    assert len(gpu) == len(ora)
    for l, (a, b) in enumerate(zip(gpu, ora)):
        assert (a.n_dst, a.n_src, a.n_edges) == (b.n_dst, b.n_src, b.n_edges), l
        for name, x, y in [("indptr", a.indptr, b.indptr), ("indices", a.indices, b.indices),
                           ("src_pos", a.src_pos, b.src_pos), ("src_gid", a.src_gid, b.src_gid),
                           ("t_indptr", a.t_indptr, b.t_indptr), ("t_indices", a.t_indices, b.t_indices)]:
            np.testing.assert_array_equal(x.cpu().numpy(), y, err_msg=f"layer {l} {name}")


# ------------------------------------------------------------------ REG (a1)
def test_reg_golden(B, ctx):
    g, full = golden_full()
    dev = B.blocks_to_device(full)
    ip, col, w = B.betty_reg_build(ctx, dev[1])
    assert ip.tolist() == g["reg"]["indptr"] and col.tolist() == g["reg"]["col"] and w.tolist() == g["reg"]["w"]


@pytest.mark.parametrize("seed", range(4))
def test_reg_random_small(B, ctx, seed):
    g, sd, blocks, feats, labels = tiny(n=500, pairs=3000, fanouts=(4, 7), n_out=120, seed=seed)
    reg_equal(B, ctx, B.blocks_to_device(blocks)[-1], blocks[-1])


@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_reg_row_shards(B, ctx, world):
    """Row-sharded REG (one share per rank): every rank's rows [r n / R, (r+1) n / R)
    equal the oracle's REG rows, bit-exact, with global column ids; an empty share and a bad range."""
    g, sd, blocks, feats, labels = tiny(n=500, pairs=3000, fanouts=(4, 7), n_out=120, seed=7)
    dev = B.blocks_to_device(blocks)[-1]
    rp, rc, rw = oracle.reg(blocks[-1].n_src, blocks[-1].indptr, blocks[-1].nbr_pos)
    n = blocks[-1].n_dst
    for r in range(world):
        r0, r1 = r * n // world, (r + 1) * n // world
        ip, col, w = B.betty_reg_build_rows(ctx, dev, r0, r1)
        np.testing.assert_array_equal(ip.cpu().numpy(), rp[r0:r1 + 1] - rp[r0])
        np.testing.assert_array_equal(col.cpu().numpy(), rc[rp[r0]:rp[r1]])
        np.testing.assert_array_equal(w.cpu().numpy(), rw[rp[r0]:rp[r1]])
    ip, col, w = B.betty_reg_build_rows(ctx, dev, 5, 5)           # empty share
    assert ip.tolist() == [0] and col.numel() == 0
    with pytest.raises(B.BettyError):
        B.betty_reg_build_rows(ctx, dev, 10, n + 1)


def test_plan_reg_rows(B, ctx):
    """A plan's in-step REG restricted to one rank's rows: sized to that share's nnz, and the step
    (graph replay included) still produces the oracle's gradient."""
    g, sd, blocks, feats, labels = tiny(n=400, pairs=2000, fanouts=(3, 5), n_out=60, F=8, C=4, seed=3)
    dims = [8, 16, 4]
    dev = B.blocks_to_device(blocks)
    K = 3
    part = synth.random_partition(len(sd), K, 1)
    params = synth.init_params(dims, "mean", seed=2)
    og, ol = oracle.step(dims, "mean", False, blocks, part, K, list(range(K)), params, feats, labels, 1.0 / len(sd))
    rp, rc, rw = oracle.reg(blocks[-1].n_src, blocks[-1].indptr, blocks[-1].nbr_pos)
    model = B.Model(dims, "mean", "fp32", "fp32")
    plan = B.betty_plan_create(ctx, model, dev, torch.as_tensor(part).cuda(), K, list(range(K)), group=0,
                               flags=B.PLAN_GRAPH | B.PLAN_REG)
    assert plan.info()["reg_nnz"] == len(rc)
    P = torch.as_tensor(params).cuda()
    X = torch.as_tensor(feats).cuda()
    Y = torch.as_tensor(labels).cuda()
    for r0, r1 in ((0, 60), (20, 40), (59, 60)):
        plan.set_reg_rows(r0, r1)
        assert plan.info()["reg_nnz"] == rp[r1] - rp[r0]
        for rep in range(2):
            grad = torch.zeros_like(P)
            loss = torch.zeros(1, device="cuda")
            B.betty_step(ctx, plan, P, X, Y, 1.0 / len(sd), grad, loss)
            B.betty_sync_check(ctx)
            assert_grad_close(grad.cpu().numpy(), og, dims, "mean", 1e-5, f"rows {r0}:{r1} rep {rep}")
    with pytest.raises(B.BettyError):
        plan.set_reg_rows(0, 61)
    plan.free()


@pytest.mark.parametrize("n,m,d", [(2000, 150, 60), (600, 40, 30)])
def test_reg_hub_rows(B, ctx, n, m, d):
    """Hub rows: every output samples d of m shared sources, so each column has ~n d / m outputs and a
    row has ~d (n d / m - 1) candidate products -- (2000, 150, 60): ~48 k > 32768, the bitmap-rank
    path (no degree bound in Eq. 2-4); (600, 40, 30): ~13 k, the CTA sort path.
    A mixed block (hub rows + short rows) as well.  Bit-exact against the oracle."""
    rng = np.random.default_rng(n + m)
    rows = [np.sort(rng.choice(m, size=d, replace=False)).astype(np.int32) for _ in range(n)]
    # a few short rows on private sources (warp path) in the same block
    rows += [np.array([m + k], np.int32) for k in range(50)]
    indptr = np.concatenate([[0], np.cumsum([len(r) for r in rows])]).astype(np.int64)
    idx = np.concatenate(rows).astype(np.int32)
    host = synth.Block(len(rows), m + 50, indptr, idx, np.arange(m + 50, dtype=np.int32))
    nnz = reg_equal(B, ctx, B.blocks_to_device([host])[0], host)
    assert nnz > 0


def test_reg_rejects_duplicate_edges(B, ctx):
    blk = B.Block(2, 3, torch.tensor([0, 2, 3], dtype=torch.int64, device="cuda"),
                  torch.tensor([1, 1, 2], dtype=torch.int32, device="cuda"),
                  torch.arange(3, dtype=torch.int32, device="cuda"))
    with pytest.raises(B.BettyError, match="EINVAL"):
        B.betty_reg_build(ctx, blk)


def test_reg_hub_rows_use_cta_path(B, ctx):
    """Star + K_mn shapes: rows with > 256 candidate products (CTA bitonic path)."""
    n, m = 400, 3
    indptr = np.arange(n + 1, dtype=np.int64) * m
    idx = np.tile(np.arange(m, dtype=np.int32), n)
    host = synth.Block(n, m, indptr, idx, np.arange(m, dtype=np.int32))
    reg_equal(B, ctx, B.blocks_to_device([host])[0], host)


# ----------------------------------------------------------- extraction (a2)
def test_extract_golden(B, ctx):
    g, full = golden_full()
    dev = B.blocks_to_device(full)
    part = torch.tensor(g["part"], dtype=torch.int32, device="cuda")
    for k in range(g["K"]):
        mb = B.betty_extract_blocks(ctx, dev, part, g["K"], k)
        blocks_equal(mb, oracle.extract(full, np.array(g["part"]), g["K"], k))


@pytest.mark.parametrize("seed,K,fan", [(1, 1, (3, 4)), (2, 3, (2, 3, 4)), (3, 7, (3, 5)), (4, 40, (2, 2, 3))])
def test_extract_random(B, ctx, seed, K, fan):
    g, sd, blocks, feats, labels = tiny(n=400, pairs=1500, fanouts=fan, n_out=40, seed=seed)
    part = synth.random_partition(len(sd), K, seed)       # K=40 leaves parts empty
    dev = B.blocks_to_device(blocks)
    dpart = torch.as_tensor(part).cuda()
    for k in range(K):
        blocks_equal(B.betty_extract_blocks(ctx, dev, dpart, K, k), oracle.extract(blocks, part, K, k))


def concat_oracle(blocks, part, K, ks):
    """The layout of a launch group: the block-diagonal union
    of the oracle's micro-batches ks with the dst rows of ALL of them first
    (so dst ids stay a prefix of src ids), then each micro-batch's new
    sources in micro-batch order; the output layer lists the micro-batches'
    outputs in order; a layer's dst list is the src list of the layer above."""
    mbs = [oracle.extract(blocks, part, K, k) for k in ks]
    L = len(blocks)
    D = [(j, t) for j, mb in enumerate(mbs) for t in range(mb[L - 1].n_dst)]
    out = [None] * L
    for l in range(L - 1, -1, -1):
        gid = {jt: r for r, jt in enumerate(D)}
        S = list(D)
        for j, mb in enumerate(mbs):
            for t in range(mb[l].n_dst, mb[l].n_src):
                gid[(j, t)] = len(S)
                S.append((j, t))
        indptr, idx = [0], []
        for (j, t) in D:
            b = mbs[j][l]
            idx += [gid[(j, int(u))] for u in b.indices[b.indptr[t]:b.indptr[t + 1]]]
            indptr.append(len(idx))
        cols = [[] for _ in S]
        for r in range(len(D)):
            for e in range(indptr[r], indptr[r + 1]):
                cols[idx[e]].append(r)
        t_indptr = np.cumsum([0] + [len(c) for c in cols]).astype(np.int64)
        t_idx = np.array([r for c in cols for r in c], dtype=np.int32)
        out[l] = oracle.MBlock(len(D), len(S), np.array(indptr, np.int64), np.array(idx, np.int32),
                               np.array([mbs[j][l].src_pos[t] for j, t in S], np.int32),
                               np.array([mbs[j][l].src_gid[t] for j, t in S], np.int32), t_indptr, t_idx)
        D = S
    return out


@pytest.mark.parametrize("group", [1, 2, 3, 0])
def test_group_extraction(B, ctx, group):
    """The fused step's extraction of a launch group == the block-diagonal
    union of the oracle's micro-batches (bit-exact)."""
    g, sd, blocks, feats, labels = tiny(n=500, pairs=2000, fanouts=(3, 4, 5), n_out=50, seed=8)
    K = 6
    part = synth.random_partition(len(sd), K, 2)
    ks = [5, 0, 2, 3, 4]
    dev = B.blocks_to_device(blocks)
    dpart = torch.as_tensor(part).cuda()
    model = B.Model([8, 12, 12, 3], "mean", "fp32")
    plan = B.betty_plan_create(ctx, model, dev, dpart, K, ks, group=group, flags=0)
    c = len(ks) if group == 0 else group
    groups = [ks[i:i + c] for i in range(0, len(ks), c)]
    for gi, gk in enumerate(groups):
        got = plan.group_blocks(gi)
        want = concat_oracle(blocks, part, K, gk)
        for l, (a, b) in enumerate(zip(got, want)):
            assert (a.n_dst, a.n_src, a.n_edges) == (b.n_dst, b.n_src, b.n_edges), (gi, l)
            for name in ("indptr", "indices", "src_pos", "src_gid"):
                np.testing.assert_array_equal(getattr(a, name).cpu().numpy(), getattr(b, name),
                                              err_msg=f"group {gi} layer {l} {name}")
            if a.t_indptr is not None:
                np.testing.assert_array_equal(a.t_indptr.cpu().numpy(), b.t_indptr, err_msg=f"g{gi} l{l} t_indptr")
                np.testing.assert_array_equal(a.t_indices.cpu().numpy(), b.t_indices, err_msg=f"g{gi} l{l} t_idx")
    plan.free()


def test_wide_launch_group_and_many_parts(B, ctx):
    """The output selection at its limits: K = 700 parts over 600 outputs (most parts empty), a launch
    group of 512 micro-batches (the largest one pass handles) holding every non-empty and many empty
    ones, bit-exact against the oracle's union; K beyond 16384 is refused (EUNSUPPORTED)."""
    g, sd, blocks, feats, labels = tiny(n=3000, pairs=9000, fanouts=(3, 4), n_out=600, seed=9)
    K = 700
    part = synth.random_partition(len(sd), K, 4)
    ks = list(range(0, K, 1))[:512]
    dev = B.blocks_to_device(blocks)
    dpart = torch.as_tensor(part).cuda()
    model = B.Model([8, 12, 3], "mean", "fp32")
    plan = B.betty_plan_create(ctx, model, dev, dpart, K, ks, group=512, flags=0)
    got = plan.group_blocks(0)
    want = concat_oracle(blocks, part, K, ks)
    for l, (a, b) in enumerate(zip(got, want)):
        assert (a.n_dst, a.n_src, a.n_edges) == (b.n_dst, b.n_src, b.n_edges), l
        for name in ("indptr", "indices", "src_pos", "src_gid"):
            np.testing.assert_array_equal(getattr(a, name).cpu().numpy(), getattr(b, name), err_msg=f"l{l} {name}")
    plan.free()
    with pytest.raises(B.BettyError, match="EUNSUPPORTED"):
        B.betty_extract_blocks(ctx, dev, torch.zeros(len(sd), dtype=torch.int32, device="cuda"), 20000, 0)
    with pytest.raises(B.BettyError, match="EUNSUPPORTED"):
        B.betty_plan_create(ctx, model, dev, dpart, K, list(range(K)), group=600, flags=0)


def test_extract_bad_input(B, ctx):
    g, sd, blocks, feats, labels = tiny(seed=5)
    dev = B.blocks_to_device(blocks)
    part = torch.zeros(len(sd), dtype=torch.int32, device="cuda")
    with pytest.raises(B.BettyError, match="EINVAL"):
        B.betty_extract_blocks(ctx, dev, part, 2, 2)
    part[3] = 9
    with pytest.raises(B.BettyError, match="EINVAL"):
        B.betty_extract_blocks(ctx, dev, part, 2, 0)


# ------------------------------------------------------- SAGE fwd/bwd (a3-a6)
CASES = [
    dict(name="mean2", aggr="mean", fanouts=(3, 4), dims=[20, 32, 5]),
    dict(name="mean2-wide", aggr="mean", fanouts=(5, 8), dims=[100, 256, 47]),
    dict(name="mean3", aggr="mean", fanouts=(3, 3, 4), dims=[24, 40, 40, 6]),
    dict(name="mean2-pf0", aggr="mean", fanouts=(3, 4), dims=[70, 16, 4]),
    dict(name="pool2", aggr="pool", fanouts=(3, 4), dims=[16, 24, 5]),
    dict(name="pool3", aggr="pool", fanouts=(2, 3, 3), dims=[12, 16, 16, 3]),
    # full neighbourhoods on dense graphs: rows longer than the gather pipeline's stage ("long rows")
    dict(name="mean2-full-hub", aggr="mean", fanouts=(-1, -1), dims=[8, 16, 3], n=400, pairs=30000),
    dict(name="mean2-full-wide", aggr="mean", fanouts=(-1, -1), dims=[100, 128, 5], n=400, pairs=8000),
    # aggregate-first hidden layer of width 64: the lane-group CSC backward (2 lanes per source)
    dict(name="mean3-agg64", aggr="mean", fanouts=(3, 4, 5), dims=[32, 64, 64, 5]),
    # pool rows longer than one warp-wide position search (byte-position argmax, rows of ~150 edges)
    dict(name="pool2-full-hub", aggr="pool", fanouts=(-1, -1), dims=[8, 16, 3], n=400, pairs=30000),
    # the sum aggregator (Table 1 "Sum"): aggregate-first, project-first, the 3-layer hidden CSC path
    dict(name="sum2", aggr="sum", fanouts=(3, 4), dims=[20, 32, 5]),
    dict(name="sum2-pf", aggr="sum", fanouts=(3, 4), dims=[70, 16, 4]),
    dict(name="sum3-agg64", aggr="sum", fanouts=(3, 4, 5), dims=[32, 64, 64, 5]),
]


def make_case(c, seed=1, n=600, pairs=2400, n_out=60):
    n, pairs = c.get("n", n), c.get("pairs", pairs)
    F = c["dims"][0]
    ld = (F + 7) // 8 * 8
    g, sd, blocks, feats, _ = tiny(n=n, pairs=pairs, fanouts=c["fanouts"], n_out=n_out, F=F, C=c["dims"][-1],
                                   seed=seed, ld=ld)
    labels = (np.arange(n) * 5 % c["dims"][-1]).astype(np.int32)
    params = synth.init_params(c["dims"], c["aggr"], seed=seed)
    return sd, blocks, feats, labels, params


def dev_feats(feats, mode):
    t = torch.as_tensor(feats).cuda()
    return t.to(torch.bfloat16).contiguous() if mode == "bf16" else t


@pytest.mark.parametrize("mode", ["fp32", "bf16"])
@pytest.mark.parametrize("c", CASES, ids=lambda c: c["name"])
def test_sage_micro_batch(B, ctx, c, mode):
    sd, blocks, feats, labels, params = make_case(c)
    K = 3
    part = synth.random_partition(len(sd), K, 7)
    dev = B.blocks_to_device(blocks)
    dpart = torch.as_tensor(part).cuda()
    model = B.Model(c["dims"], c["aggr"], mode, mode)
    assert B.betty_num_params(model) == len(params)
    P = torch.as_tensor(params).cuda()
    X = dev_feats(feats, mode)
    Y = torch.as_tensor(labels).cuda()
    scale = 1.0 / len(sd)
    for k in range(K):
        mb = B.betty_extract_blocks(ctx, dev, dpart, K, k)
        if mb[-1].n_dst == 0:
            continue
        saved, logits = B.betty_sage_fwd(ctx, model, P, mb, X)
        grad = torch.zeros_like(P)
        loss = torch.zeros(1, device="cuda")
        B.betty_sage_bwd(ctx, model, P, mb, saved, Y, scale, grad, loss)
        torch.cuda.synchronize()
        om = oracle.extract(blocks, part, K, k)
        og, ol, olog = oracle.sage(c["dims"], c["aggr"], mode == "bf16", om, params, feats, labels, scale,
                                   want_logits=True)
        assert_close(logits.cpu().numpy(), olog, RTOL[mode], f"logits k={k}")
        assert_grad_close(grad.cpu().numpy(), og, c["dims"], c["aggr"], RTOL[mode], f"grad k={k}")
        assert loss.item() == pytest.approx(ol, rel=RTOL[mode])
        saved.free()


@pytest.mark.parametrize("mode", ["fp32", "bf16"])
@pytest.mark.parametrize("group", [1, 2, 0])
@pytest.mark.parametrize("graph", [False, True])
@pytest.mark.parametrize("c", [CASES[1], CASES[2], CASES[4], CASES[7], CASES[8], CASES[9], CASES[10], CASES[11],
                               CASES[12]], ids=lambda c: c["name"])
def test_step_matches_oracle(B, ctx, c, mode, group, graph):
    """betty_step (fused extraction + fwd + loss + bwd + accumulation over a
    rank's micro-batches) vs oracle_step, for several launch groupings."""
    sd, blocks, feats, labels, params = make_case(c, seed=2)
    K = 5
    part = synth.random_partition(len(sd), K, 11)
    ks = [0, 2, 3, 4]
    dev = B.blocks_to_device(blocks)
    dpart = torch.as_tensor(part).cuda()
    model = B.Model(c["dims"], c["aggr"], mode, mode)
    P = torch.as_tensor(params).cuda()
    X = dev_feats(feats, mode)
    Y = torch.as_tensor(labels).cuda()
    scale = 1.0 / len(sd)
    plan = B.betty_plan_create(ctx, model, dev, dpart, K, ks, group=group, flags=B.PLAN_GRAPH if graph else 0)
    og, ol = oracle.step(c["dims"], c["aggr"], mode == "bf16", blocks, part, K, ks, params, feats, labels, scale)
    for rep in range(2):             # replay: graph / arenas reused across steps
        grad = torch.zeros_like(P)
        loss = torch.zeros(1, device="cuda")
        B.betty_step(ctx, plan, P, X, Y, scale, grad, loss)
        B.betty_sync_check(ctx)
        assert_grad_close(grad.cpu().numpy(), og, c["dims"], c["aggr"], RTOL[mode], f"grad rep={rep}")
        assert loss.item() == pytest.approx(ol, rel=RTOL[mode])
    info = plan.info()
    assert info["kernels_per_step"] > 0
    plan.free()


@pytest.mark.parametrize("mode", ["fp32", "bf16"])
@pytest.mark.parametrize("c", [CASES[0], CASES[4], CASES[11]], ids=lambda c: c["name"])
def test_step_degenerate_inputs(B, ctx, c, mode):
    """Degenerate cases of the method through the fused step (graph replay): a sparse graph whose
    sampled rows are often empty (D_v = 0: h_N = 0, readings #12, #14, S1), micro-batches
    with no outputs at all (labels 1, 3, 4 of K = 6 unused, reading #10), a ragged last launch group (4 + 2), and
    a plan whose every micro-batch is empty (zero gradient, zero loss)."""
    n, pairs, n_out = 600, 150, 60
    F = c["dims"][0]
    ld = (F + 7) // 8 * 8
    g, sd, blocks, feats, _ = tiny(n=n, pairs=pairs, fanouts=c["fanouts"], n_out=n_out, F=F, C=c["dims"][-1],
                                   seed=5, ld=ld)
    empty_rows = sum(int(np.sum(np.diff(b.indptr) == 0)) for b in blocks)
    assert empty_rows > 0                               # the case really has rows with D_v = 0
    labels = (np.arange(n) * 5 % c["dims"][-1]).astype(np.int32)
    params = synth.init_params(c["dims"], c["aggr"], seed=5)
    K = 6
    part = np.array([(0, 2, 5)[i % 3] for i in range(len(sd))], dtype=np.int32)
    dev = B.blocks_to_device(blocks)
    dpart = torch.as_tensor(part).cuda()
    model = B.Model(c["dims"], c["aggr"], mode, mode)
    P = torch.as_tensor(params).cuda()
    X = dev_feats(feats, mode)
    Y = torch.as_tensor(labels).cuda()
    scale = 1.0 / len(sd)
    for ks, group in (([0, 1, 2, 3, 4, 5], 4), ([1, 3], 0)):
        plan = B.betty_plan_create(ctx, model, dev, dpart, K, ks, group=group, flags=B.PLAN_GRAPH)
        og, ol = oracle.step(c["dims"], c["aggr"], mode == "bf16", blocks, part, K, ks, params, feats, labels, scale)
        for rep in range(2):
            grad = torch.zeros_like(P)
            loss = torch.zeros(1, device="cuda")
            B.betty_step(ctx, plan, P, X, Y, scale, grad, loss)
            B.betty_sync_check(ctx)
            if not np.any(og):
                assert not torch.any(grad).item() and loss.item() == 0.0
            else:
                assert_grad_close(grad.cpu().numpy(), og, c["dims"], c["aggr"], RTOL[mode], f"ks={ks} rep={rep}")
                assert loss.item() == pytest.approx(ol, rel=RTOL[mode])
        plan.free()


@pytest.mark.parametrize("mode", ["fp32", "bf16"])
@pytest.mark.parametrize("c", [CASES[1], CASES[2], CASES[11]], ids=lambda c: c["name"])
def test_fresh_plan_follows_the_buffers(B, ctx, c, mode):
    """BETTY_PLAN_FRESH (the e2e path): every step re-derives the full-batch CSCs, the REG's CSC and
    the edge -> gid array from the CURRENT block buffers.  (1) A different batch of the same sizes is
    written into the bound buffers -- the input layer's source node ids permuted (other feature rows,
    same structure) -- and the next steps must match the oracle on the NEW blocks.  (2) A batch that
    outgrows the plan's capacities (every output row's neighbours shifted by one source position)
    must either fit and match the oracle or fail cleanly with EOVERFLOW at the synchronising call."""
    import dataclasses
    sd, blocks, feats, labels, params = make_case(c, seed=4)
    K = 5
    part = synth.random_partition(len(sd), K, 13)
    ks = [0, 1, 2, 3, 4]
    dev = B.blocks_to_device(blocks)
    dpart = torch.as_tensor(part).cuda()
    model = B.Model(c["dims"], c["aggr"], mode, mode)
    P = torch.as_tensor(params).cuda()
    X = dev_feats(feats, mode)
    Y = torch.as_tensor(labels).cuda()
    scale = 1.0 / len(sd)
    plan = B.betty_plan_create(ctx, model, dev, dpart, K, ks, group=0,
                               flags=B.PLAN_GRAPH | B.PLAN_REG | B.PLAN_FRESH)

    def run(bl):
        og, ol = oracle.step(c["dims"], c["aggr"], mode == "bf16", bl, part, K, ks, params, feats, labels, scale)
        for rep in range(2):
            grad = torch.zeros_like(P)
            loss = torch.zeros(1, device="cuda")
            B.betty_step(ctx, plan, P, X, Y, scale, grad, loss)
            B.betty_sync_check(ctx)
            assert_grad_close(grad.cpu().numpy(), og, c["dims"], c["aggr"], RTOL[mode], f"rep={rep}")
            assert loss.item() == pytest.approx(ol, rel=RTOL[mode])

    run(blocks)
    # (1) the input layer's sources are other nodes: permute the src ids beyond the dst prefix
    b0 = blocks[0]
    rng = np.random.default_rng(7)
    gid = b0.src_gid.copy()
    tail = gid[b0.n_dst:].copy()
    gid[b0.n_dst:] = rng.permutation(tail)
    moved = blocks[:]
    moved[0] = dataclasses.replace(b0, src_gid=gid)
    dev[0].src_gid.copy_(torch.as_tensor(gid))
    og_new, _ = oracle.step(c["dims"], c["aggr"], mode == "bf16", moved, part, K, ks, params, feats, labels, scale)
    og_old, _ = oracle.step(c["dims"], c["aggr"], mode == "bf16", blocks, part, K, ks, params, feats, labels, scale)
    assert np.abs(og_new - og_old).max() > 1e-3              # the change is visible in the gradient
    run(moved)
    # (2) a batch beyond the plan's capacities: clean EOVERFLOW (no fault), or it fits and matches
    top = moved[-1]
    shifted = moved[:-1] + [dataclasses.replace(
        top, nbr_pos=((top.nbr_pos.astype(np.int64) + 1) % top.n_src).astype(np.int32))]
    dev[-1].indices.copy_(torch.as_tensor(shifted[-1].nbr_pos))
    try:
        run(shifted)
    except B.BettyError as e:
        assert "EOVERFLOW" in str(e), str(e)
    plan.free()


def test_sum_of_micro_batches_equals_full_batch_on_gpu(B, ctx):
    """Betty's invariant on the GPU path itself: K=8 step == K=1 step (fp32)."""
    c = CASES[1]
    sd, blocks, feats, labels, params = make_case(c, seed=3)
    dev = B.blocks_to_device(blocks)
    model = B.Model(c["dims"], "mean", "fp32")
    P = torch.as_tensor(params).cuda()
    X = dev_feats(feats, "fp32")
    Y = torch.as_tensor(labels).cuda()
    res = []
    for K in (1, 8):
        part = torch.as_tensor(synth.random_partition(len(sd), K, 1)).cuda()
        plan = B.betty_plan_create(ctx, model, dev, part, K, list(range(K)), group=3)
        grad = torch.zeros_like(P)
        loss = torch.zeros(1, device="cuda")
        B.betty_step(ctx, plan, P, X, Y, 1.0 / len(sd), grad, loss)
        torch.cuda.synchronize()
        res.append((grad.cpu().numpy(), loss.item()))
        plan.free()
    assert_grad_close(res[1][0], res[0][0], c["dims"], "mean", 1e-5, "sum_k g_k vs g_full")
    assert res[1][1] == pytest.approx(res[0][1], rel=1e-5)


def test_adam_matches_torch(B, ctx):
    n = 10007
    g = torch.randn(n, device="cuda")
    p0 = torch.randn(n, device="cuda")
    p, m, v = p0.clone(), torch.zeros(n, device="cuda"), torch.zeros(n, device="cuda")
    ref = p0.clone().requires_grad_(True)
    opt = torch.optim.Adam([ref], lr=1e-3)
    for t in range(1, 4):
        B.betty_adam(ctx, p, g, m, v, t)
        ref.grad = g.clone()
        opt.step()
    torch.cuda.synchronize()
    torch.testing.assert_close(p, ref.detach(), rtol=1e-5, atol=1e-6)


# --------------------------------------------- Cora-shaped config (C1) end to end
def test_c1_cora_config(B, ctx):
    cfg = synth.CONFIGS["C1"]
    ds = synth.make(cfg)
    reg_equal(B, ctx, B.blocks_to_device(ds.blocks)[-1], ds.blocks[-1])
    part = synth.random_partition(cfg.n_out, 2, 3)
    dev = B.blocks_to_device(ds.blocks)
    dpart = torch.as_tensor(part).cuda()
    for mode in ("fp32", "bf16"):
        model = B.Model(cfg.dims, "mean", mode, mode)
        params = synth.init_params(cfg.dims, "mean")
        plan = B.betty_plan_create(ctx, model, dev, dpart, 2, [0, 1], group=1)
        grad = torch.zeros(len(params), device="cuda")
        loss = torch.zeros(1, device="cuda")
        B.betty_step(ctx, plan, torch.as_tensor(params).cuda(), dev_feats(ds.feats, mode),
                     torch.as_tensor(ds.labels).cuda(), 1.0 / cfg.n_out, grad, loss)
        torch.cuda.synchronize()
        og, ol = oracle.step(cfg.dims, "mean", mode == "bf16", ds.blocks, part, 2, [0, 1], params, ds.feats,
                             ds.labels, 1.0 / cfg.n_out)
        assert_grad_close(grad.cpu().numpy(), og, cfg.dims, "mean", RTOL[mode], f"C1 grad {mode}")
        assert loss.item() == pytest.approx(ol, rel=RTOL[mode])
        plan.free()


@pytest.mark.parametrize("pos8", ["0", "1"])
@pytest.mark.parametrize("mode", ["fp32", "bf16"])
def test_pool_byte_positions(B, ctx, mode, pos8, monkeypatch):
    """Both argmax encodings of the pool layers (plan path): byte positions in the row (default) and
    int32 source ids (BETTY_POOL_POS8=0) route the gradient like the oracle."""
    monkeypatch.setenv("BETTY_POOL_POS8", pos8)
    c = CASES[5]
    sd, blocks, feats, labels, params = make_case(c, seed=3)
    K = 3
    part = synth.random_partition(len(sd), K, 5)
    dev = B.blocks_to_device(blocks)
    model = B.Model(c["dims"], c["aggr"], mode, mode)
    P = torch.as_tensor(params).cuda()
    plan = B.betty_plan_create(ctx, model, dev, torch.as_tensor(part).cuda(), K, [0, 1, 2], group=0, flags=0)
    grad = torch.zeros_like(P)
    loss = torch.zeros(1, device="cuda")
    B.betty_step(ctx, plan, P, dev_feats(feats, mode), torch.as_tensor(labels).cuda(), 1.0 / len(sd), grad, loss)
    B.betty_sync_check(ctx)
    og, ol = oracle.step(c["dims"], c["aggr"], mode == "bf16", blocks, part, K, [0, 1, 2], params, feats, labels,
                         1.0 / len(sd))
    assert_grad_close(grad.cpu().numpy(), og, c["dims"], c["aggr"], RTOL[mode], "grad")
    plan.free()
