"""GPU parity of §4.4 memory-aware partitioning: the
count-only extraction equals the oracle's micro-batch sizes bit-exactly, and
betty_memory_aware_k picks the same K, partition and peak as the oracle's
loop fed the same partitioner."""
import numpy as np
import pytest
import torch

import oracle
import synth
from tests.helpers import tiny

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def B():
    import paper_conf_asplos_yangzd023_b200 as B
    assert torch.cuda.is_available()
    return B


@pytest.fixture(scope="module")
def ctx(B):
    return B.betty_ctx_create(0)


def oracle_sizes(blocks, part, K):
    out = np.zeros((K, len(blocks), 3), dtype=np.int64)
    for k in range(K):
        for l, b in enumerate(oracle.extract(blocks, part, K, k)):
            out[k, l] = (b.n_dst, b.n_src, b.n_edges)
    return out


@pytest.mark.parametrize("K,kind", [(1, "range"), (3, "random"), (7, "random"), (40, "random")])
def test_mb_sizes(B, ctx, K, kind):
    g, sd, blocks, feats, labels = tiny(n=2000, pairs=9000, fanouts=(3, 5, 6), n_out=120, n_comm=10, seed=8)
    part = synth.range_partition(120, K) if kind == "range" else synth.random_partition(120, K, 9)
    dev = B.blocks_to_device(blocks)
    got = B.betty_mb_sizes(ctx, dev, torch.as_tensor(part).cuda(), K)
    np.testing.assert_array_equal(got, oracle_sizes(blocks, part, K))


def test_mb_sizes_c1(B, ctx):
    ds = synth.make(synth.CONFIGS["C1"])
    part = synth.random_partition(ds.cfg.n_out, 2, 3)
    got = B.betty_mb_sizes(ctx, B.blocks_to_device(ds.blocks), torch.as_tensor(part).cuda(), 2)
    np.testing.assert_array_equal(got, oracle_sizes(ds.blocks, part, 2))


@pytest.mark.parametrize("aggr,dims", [("mean", [5, 16, 3]), ("pool", [5, 8, 8, 3])])
def test_memory_aware_k(B, ctx, aggr, dims):
    fan = (3, 5) if len(dims) == 3 else (3, 4, 5)
    g, sd, blocks, feats, labels = tiny(n=1500, pairs=6000, fanouts=fan, n_out=90, n_comm=9, seed=12)
    reg = oracle.reg(blocks[-1].n_src, blocks[-1].indptr, blocks[-1].nbr_pos)
    fn = lambda K: B.betty_reg_partition(*reg, K, method="multilevel")
    dev = B.blocks_to_device(blocks)
    model = B.Model(dims, aggr)
    full_peak = int(oracle.mem_estimate(dims, aggr, blocks)[8])
    for frac in (1.0, 0.8, 0.6, 0.45):
        cap = int(full_peak * frac)
        ko, po, peak_o = oracle.memory_aware_k(blocks, dims, aggr, cap, fn, K_max=30)
        k, p, peak = B.betty_memory_aware_k(ctx, model, dev, reg, 4 * cap, K_max=30)
        assert k == ko, (frac, k, ko)
        assert peak == 4 * peak_o
        if k > 0:
            np.testing.assert_array_equal(p, po)
