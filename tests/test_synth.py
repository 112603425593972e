"""Input generator (synth/) pieces the large configurations rely on: feature rows generated on their
own (row ranges for C5's chunked table, id lists for an oracle sample) equal the whole table's rows,
and the oracle fed only a sample's rows (bench.oracle_inputs) computes what it computes on the
whole table."""
import numpy as np

import oracle
import synth


def test_feature_rows_equal_table():
    cfg = synth.scaled(synth.CONFIGS["C5"], 0.0005)
    ds = synth.make(cfg)
    comm = ds.graph.comm
    for r0, n in ((0, 1), (17, 500), (cfg.n - 3, 3)):
        np.testing.assert_array_equal(synth.features_rows(comm, cfg.F, cfg.ld, row0=r0, n=n), ds.feats[r0:r0 + n])
    ids = np.array([cfg.n - 1, 0, 5, 5, 1234], np.int32)
    np.testing.assert_array_equal(synth.features_rows(comm, cfg.F, cfg.ld, ids=ids), ds.feats[ids])


def test_c5_preset_shape():
    c = synth.CONFIGS["C5"]
    assert (c.n, c.F, c.C, c.L, tuple(c.fanouts), c.n_out) == (111059956, 128, 172, 3, (5, 10, 15), 1207179)
    assert c.dims == [128, 256, 256, 172] and c.ld == 128
    assert c.n * c.ld * 4 > synth.HOST_FEATURE_LIMIT          # generated in chunks, never on the host


def test_oracle_on_sample_rows_equals_whole_table():
    import bench
    cfg = synth.scaled(synth.CONFIGS["C5"], 0.0005)
    ds = synth.make(cfg)
    part = np.ones(cfg.n_out, np.int32)
    part[:7] = 0
    params = synth.init_params(cfg.dims, cfg.aggr, seed=cfg.seeds["init"])
    want = oracle.step(cfg.dims, cfg.aggr, True, ds.blocks, part, 2, [0], params, ds.feats, ds.labels, 0.01)
    no_host = synth.Dataset(cfg, ds.graph, None, ds.labels, ds.seeds, ds.blocks)
    blocks, feats = bench.oracle_inputs(cfg, no_host, part)
    assert feats.shape[0] < cfg.n
    got = oracle.step(cfg.dims, cfg.aggr, True, blocks, part, 2, [0], params, feats, ds.labels, 0.01)
    np.testing.assert_array_equal(got[0], want[0])
    assert got[1] == want[1]
