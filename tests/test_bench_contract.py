"""The bench line contract (task statement / SURVEY.md §8(d)) on the committed measurement
(profiles/r09_bench_C3.jsonl, written by bench.py on a B200): every key the driver and the judge
read is present with a sane value.  CPU only (reads the committed JSON)."""
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _line(name):
    with open(os.path.join(ROOT, "profiles", name)) as f:
        return json.loads(f.read().strip().splitlines()[-1])


def test_c3_bench_line_contract():
    d = _line("r09_bench_C3.jsonl")
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "e2e", "gpu_launches", "clocks", "roofline", "cpu_baseline"):
        assert k in d, k
    assert d["warmup"] >= 3 and d["steps"] >= 1 and d["n_gpus"] == 1
    assert d["higher_is_better"] is True and d["unit"] == "edges/s" and d["data"] == "synthetic"
    assert d["vs_baseline"] is None                     # BASELINE.md has no number for this metric
    assert d["config"]["workload"].startswith("C3") and "l2" in d["config"]
    # value = aggregated edges / epoch time
    assert abs(d["value"] - d["edges_per_step"] / (d["ms_per_step"] * 1e-3)) < 1e-6 * d["value"]
    e = d["e2e"]
    assert e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0 and 0 < e["value"] < d["value"]
    assert e["input_buffers"] in (1, 2)
    r = d["roofline"]
    assert r["bound"] == "hbm" and r["unit"] == "GB/s" and 0 < r["frac"] < 1
    assert abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-9
    assert r["traffic"] is not None and r["traffic"] > 0
    c = d["cpu_baseline"]
    assert c["kind"] == "oracle" and c["cores"] >= 1 and c["value"] > 0 and c["sample"]
    assert d["gpu_launches"] > 0 and not set(d["clocks"]["reasons"]) & {"hw_slowdown", "hw_thermal_slowdown",
                                                                         "sw_thermal_slowdown"}
    # round 2: the paper's precision (fp32, 3xTF32 GEMMs) beside the bf16 headline, with its own roofline;
    # e2e through BETTY_PLAN_FRESH plans; the §8(d) roofline bytes; the oracle on every host core
    p = d["paper_precision"]
    assert p["dtype"].startswith("fp32") and p["ms_per_step"] > d["ms_per_step"] and p["roofline"]["frac"] > 0
    assert e["fresh_inputs"] is True
    assert r["alg_bytes_formula"].startswith("4E + 8(n_dst+1)")
    assert abs(d["full_batch_edges_per_s"] - d["full_batch_edges"] / (d["ms_per_step"] * 1e-3)) < 1e-6 * d["value"]
    assert c["cores"] > 1
    # the stream form of the aggregation bytes and the row-fetch rate ride along as context only
    st = r["stream"]
    assert st["alg_bytes_per_launch"] > r["alg_bytes_per_launch"] and 0 < st["frac"] < 1
    assert r["row_fetches_per_ns"] > 0
    assert e["loss_reads"] >= 1                         # every e2e step's loss read on the host


def test_other_config_lines():
    for name, cfg in (("r08_bench_C4.jsonl", "C4"), ("r08_bench_C5.jsonl", "C5"), ("r08_bench_C1.jsonl", "C1"),
                      ("r08_bench_C2.jsonl", "C2")):
        d = _line(name)
        assert d["config"]["workload"].startswith(cfg) and d["value"] > 0 and d["ms_per_step"] > 0
