"""Summarise an ncu launch list (`--metrics gpu__time_duration.sum[,dram__bytes_*]
--csv --log-file ...`) of ONE step (tools/prof_step.py profiles exactly one):
per kernel name: launches, serialised time, share, DRAM bytes.

    python tools/launch_summary.py gpurun_out/launches_TAG.csv
"""
import csv
import sys
from collections import OrderedDict, defaultdict

UNIT = {"nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3, "ns": 1e-3, "us": 1.0, "ms": 1e3,
        "byte": 1e-6, "Kbyte": 1e-3, "Mbyte": 1.0, "Gbyte": 1e3}


def main(path):
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    iid, ik, im, iu, iv = (h.index(x) for x in ("ID", "Kernel Name", "Metric Name", "Metric Unit", "Metric Value"))
    launches = OrderedDict()
    for r in rows[hi + 1:]:
        if len(r) <= iv:
            continue
        d = launches.setdefault(r[iid], {"name": r[ik].split("(")[0].replace("void ", "").split("<")[0]})
        d[r[im]] = float(r[iv].replace(",", "")) * UNIT.get(r[iu], 1.0)
    agg = defaultdict(lambda: [0, 0.0, 0.0, 0.0])
    for d in launches.values():
        a = agg[d["name"]]
        a[0] += 1
        a[1] += d.get("gpu__time_duration.sum", 0.0)
        a[2] += d.get("dram__bytes_read.sum", 0.0)
        a[3] += d.get("dram__bytes_write.sum", 0.0)
    tot = sum(a[1] for a in agg.values())
    print(f"one step: {len(launches)} launches, {tot / 1e3:.3f} ms serialised (ncu; cache control as launched: launches.sh CACHE, default all = cold)")
    print(f"{'kernel':34s} {'n':>3s} {'us':>9s} {'share':>6s} {'rd MB':>9s} {'wr MB':>9s}")
    for k, a in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"{k[:34]:34s} {a[0]:3d} {a[1]:9.1f} {100 * a[1] / tot:5.1f}% {a[2]:9.1f} {a[3]:9.1f}")


if __name__ == "__main__":
    main(sys.argv[1])
