"""Per-launch table from an `ncu --page raw --csv` export (one bench step):
time, DRAM bytes, DRAM/SM/tensor utilisation, warps active, top stall.

    python tools/ncu_table.py gpurun_out/full_TAG_raw.csv [--by-name]
"""
import csv
import io
import sys
from collections import defaultdict

COLS = {
    "t_us": "gpu__time_duration.sum",
    "rd_MB": "dram__bytes_read.sum",
    "wr_MB": "dram__bytes_write.sum",
    "dram%": "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "sm%": "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "l2%": "lts__t_sectors.avg.pct_of_peak_sustained_elapsed",
    "l2hit": "lts__t_sector_hit_rate.pct",
    "warps%": "sm__warps_active.avg.pct_of_peak_sustained_active",
    "tc%": "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
    "regs": "launch__registers_per_thread",
    "grid": "launch__grid_size",
}
UNIT = {"ns": 1e-3, "us": 1.0, "ms": 1e3, "s": 1e6, "byte": 1e-6, "Kbyte": 1e-3, "Mbyte": 1.0, "Gbyte": 1e3}
STALLS = ["long_scoreboard", "lg_throttle", "barrier", "membar", "short_scoreboard", "wait", "math_pipe_throttle",
          "mio_throttle", "no_instruction", "not_selected", "selected", "dispatch_stall", "drain", "sleeping",
          "tex_throttle", "branch_resolving", "imc_miss", "misc"]


def load(path):
    rows = list(csv.reader(io.open(path, encoding="utf-8", errors="replace")))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h, units = rows[hi], rows[hi + 1]
    out = []
    for r in rows[hi + 2:]:
        if len(r) < len(h):
            continue
        d = {"name": r[h.index("Kernel Name")].split("(")[0].replace("void ", "")}
        for k, m in COLS.items():
            if m in h:
                i = h.index(m)
                try:
                    v = float(r[i].replace(",", ""))
                except ValueError:
                    v = float("nan")
                d[k] = v * UNIT.get(units[i], 1.0) if k in ("t_us", "rd_MB", "wr_MB") else v
        best, bv = "", -1.0
        for st in STALLS:
            m2 = f"smsp__average_warps_issue_stalled_{st}_per_issue_active.ratio"
            for mm in (m2,):
                if mm in h:
                    try:
                        v = float(r[h.index(mm)].replace(",", ""))
                    except ValueError:
                        continue
                    if v > bv:
                        best, bv = st, v
        d["stall"] = f"{best}:{bv:.1f}" if best else ""
        out.append(d)
    return out


def main():
    rows = load(sys.argv[1])
    by_name = "--by-name" in sys.argv
    if by_name:
        agg = defaultdict(lambda: defaultdict(float))
        for d in rows:
            a = agg[d["name"]]
            a["n"] += 1
            for k in ("t_us", "rd_MB", "wr_MB"):
                a[k] += d.get(k, 0.0)
        tot = sum(a["t_us"] for a in agg.values())
        print(f"{'kernel':40s} {'n':>3s} {'t_us':>9s} {'share':>6s} {'rd_MB':>9s} {'wr_MB':>9s} {'GB/s':>7s}")
        for k, a in sorted(agg.items(), key=lambda x: -x[1]["t_us"]):
            gbs = (a["rd_MB"] + a["wr_MB"]) / a["t_us"] * 1e-3 * 1e3 if a["t_us"] else 0
            print(f"{k[:40]:40s} {int(a['n']):3d} {a['t_us']:9.1f} {100 * a['t_us'] / tot:5.1f}% {a['rd_MB']:9.1f} "
                  f"{a['wr_MB']:9.1f} {gbs:7.0f}")
        print(f"total {tot:.1f} us")
        return
    print(f"{'#':>3s} {'kernel':34s} {'t_us':>8s} {'rd_MB':>8s} {'wr_MB':>8s} {'dram%':>6s} {'sm%':>5s} {'l2%':>5s} "
          f"{'l2hit':>5s} {'warp%':>5s} {'tc%':>5s} {'regs':>4s} {'grid':>6s}  stall")
    for i, d in enumerate(rows):
        print(f"{i:3d} {d['name'][:34]:34s} {d.get('t_us', 0):8.1f} {d.get('rd_MB', 0):8.1f} {d.get('wr_MB', 0):8.1f} "
              f"{d.get('dram%', 0):6.1f} {d.get('sm%', 0):5.1f} {d.get('l2%', 0):5.1f} {d.get('l2hit', 0):5.1f} "
              f"{d.get('warps%', 0):5.1f} {d.get('tc%', 0):5.1f} {d.get('regs', 0):4.0f} {d.get('grid', 0):6.0f}  "
              f"{d['stall']}")


if __name__ == "__main__":
    main()
