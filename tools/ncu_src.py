"""Top stalled SASS instructions per kernel from an `ncu --page source --csv
--print-source sass` export (optionally gzipped).

    python tools/ncu_src.py gpurun_out/k_TAG_src.csv.gz [kernel-substring] [N]
"""
import csv
import gzip
import io
import sys


def blocks(path):
    f = gzip.open(path, "rt", errors="replace") if path.endswith(".gz") else open(path, errors="replace")
    cur = None
    for r in csv.reader(f):
        if r and r[0] == "Kernel Name":
            cur = {"name": r[1], "rows": []}
            yield cur
            continue
        if r and r[0] == "Address" and cur is not None:
            cur["h"] = r
            continue
        if cur is not None and "h" in cur and len(r) == len(cur["h"]):
            cur["rows"].append(r)


def main():
    path = sys.argv[1]
    sub = sys.argv[2] if len(sys.argv) > 2 else ""
    n = int(sys.argv[3]) if len(sys.argv) > 3 else 25
    for b in list(blocks(path)):
        if sub not in b["name"]:
            continue
        h = b["h"]
        i_s = h.index("Warp Stall Sampling (All Samples)")
        i_src = h.index("Source")
        i_ie = h.index("Instructions Executed")
        tot = sum(float(r[i_s] or 0) for r in b["rows"]) or 1.0
        ie = sum(float(r[i_ie] or 0) for r in b["rows"])
        print(f"== {b['name'][:90]}  samples {tot:.0f}  warp-instr {ie:.3g}")
        for r in sorted(b["rows"], key=lambda r: -float(r[i_s] or 0))[:n]:
            print(f"  {100 * float(r[i_s] or 0) / tot:5.1f}% {float(r[i_ie] or 0):10.0f} {r[0][-5:]} {r[i_src][:100]}")


if __name__ == "__main__":
    main()
