"""Write profiles/traffic.json: ncu DRAM bytes (read + write) per launch of the
bench's dominant kernel, from an `ncu --page raw --csv` export of one step.

    python tools/traffic.py gpurun_out/full_TAG_raw.csv KERNEL_REGEX KEY SITE
    e.g. ... 'k_agg_mean' C3:K32:bf16:n1 agg_l0
"""
import csv
import json
import os
import re
import sys

UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}


def main(path, regex, key, site):
    rows = list(csv.reader(open(path)))
    h, units = rows[0], rows[1]
    ik = h.index("Kernel Name")
    ir, iw = h.index("dram__bytes_read.sum"), h.index("dram__bytes_write.sum")
    tot, n = 0.0, 0
    for r in rows[2:]:
        if re.search(regex, r[ik]):
            tot += float(r[ir].replace(",", "")) * UNIT[units[ir]] + float(r[iw].replace(",", "")) * UNIT[units[iw]]
            n += 1
    out = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "traffic.json")
    d = json.load(open(out)) if os.path.exists(out) else {}
    d.setdefault(key, {})[site] = tot / max(n, 1)
    d["_source"] = "ncu --set full --clock-control none, one bench step (tools/prof_step.py); bytes per launch"
    json.dump(d, open(out, "w"), indent=1)
    print(key, site, tot / max(n, 1), "bytes/launch over", n, "launches")


if __name__ == "__main__":
    main(*sys.argv[1:5])
