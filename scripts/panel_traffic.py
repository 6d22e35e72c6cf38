#!/usr/bin/env python3
"""ncu per-launch DRAM bytes of every panel launch -> profiles/panel_traffic.json (bench.py's
roofline `traffic`).

  python scripts/panel_traffic.py panel_traffic.csv N NB [out.json]

Input: `ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum
--clock-control none -k regex:k_panel --csv` of one reduction (ncu flushes caches per launch:
cold-cache traffic)."""
import collections
import csv
import json
import sys


def main():
    f, n, nb = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
    out = sys.argv[4] if len(sys.argv) > 4 else "profiles/panel_traffic.json"
    rows = [r for r in csv.reader(open(f)) if len(r) > 10]
    h = rows[0]
    ii, mi, vi, ui = h.index("ID"), h.index("Metric Name"), h.index("Metric Value"), h.index("Metric Unit")
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}
    per = collections.OrderedDict()
    for r in rows[1:]:
        if r[mi].startswith("dram__bytes"):
            per[r[ii]] = per.get(r[ii], 0.0) + float(r[vi].replace(",", "")) * scale.get(r[ui], 1)
    vals = list(per.values())
    json.dump({"n": n, "nb": nb, "launches": len(vals), "dram_bytes_per_launch": sum(vals) / max(len(vals), 1),
               "source": "ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum (cold cache per launch: ncu "
                         "flushes caches), every k_panel launch of one ABFT reduction (scripts/profile.sh)",
               "per_launch_bytes": vals}, open(out, "w"), indent=1)
    print(f"{len(vals)} launches, mean {sum(vals) / max(len(vals), 1):.0f} bytes")


if __name__ == "__main__":
    main()
