#!/usr/bin/env python3
"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv): per-kernel totals.

  python scripts/launch_summary.py launches.csv [--last-fraction F]
"""
import collections
import csv
import sys


def main():
    f = sys.argv[1]
    frac = float(sys.argv[sys.argv.index("--last-fraction") + 1]) if "--last-fraction" in sys.argv else 1.0
    rows = [r for r in csv.reader(open(f)) if len(r) > 10]
    h = rows[0]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    data = rows[1:]
    data = data[int(len(data) * (1 - frac)):]
    scale = {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3, "s": 1e6, "second": 1e6}
    d = collections.OrderedDict()
    tot = 0.0
    for r in data:
        v = float(r[vi].replace(",", "")) * scale.get(r[ui], 1.0)
        name = r[ki].split("(")[0][:44]
        c, s = d.get(name, (0, 0.0))
        d[name] = (c + 1, s + v)
        tot += v
    print(f"{'kernel':46s} {'launches':>8s} {'total ms':>10s} {'us/launch':>10s} {'share':>7s}")
    for k, (c, s) in sorted(d.items(), key=lambda x: -x[1][1]):
        print(f"{k:46s} {c:8d} {s / 1e3:10.3f} {s / c:10.1f} {100 * s / tot:6.1f}%")
    print(f"total {tot / 1e3:.3f} ms over {sum(c for c, _ in d.values())} launches")


if __name__ == "__main__":
    main()
