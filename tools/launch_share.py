#!/usr/bin/env python3
"""Per-kernel share of device time from an ncu --metrics gpu__time_duration.sum --csv launch list."""
import csv
import sys
from collections import defaultdict


def main(path, skip_plan=True):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if r and r[0] == "ID"][0]
    h = rows[hi]
    ki, mi, vi, ui = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("Metric Unit")
    tot = defaultdict(float)
    cnt = defaultdict(int)
    for r in rows[hi + 1:]:
        if r[mi] != "gpu__time_duration.sum":
            continue
        v = float(r[vi].replace(",", ""))
        scale = {"ns": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3, "nsecond": 1e-3}.get(r[ui], 1.0)
        name = r[ki].split("(")[0].replace("void ", "")
        tot[name] += v * scale
        cnt[name] += 1
    T = sum(tot.values())
    print(f"{'kernel':60s} {'launches':>8s} {'total_us':>12s} {'avg_us':>10s} {'share':>7s}")
    for k in sorted(tot, key=tot.get, reverse=True):
        print(f"{k[:60]:60s} {cnt[k]:8d} {tot[k]:12.1f} {tot[k]/cnt[k]:10.2f} {100*tot[k]/T:6.2f}%")


if __name__ == "__main__":
    main(sys.argv[1])
