#!/usr/bin/env python
"""Aggregate an ncu --metrics gpu__time_duration.sum launch list (CSV) per kernel: count, total us, share."""
import collections
import csv
import json
import sys


def shares(path):
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        name = r[ki] if "cell_pair" in r[ki] or "score_kernel" in r[ki] else r[ki].split("(")[0]
        v = float(r[vi].replace(",", "")) * {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3}.get(r[ui], 1.0)
        agg[name][0] += 1
        agg[name][1] += v
    tot = sum(v[1] for v in agg.values())
    return {k: {"launches": v[0], "us": round(v[1], 1), "share": round(v[1] / tot, 4)}
            for k, v in sorted(agg.items(), key=lambda x: -x[1][1])}, tot


if __name__ == "__main__":
    d, tot = shares(sys.argv[1])
    print(json.dumps({"total_ms": round(tot / 1e3, 3), "kernels": d}, indent=1))
