#!/usr/bin/env python
"""Instruction mix and warp-stall samples by SASS opcode of one kernel launch (ncu source page CSV).

usage: ncu -i R.ncu-rep --page source --csv --print-source sass --launch-count 1 > s.csv
       tools/ncu_source_mix.py s.csv [--out profiles/x.json]
"""
import argparse
import csv
import json
from collections import defaultdict

ap = argparse.ArgumentParser()
ap.add_argument("csv")
ap.add_argument("--out")
args = ap.parse_args()
rows = list(csv.reader(open(args.csv)))
kernel = rows[0][1]
hdr = rows[1]
ix = {h: i for i, h in enumerate(hdr)}
stall_cols = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
inst = defaultdict(float)
samp = defaultdict(float)
stalls = defaultdict(float)
tot_i = tot_s = 0.0
for r in rows[2:]:
    if r and r[0] == "Kernel Name":
        break  # the next launch of the report: this summary covers the first one only
    if len(r) != len(hdr):
        continue
    op = r[ix["Source"]].strip().split()
    if not op:
        continue
    o = op[0]
    if o.startswith("@"):
        o = op[1] if len(op) > 1 else o
    o = o.split(".")[0]
    i = float(r[ix["Instructions Executed"]] or 0)
    s = float(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
    inst[o] += i
    samp[o] += s
    tot_i += i
    tot_s += s
    for c in stall_cols:
        stalls[c[6:]] += float(r[ix[c]] or 0)
top = sorted(inst, key=lambda k: -inst[k])[:24]
out = {"kernel": kernel, "inst_executed": tot_i, "stall_samples": tot_s,
       "by_opcode": {k: {"inst_share": round(inst[k] / tot_i, 4), "sample_share": round(samp[k] / tot_s, 4)}
                     for k in top},
       "stalls": {k: round(v / tot_s, 4) for k, v in sorted(stalls.items(), key=lambda kv: -kv[1]) if v > 0}}
s = json.dumps(out, indent=1)
if args.out:
    open(args.out, "w").write(s + "\n")
print(s)
