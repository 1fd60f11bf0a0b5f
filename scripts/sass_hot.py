#!/usr/bin/env python
"""Top SASS instructions / regions of an ncu report by executed instructions and stall samples.
usage: ncu -i rep --page source --csv --print-source sass > x.csv; python scripts/sass_hot.py x.csv [N]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
ix = {k: i for i, k in enumerate(hdr)}
data = [r for r in rows[2:] if len(r) == len(hdr)]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 40
tot_i = sum(float(r[ix["Instructions Executed"]] or 0) for r in data)
tot_s = sum(float(r[ix["Warp Stall Sampling (All Samples)"]] or 0) for r in data)
print(f"total warp instr {tot_i:.4g}, stall samples {tot_s:.4g}")
# group by opcode
from collections import Counter
op_i, op_s = Counter(), Counter()
for r in data:
    op = r[ix["Source"]].split()[0] if r[ix["Source"]].split() else "?"
    if op.startswith("@"):
        op = r[ix["Source"]].split()[1]
    op = op.split(".")[0]
    op_i[op] += float(r[ix["Instructions Executed"]] or 0)
    op_s[op] += float(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
print("by opcode (instr share, stall share):")
for op, v in op_i.most_common(25):
    print(f"  {op:10s} {v / tot_i:6.1%}  {op_s[op] / max(tot_s, 1):6.1%}")
stall_cols = [k for k in hdr if k.startswith("stall_")]
agg = Counter()
for r in data:
    for k in stall_cols:
        try:
            agg[k] += float(r[ix[k]] or 0)
        except ValueError:
            pass
print("stall reasons:", ", ".join(f"{k[6:]}={v / max(sum(agg.values()), 1):.1%}" for k, v in agg.most_common(8)))
print("hottest instructions by stall samples:")
for r in sorted(data, key=lambda r: -float(r[ix["Warp Stall Sampling (All Samples)"]] or 0))[:N]:
    print(f"  {r[ix['Address']]:>6} {float(r[ix['Warp Stall Sampling (All Samples)']] or 0):7.0f} "
          f"{float(r[ix['Instructions Executed']] or 0):10.0f}  {r[ix['Source']][:90]}")
