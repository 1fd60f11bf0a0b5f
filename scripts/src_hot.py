#!/usr/bin/env python
"""Aggregate an ncu source page (--print-source cuda,sass --csv) by CUDA source line:
instructions executed and stall samples per line.  usage: src_hot.py report.ncu-rep [N] [launch]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 30
extra = ["--launch-skip", sys.argv[3], "--launch-count", "1"] if len(sys.argv) > 3 else []
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass", *extra],
                     capture_output=True, text=True).stdout
fname, rows = None, []
for r in csv.reader(io.StringIO(out)):
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] in ("Function Name", "Line No"):
        continue
    if r[0] and r[0] != "" and len(r) > 7 and r[2] == "-":
        try:
            rows.append((fname, int(r[0]), r[1].strip()[:70], float(r[7] or 0), float(r[4] or 0)))
        except ValueError:
            pass
ti = sum(x[3] for x in rows)
ts = sum(x[4] for x in rows)
print(f"total instr {ti:.4g}  stall samples {ts:.4g}")
for f, ln, src, ins, st in sorted(rows, key=lambda x: -x[3])[:N]:
    print(f"{ins / ti:6.1%} {st / max(ts, 1):6.1%}  {f}:{ln:<5d} {src}")
