#!/bin/bash
# usage: scripts/ncu_export.sh <name> -- export an .ncu-rep (gpurun_out/<name>.ncu-rep) to text pages
# (details, raw csv, source csv with SASS) so the report itself need not travel back
set -e
R=gpurun_out/$1.ncu-rep
ncu -i $R --page details > gpurun_out/$1.details.txt 2>&1 || true
ncu -i $R --page raw --csv > gpurun_out/$1.raw.csv 2>&1 || true
ncu -i $R --page source --csv --print-source sass > gpurun_out/$1.sass.csv 2>&1 || true
ncu -i $R --page source --csv --print-source cuda > gpurun_out/$1.cuda.csv 2>&1 || true
gzip -f gpurun_out/$1.sass.csv || true
