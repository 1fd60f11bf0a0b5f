#!/usr/bin/env python
"""SASS instruction count per source line of one kernel (code-size / I-cache audits), no GPU.
usage: sass_lines.py <lib.so> <kernel-name-substring> [N]"""
import os
import re
import subprocess
import sys
import tempfile
from collections import Counter

lib, pat = sys.argv[1], sys.argv[2]
N = int(sys.argv[3]) if len(sys.argv) > 3 else 25
d = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(lib)], cwd=d, capture_output=True)
for cub in os.listdir(d):
    out = subprocess.run(["nvdisasm", "-g", os.path.join(d, cub)], capture_output=True, text=True).stdout
    fn, cur, cnt, total = None, None, Counter(), 0
    for line in out.splitlines():
        m = re.match(r"\s*\.text\.(\S+):", line)
        if m:
            fn = m.group(1)
            continue
        if not fn or pat not in fn:
            continue
        m = re.search(r'//## File "(.*?)", line (\d+)', line)
        if m:
            cur = (m.group(1).split("/")[-1], int(m.group(2)))
            continue
        if re.match(r"\s+/\*[0-9a-f]{4,}\*/", line):
            total += 1
            if cur:
                cnt[cur] += 1
    if total:
        print(cub, "instructions:", total)
        for k, v in cnt.most_common(N):
            print(f"{v:6d}  {k[0]}:{k[1]}")
