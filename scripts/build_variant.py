#!/usr/bin/env python
"""Build an experiment variant of libtilepack.so with extra -D flags into build_ab/ (the main
library is untouched).  usage: build_variant.py NAME "-DFLAG=1 -DOTHER=2" """
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import __graft_entry__ as ge  # noqa: E402

name, flags = sys.argv[1], sys.argv[2].split()
out = os.path.join(ROOT, "build_ab", name)
os.makedirs(out, exist_ok=True)
cmds, objs = [], []
for s in ge.SOURCES:
    o = os.path.join(out, s + ".o")
    cmds.append([ge.NVCC, *ge.ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O3", *flags,
                 "-I", os.path.join(ROOT, "include"), "-c", os.path.join(ge.CSRC, s), "-o", o])
    objs.append(o)
with ThreadPoolExecutor(len(cmds)) as ex:
    for f in [ex.submit(subprocess.check_call, c) for c in cmds]:
        f.result()
lib = os.path.join(ROOT, "build_ab", f"libtilepack_{name}.so")
subprocess.check_call([ge.NVCC, *ge.ARCH, "-shared", "-o", lib, *objs, "-lpthread"])
print(lib)
