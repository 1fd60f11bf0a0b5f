#!/usr/bin/env python
"""A/B of tp_decode_sum between two builds of the library on one box (alternating processes).
usage: ab_decode.py LIB_A LIB_B [bits] [reps]   (runs itself in child processes)"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def child(bits):
    sys.path.insert(0, ROOT)
    import numpy as np
    import torch
    import datagen
    from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp
    x = datagen.uniform_bits(bits, 500_000_000, seed=2000 + bits)
    d = tp.encode(x, "for").to_device()
    acc = torch.zeros(1, dtype=torch.int64, device="cuda")
    for _ in range(5):
        tp.tp_decode_sum(d.col, acc)
    torch.cuda.synchronize()
    ts = []
    for _ in range(50):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        tp.tp_decode_sum(d.col, acc)
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    print("ms", float(np.median(ts)), float(np.mean(ts)))


if __name__ == "__main__":
    if sys.argv[1] == "--child":
        child(int(sys.argv[2]))
        sys.exit(0)
    libs = [a for a in sys.argv[1:] if a.endswith(".so")]
    rest = [a for a in sys.argv[1:] if not a.endswith(".so")]
    bits = rest[0] if rest else "16"
    reps = int(rest[1]) if len(rest) > 1 else 3
    for r in range(reps):
        for lib in libs:
            env = dict(os.environ, TILEPACK_LIB_OVERRIDE=os.path.abspath(lib))
            out = subprocess.run([sys.executable, __file__, "--child", bits], env=env, capture_output=True, text=True)
            print(os.path.basename(lib), bits, out.stdout.strip().splitlines()[-1] if out.stdout.strip() else out.stderr[-300:], flush=True)
