#!/usr/bin/env python
"""Miniblock ablation: GPU-FOR with 4 miniblocks of 32 per
128-value block vs one bitwidth per block ("bit-packing without miniblocks"; paper V100: 2.0 vs
2.1 ms for 500M U(0,2^16)).  Footprint (bits/int) and decode->sum / decode->global kernel times
(CUDA events, median of --reps after an L2 flush) at --rows, parity (sum == int64 sum, decode ==
input) at every point.

  python scripts/bench_nomb.py [--rows 500000000] [--out profiles/r01_nomb.json]
"""
import argparse
import json
import os
import statistics
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import datagen  # noqa: E402


def skewed(n, seed=8000):
    """6-bit values with 0.1 % 20-bit outliers: one outlier widens its whole block without
    miniblocks, only its 32-entry miniblock with them"""
    rng = np.random.default_rng(seed)
    x = rng.integers(0, 2**6, n, dtype=np.int32)
    k = n // 1000
    x[rng.integers(0, n, k)] = rng.integers(2**19, 2**20, k, dtype=np.int32)
    return x


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rows", type=int, default=500_000_000)
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    import torch
    from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp
    n = args.rows
    dev = torch.device("cuda", 0)
    stream = torch.cuda.current_stream(dev)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    acc = torch.zeros(1, dtype=torch.int64, device=dev)
    peak = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])

    def timed(fn):
        for _ in range(2):
            fn()
        torch.cuda.synchronize()
        ts = []
        for _ in range(args.reps):
            flush.sum()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            fn()
            b.record(stream)
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        return statistics.median(ts)

    res = {"rows": n, "peak_hbm_gbs": peak, "columns": {}}
    cols = [("uniform_b4", lambda: datagen.uniform_bits(4, n)), ("uniform_b16", lambda: datagen.uniform_bits(16, n)),
            ("skewed_6b_outliers", lambda: skewed(n))]
    for name, gen in cols:
        x = gen()
        truth = int(x.astype(np.int64).sum())
        xd = torch.from_numpy(x).to(dev)
        out = torch.empty(n, dtype=torch.int32, device=dev)
        row = {}
        for scheme in ("for", "fornm"):
            h = tp.encode(x, scheme)
            d = h.to_device(dev)

            def s():
                acc.zero_()
                tp.tp_decode_sum(d.col, acc, stream)
            ms_sum = timed(s)
            ok = int(acc.item()) == truth
            ms_g = timed(lambda: tp.tp_decode(d.col, out, stream))
            ok = ok and bool(torch.equal(out, xd))
            cb = h.nbytes()
            row[scheme] = {"compressed_bytes": cb, "bits_per_int": 8 * cb / n, "sum_ms": ms_sum,
                           "sum_hbm_frac": cb / ms_sum / 1e6 / peak, "global_ms": ms_g,
                           "global_hbm_frac": (cb + 4 * n) / ms_g / 1e6 / peak, "parity": ok}
            del d, h
            torch.cuda.empty_cache()
        res["columns"][name] = row
        print(name, json.dumps({k: {q: (round(w, 4) if isinstance(w, float) else w) for q, w in v.items()}
                                for k, v in row.items()}), flush=True)
        del x, xd, out
    res["paper_v100_ms_500M_u16"] = {"for": 2.1, "fornm": 2.0}  # P:916-918, 980-982 (context)
    if args.out:
        json.dump(res, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
