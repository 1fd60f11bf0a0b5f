#!/usr/bin/env python
"""Random access under a predicate bitvector: 250M-row
columns, selectivity swept 0..1, compressed (GPU-FOR / GPU-DFOR / GPU-RFOR) vs uncompressed
(None).  Kernel time (CUDA events, median of --reps after an L2 flush) of tp_bitmap_sum and
parity with the oracle's plain definition at every point.

  python scripts/bench_random_access.py [--rows 250000000] [--out profiles/r01_random_access.json]
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
import oracle  # noqa: E402  (parity only)

SIGMAS = (0.0, 1e-6, 1e-5, 1e-4, 1 / 512, 1e-2, 1 / 32, 0.1, 0.5, 1.0)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rows", type=int, default=250_000_000)
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
    cols = {"for_b16": ("for", datagen.uniform_bits(16, n)), "none_b16": ("none", datagen.uniform_bits(16, n)),
            "dfor_sorted": ("dfor", datagen.sorted_uniform(n)), "rfor_runs8": ("rfor", datagen.runs(n, 8))}
    dcols = {k: (tp.encode(x, s).to_device(dev), x) for k, (s, x) in cols.items()}
    res = {"rows": n, "peak_hbm_gbs": peak, "points": []}
    for si, sigma in enumerate(SIGMAS):
        bm = datagen.bernoulli_bitmap(n, sigma, seed=7000 + si)
        dbm = torch.from_numpy(bm.view(np.int32)).to(dev)
        for name, (d, x) in dcols.items():
            def run():
                acc.zero_()
                tp.tp_bitmap_sum(d.col, dbm, acc, stream)
            for _ in range(2):
                run()
            torch.cuda.synchronize()
            ts = []
            for _ in range(args.reps):
                flush.sum()
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                run()
                b.record(stream)
                torch.cuda.synchronize()
                ts.append(a.elapsed_time(b))
            ms = statistics.median(ts)
            import time as _t
            t1 = _t.perf_counter()
            want = oracle.bitmap_sum(x, bm)  # the oracle's plain definition, timed beside (numpy, host)
            osec = _t.perf_counter() - t1
            ok = int(acc.item()) == want
            p = {"sigma": sigma, "column": name, "ms": ms, "compressed_bytes": d.nbytes(),
                 "full_scan_frac": (d.nbytes() + n / 8) / ms / 1e6 / peak, "parity": ok,
                 "oracle_ms": osec * 1e3}
            res["points"].append(p)
            print(json.dumps({k: (round(v, 5) if isinstance(v, float) else v) for k, v in p.items()}), flush=True)
    if args.out:
        json.dump(res, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
