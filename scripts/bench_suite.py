#!/usr/bin/env python
"""Per-configuration decode measurements (BASELINE configs 2-4) on one GPU.

For every column: decode->sum and decode->global kernel times (CUDA events, median of
--reps after an L2 flush), compressed bytes, bits/int, HBM fractions, and a full-size
parity check (sum == plain int64 sum; decoded column == the generated column).

  python scripts/bench_suite.py [--rows 500000000] [--only for|dfor|rfor] [--out profiles/x.json]
"""
import argparse
import json
import os
import statistics
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import datagen  # noqa: E402


def configs(rows, only, bits):
    out = []
    if only in (None, "for"):
        for b in bits:
            out.append((f"for_b{b}", "for", lambda b=b: datagen.uniform_bits(b, rows)))
    if only in (None, "dfor"):
        out += [("dfor_d1_2^28", "dfor", lambda: datagen.d1_sorted(rows, 2**28)),
                ("dfor_sorted_uniform", "dfor", lambda: datagen.sorted_uniform(rows)),
                ("dfor_near_sorted", "dfor", lambda: datagen.near_sorted(rows)),
                ("dfor_consecutive", "dfor", lambda: datagen.consecutive(rows))]
    if only in (None, "rfor"):
        for L in (4, 8, 16, 32, 64):
            out.append((f"rfor_runs{L}", "rfor", lambda L=L: datagen.runs(rows, L)))
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rows", type=int, default=500_000_000)
    ap.add_argument("--only", default=None)
    ap.add_argument("--bits", default="0,1,2,3,4,6,8,10,12,14,16,20,24,28,32")
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--out", default=None)
    ap.add_argument("--no-global", action="store_true")
    args = ap.parse_args()
    import torch
    from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp
    peak = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])
    dev = torch.device("cuda", 0)
    stream = torch.cuda.current_stream(dev)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    acc = torch.zeros(1, dtype=torch.int64, device=dev)
    res = {"rows": args.rows, "peak_hbm_gbs": peak, "configs": {}}
    bits = [int(b) for b in args.bits.split(",")]
    for name, scheme, gen in configs(args.rows, args.only, bits):
        t0 = time.time()
        x = gen()
        h = tp.encode(x, scheme)
        d = h.to_device(dev)
        cb = h.nbytes()
        truth = int(x.astype(np.int64).sum())

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

        def do_sum():
            acc.zero_()
            tp.tp_decode_sum(d.col, acc, stream)
        ms_sum = timed(do_sum)
        ok_sum = int(acc.item()) == truth
        r = {"scheme": scheme, "compressed_bytes": cb, "bits_per_int": 8 * cb / args.rows,
             "sum_ms": ms_sum, "sum_decoded_gbs": 4 * args.rows / ms_sum / 1e6,
             "sum_hbm_gbs": cb / ms_sum / 1e6, "sum_hbm_frac": cb / ms_sum / 1e6 / peak, "sum_parity": ok_sum}
        if not args.no_global:
            out = torch.empty(args.rows, dtype=torch.int32, device=dev)
            ms_g = timed(lambda: tp.tp_decode(d.col, out, stream))
            xd = torch.from_numpy(x).to(dev)
            r.update({"global_ms": ms_g, "global_decoded_gbs": 4 * args.rows / ms_g / 1e6,
                      "global_hbm_frac": (cb + 4 * args.rows) / ms_g / 1e6 / peak,
                      "global_parity": bool(torch.equal(out, xd))})
            del out, xd
        r["setup_s"] = time.time() - t0
        res["configs"][name] = r
        print(name, json.dumps({k: (round(v, 4) if isinstance(v, float) else v) for k, v in r.items()}), flush=True)
        del d, h, x
        torch.cuda.empty_cache()
    if args.out:
        json.dump(res, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
