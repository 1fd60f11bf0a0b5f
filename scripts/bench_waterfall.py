#!/usr/bin/env python
"""NEXT-2 (Fig. 9 / Fig. 10): every SSB lineorder column at SF 20 --
its footprint under None, GPU-FOR, GPU-DFOR, GPU-RFOR and GPU-* (the smallest),
and the decode time of the GPU-* encoding, tile-based (decode -> global, one pass) against the
cascading model (tp_decode_cascaded, one kernel per layer through global memory; the paper's
nvCOMP comparison, Fig. 10a).  Every GPU decode is checked against the column (exact).

  python scripts/bench_waterfall.py [--sf 20] [--reps 5] [--out profiles/x.json]
"""
import argparse
import json
import math
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sf", type=float, default=20)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    import numpy as np
    import torch
    import datagen.ssb as gen
    from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp
    dev = torch.device("cuda", 0)
    stream = torch.cuda.current_stream(dev)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    peak = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])

    def timed(fn):
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

    db = gen.generate(args.sf, seed=5000, columns=gen.LINEORDER_COLUMNS)
    lo = db["lineorder"]
    n = len(lo["lo_orderkey"])
    out = torch.empty(n, dtype=torch.int32, device=dev)
    acc = torch.zeros(1, dtype=torch.int64, device=dev)
    res = {"sf": args.sf, "rows": n, "columns": {}}
    tot = {"none": 0, "for": 0, "dfor": 0, "rfor": 0, "gpu*": 0}
    speedups = []
    for name in gen.LINEORDER_COLUMNS:
        x = np.ascontiguousarray(lo[name], np.int32)
        sizes = {"none": 4 * n}
        for sc in ("for", "dfor", "rfor"):
            nb, w0, w1 = tp.tp_encode_size(tp.SCHEMES[sc], x)
            sizes[sc] = 4 * (3 + (nb + 1) * (2 if sc == "rfor" else 1) + w0 + w1)
        best, best_bytes = tp.tp_choose_scheme(x)
        scheme = tp.SCHEME_NAMES[best]
        sizes["gpu*"] = best_bytes
        for k in tot:
            tot[k] += sizes[k]
        d = tp.encode(x, scheme).to_device(dev)
        xd = torch.from_numpy(x).to(dev)
        t_tile = timed(lambda: tp.tp_decode(d.col, out, stream))
        ok = bool(torch.equal(out, xd))
        t_sum = timed(lambda: tp.tp_decode_sum(d.col, acc, stream))
        work = torch.empty(max(1, tp.tp_cascaded_workspace_words(d.col)), dtype=torch.int32, device=dev)
        t_casc = timed(lambda: tp.tp_decode_cascaded(d.col, out, work, stream))
        ok = ok and bool(torch.equal(out, xd))
        alg = d.nbytes() + 4 * n  # compressed bytes read + decoded bytes written
        r = {"scheme": scheme, "bytes": sizes, "bits_per_int": {k: 8 * v / n for k, v in sizes.items()},
             "tile_global_ms": t_tile, "tile_sum_ms": t_sum, "cascaded_ms": t_casc, "speedup": t_casc / t_tile,
             "tile_global_hbm_frac": alg / (t_tile / 1e3) / 1e9 / peak, "parity": ok}
        res["columns"][name] = r
        speedups.append(t_casc / t_tile)
        print(name, json.dumps({k: (round(v, 4) if isinstance(v, float) else v) for k, v in r.items()
                                if k not in ("bytes", "bits_per_int")}),
              "bits/int", {k: round(v, 2) for k, v in r["bits_per_int"].items()}, flush=True)
        del d, xd, work
        torch.cuda.empty_cache()
    res["total_bytes"] = tot
    res["footprint_ratio_none_over_gpu*"] = tot["none"] / tot["gpu*"]
    res["decode_speedup_geomean_vs_cascaded"] = math.exp(sum(math.log(s) for s in speedups) / len(speedups))
    print(json.dumps({k: v for k, v in res.items() if k != "columns"}), flush=True)
    if args.out:
        json.dump(res, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
