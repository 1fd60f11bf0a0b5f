#!/usr/bin/env python
"""NEXT-1 ablation (Fig. 7a): tile-based decode-to-global (tp_decode) against the
cascading decompression model (tp_decode_cascaded: one kernel per layer through global memory)
on the paper's varying-bitwidth datasets -- 250M values uniform in [0, 2^i), i = 2, 4, .., 30 --
for GPU-FOR (FOR+BitPack, 2 passes), GPU-DFOR (Delta+FOR+BitPack, 3) and GPU-RFOR
(RLE+FOR+BitPack, 8).  The paper reports 2.6x / 4x / 8x on a V100.

  python scripts/bench_cascaded.py [--rows 250000000] [--bits 2,4,...] [--out profiles/x.json]
"""
import argparse
import json
import math
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import datagen  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rows", type=int, default=250_000_000)
    ap.add_argument("--bits", default=",".join(str(i) for i in range(2, 31, 2)))
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    import torch
    from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp
    dev = torch.device("cuda", 0)
    stream = torch.cuda.current_stream(dev)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    out = torch.empty(args.rows, dtype=torch.int32, device=dev)

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

    res = {"rows": args.rows, "points": {}, "ratio_geomean": {}}
    for scheme in ("for", "dfor", "rfor"):
        ratios = []
        for b in [int(v) for v in args.bits.split(",")]:
            x = datagen.uniform_bits(b, args.rows, seed=7000 + b)
            d = tp.encode(x, scheme).to_device(dev)
            work = torch.empty(max(1, tp.tp_cascaded_workspace_words(d.col)), dtype=torch.int32, device=dev)
            xd = torch.from_numpy(x).to(dev)
            t_tile = timed(lambda: tp.tp_decode(d.col, out, stream))
            ok_tile = bool(torch.equal(out, xd))
            t_casc = timed(lambda: tp.tp_decode_cascaded(d.col, out, work, stream))
            ok_casc = bool(torch.equal(out, xd))
            r = {"tile_ms": t_tile, "cascaded_ms": t_casc, "speedup": t_casc / t_tile,
                 "bits_per_int": 8 * d.nbytes() / args.rows, "parity": ok_tile and ok_casc}
            res["points"][f"{scheme}_b{b}"] = r
            ratios.append(t_casc / t_tile)
            print(scheme, b, json.dumps({k: round(v, 4) if isinstance(v, float) else v for k, v in r.items()}),
                  flush=True)
            del d, work, xd, x
            torch.cuda.empty_cache()
        res["ratio_geomean"][scheme] = math.exp(sum(math.log(v) for v in ratios) / len(ratios))
    print(json.dumps(res["ratio_geomean"]))
    if args.out:
        json.dump(res, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
