#!/usr/bin/env python
"""GPU encoder measurements (the paper's encode cost).

For every column (BASELINE configs 2-4 at --rows): the tile-parallel GPU encoder
(tp_gpu_encode_launch, one kernel) and the GPU-* size pass (tp_gpu_encode_sizes) timed with
CUDA events (median of --reps after an L2 flush), the host encoder (tp_encode, all host
threads) timed by wall clock, and a full-size parity check (GPU bytes == host-encoder bytes,
GPU-encoded column decodes to the input).  Roofline: algorithmic bytes = 4 B/row read + the
compressed bytes written.

  python scripts/bench_encode.py [--rows 500000000] [--out profiles/r01_encode.json]
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
import oracle  # noqa: E402  (cpu_baseline: the oracle's encoder timed beside the GPU, bounded sample)

ORACLE_SAMPLE = 20_000_000  # rows of each column the oracle encodes (1 thread, ~1-3 s)


def configs(rows):
    return [("for_b4", "for", lambda: datagen.uniform_bits(4, rows)),
            ("for_b16", "for", lambda: datagen.uniform_bits(16, rows)),
            ("for_b32", "for", lambda: datagen.uniform_bits(32, rows)),
            ("dfor_d1_2^28", "dfor", lambda: datagen.d1_sorted(rows, 2**28)),
            ("dfor_near_sorted", "dfor", lambda: datagen.near_sorted(rows)),
            ("rfor_runs4", "rfor", lambda: datagen.runs(rows, 4)),
            ("rfor_runs64", "rfor", lambda: datagen.runs(rows, 64))]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rows", type=int, default=500_000_000)
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--only", default=None)
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    import torch
    from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp
    peak = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])
    dev = torch.device("cuda", 0)
    stream = torch.cuda.current_stream(dev)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    n = args.rows
    work = torch.empty((tp.tp_gpu_encode_workspace_bytes(n) + 7) // 8, dtype=torch.int64, device=dev)
    res = {"rows": n, "peak_hbm_gbs": peak, "host_threads": os.cpu_count(), "configs": {}}

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

    for name, scheme, gen in configs(n):
        if args.only and not name.startswith(args.only):
            continue
        x = gen()
        t0 = time.perf_counter()
        h = tp.encode(x, scheme)
        host_s = time.perf_counter() - t0
        xd = torch.from_numpy(x).to(dev)
        sc = tp.SCHEMES[scheme]
        nb, w0, w1 = tp.tp_gpu_encode_bound(sc, n)
        s0 = torch.empty(nb + 5, dtype=torch.int32, device=dev)
        d0 = torch.empty(w0 + 4, dtype=torch.int32, device=dev)
        s1 = torch.empty(nb + 5, dtype=torch.int32, device=dev) if sc == tp.TP_RFOR else None
        d1 = torch.empty(w1 + 4, dtype=torch.int32, device=dev) if sc == tp.TP_RFOR else None

        def enc():
            tp.tp_gpu_encode_launch(sc, xd, n, s0, d0, w0, s1, d1, w1, work, stream)
        ms = timed(enc)
        col = tp.tp_gpu_encode_result(sc, n, s0, d0, s1, d1, work, stream)
        cb = tp.tp_compressed_bytes(col)
        # parity: GPU bytes == host-encoder bytes (the host encoder is pinned to the oracle by
        # tests/test_host_encoder.py); decode of the GPU bytes == the input
        ok = (col.words0 == h.col.words0 and col.words1 == h.col.words1
              and np.array_equal(d0[:col.words0].cpu().numpy().view(np.uint32), h.data0[:col.words0])
              and np.array_equal(s0[:nb + 1].cpu().numpy().view(np.uint32), h.starts0[:nb + 1]))
        if sc == tp.TP_RFOR:
            ok = ok and np.array_equal(d1[:col.words1].cpu().numpy().view(np.uint32), h.data1[:col.words1])
        out = torch.empty(n, dtype=torch.int32, device=dev)
        tp.tp_decode(col, out, stream)
        ok = ok and bool(torch.equal(out, xd))
        del out

        def sizes():
            tp.tp_gpu_encode_sizes(xd, n, work, stream)
        ms_sizes = timed(sizes)
        alg = 4 * n + cb
        r = {"scheme": scheme, "compressed_bytes": cb, "bits_per_int": 8 * cb / n,
             "gpu_encode_ms": ms, "gpu_encode_input_gbs": 4 * n / ms / 1e6,
             "gpu_encode_hbm_gbs": alg / ms / 1e6, "gpu_encode_hbm_frac": alg / ms / 1e6 / peak,
             "gpu_sizes_all3_ms": ms_sizes, "gpu_sizes_hbm_frac": 4 * n / ms_sizes / 1e6 / peak,
             "host_encode_s": host_s, "gpu_vs_host": host_s * 1e3 / ms, "parity": ok}
        import time as _t
        t1 = _t.perf_counter()
        oracle.encode(scheme, x[:ORACLE_SAMPLE])
        osec = _t.perf_counter() - t1
        r["oracle_encode_rows_per_s"] = min(n, ORACLE_SAMPLE) / osec
        r["oracle_sample_rows"] = min(n, ORACLE_SAMPLE)
        r["gpu_vs_oracle"] = (n / (ms / 1e3)) / r["oracle_encode_rows_per_s"]
        res["configs"][name] = r
        print(name, json.dumps({k: (round(v, 4) if isinstance(v, float) else v) for k, v in r.items()}), flush=True)
        del xd, s0, d0, s1, d1, h, x
        torch.cuda.empty_cache()
    res["paper_cpu_encode_s_250M_6vcpu"] = {"for": 1.2, "dfor": 1.3, "rfor": 2.2}  # P:1228-1232, context
    if args.out:
        json.dump(res, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
