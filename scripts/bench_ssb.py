#!/usr/bin/env python
"""SSB (BASELINE config 5): the 13 queries with inline tile decompression (Fig. 11).

  python scripts/bench_ssb.py --sf 20 [--reps 10] [--check] [--out profiles/x.json]
  torchrun --nproc-per-node N scripts/bench_ssb.py --sf 160      (tile-range shards + NCCL allreduce)

Per query: lookup-table build ms, fused star-kernel ms (CUDA events, median, L2 flushed before
each rep), allreduce ms (N > 1), compressed bytes of the referenced columns and their HBM floor.
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sf", type=float, default=20)
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--check", action="store_true", help="compare every result with the oracle (rank 0)")
    ap.add_argument("--out", default=None)
    ap.add_argument("--queries", default="all")
    ap.add_argument("--scheme", default="auto", help="auto (GPU-*, P:1206-1217) | none (uncompressed baseline, "
                    "Fig. 11) | for | dfor | rfor for every lineorder column")
    args = ap.parse_args()
    import torch
    import torch.distributed as dist
    import datagen.ssb as gen
    from paper_conf_sigmod_shanbhagyym22_b200.ssb import QUERIES, SSBEngine

    rank, world = int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    # TILEPACK_DIST_BACKEND=gloo: a functional check of the N > 1 path with several ranks on fewer
    # GPUs (ranks share a device; NCCL needs one GPU per rank) -- never a measurement
    backend = os.environ.get("TILEPACK_DIST_BACKEND", "nccl")
    if backend != "nccl":
        local %= max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group(backend, device_id=dev if backend == "nccl" else None)
    t0 = time.time()
    db = gen.generate(args.sf, seed=5000, columns=gen.QUERY_COLUMNS)
    n = len(db["lineorder"]["lo_orderdate"])
    from paper_conf_sigmod_shanbhagyym22_b200.dist import tile_range
    r0, r1 = tile_range(n, rank, world)
    gen_s = time.time() - t0
    from paper_conf_sigmod_shanbhagyym22_b200.ssb import QUERY_COLUMNS
    eng = SSBEngine(db, dev, rows=(r0, r1), schemes={c: args.scheme for c in QUERY_COLUMNS})
    setup_s = time.time() - t0
    peak = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])
    stream = torch.cuda.current_stream(dev)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    oracle = None
    if args.check and rank == 0:
        from oracle import ssb as ossb
        t_o = time.perf_counter()
        oracle = ossb.SSB(db)
        oracle_join_s = time.perf_counter() - t_o  # date join shared by all queries
    qs = QUERIES if args.queries == "all" else args.queries.split(",")
    res = {}
    for qid in qs:
        ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
        a, b = ev(), ev()
        a.record(stream)
        prep = eng.prepare(qid)
        b.record(stream)
        torch.cuda.synchronize()
        build_ms = a.elapsed_time(b)
        cols = sorted({c[0] for c in prep["plan"]["cols"]})
        cbytes = sum(eng.host[c].nbytes() for c in cols)
        sums = torch.zeros(prep["ngroups"], dtype=torch.int64, device=dev)
        counts = torch.zeros_like(sums)
        kt, at = [], []
        for it in range(args.reps + 2):
            sums.zero_()
            counts.zero_()
            flush.sum()
            if world > 1:
                dist.barrier()
            k0, k1, k2 = ev(), ev(), ev()
            torch.cuda._sleep(2_000_000)  # the GPU busy ~1 ms: the host's launch work is not timed
            k0.record(stream)
            eng.execute(prep, sums, counts, stream)
            k1.record(stream)
            if world > 1:
                dist.all_reduce(sums)
                dist.all_reduce(counts)
            k2.record(stream)
            torch.cuda.synchronize()
            if it >= 2:
                kt.append(k0.elapsed_time(k1))
                at.append(k1.elapsed_time(k2))
        kms = statistics.median(kt)
        t = torch.tensor([kms, statistics.median(at), kms + statistics.median(at)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        kmax, ared, e2e = (float(v) for v in t.tolist())
        r = {"kernel_ms": kmax, "allreduce_ms": ared if world > 1 else 0.0, "query_ms": e2e,
             "lookup_build_ms": build_ms, "columns": cols, "compressed_bytes_per_gpu": cbytes,
             "hbm_floor_ms": cbytes / peak / 1e6, "hbm_frac": cbytes / (kmax / 1e3) / 1e9 / peak,
             "groups": prep["ngroups"]}
        if rank == 0:
            rows = eng.result(qid, prep, sums, counts)
            r["result_groups"] = len(rows)
            if oracle is not None:
                t_o = time.perf_counter()
                want = oracle.run(qid)
                r["oracle_s"] = time.perf_counter() - t_o  # numpy SQL over uncompressed columns, host
                r["parity"] = rows == want
            print(qid, json.dumps({k: (round(v, 4) if isinstance(v, float) else v) for k, v in r.items()}), flush=True)
        res[qid] = r
    if rank == 0:
        summary = {"sf": args.sf, "rows": n, "n_gpus": world, "scheme": args.scheme, "gen_s": gen_s, "setup_s": setup_s,
                   "cpu_baseline": None if oracle is None else {
                       "kind": "oracle", "cores": 1, "what": "oracle/ssb.py: numpy SQL over the uncompressed "
                       "columns, per query (oracle_s), plus a shared date join of %.2f s" % oracle_join_s},
                   "footprint": {k: [s, b] for k, (s, b) in eng.footprint().items()},
                   "geomean_query_ms": float(np.exp(np.mean([np.log(r["query_ms"]) for r in res.values()]))),
                   "queries": res}
        print(json.dumps({k: v for k, v in summary.items() if k != "queries"}), flush=True)
        if args.out:
            json.dump(summary, open(args.out, "w"), indent=1)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
