#!/usr/bin/env python
"""Write the SSB oracle's answers for one scale factor to tests/golden/ssb_sf<SF>.json.

Calls ONLY datagen (the seeded generator) and oracle/ (oracle.ssb: the 13 queries as plain
SQL over the uncompressed columns) -- no product code -- so
bench.py and the GPU tests can check the fused star-join kernel at full SSB size without
re-running a minute of numpy SQL on the GPU box.

  python scripts/make_ssb_golden.py --sf 20
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sf", type=float, default=20)
    ap.add_argument("--seed", type=int, default=5000)
    args = ap.parse_args()
    import datagen.ssb as gen
    from oracle import ssb as ossb
    t0 = time.time()
    db = gen.generate(args.sf, seed=args.seed, columns=gen.QUERY_COLUMNS)
    o = ossb.SSB(db)
    res, secs = {}, {}
    for q in ossb.QUERIES:
        t = time.time()
        res[q] = [list(r) for r in o.run(q)]
        secs[q] = round(time.time() - t, 2)
        print(q, len(res[q]), secs[q], flush=True)
    out = {"sf": args.sf, "seed": args.seed, "rows": int(db["lineorder_rows"]),
           "generator": "datagen.ssb.generate (chunked seeded streams)", "oracle": "oracle/ssb.py",
           "oracle_seconds_1core": secs, "total_s": round(time.time() - t0, 1), "results": res}
    sf = ("%g" % args.sf).replace(".", "_")
    path = os.path.join(ROOT, "tests", "golden", f"ssb_sf{sf}.json")
    json.dump(out, open(path, "w"), separators=(",", ":"))
    print("wrote", path, os.path.getsize(path), "bytes")


if __name__ == "__main__":
    main()
