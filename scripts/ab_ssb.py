#!/usr/bin/env python
"""A/B of the SSB star kernel between library builds on one box: each build runs in its own process
(TILEPACK_LIB_OVERRIDE) over the same SF 20 data, every query median of 5 (L2 flushed), results
checked against tests/golden/ssb_sf20.json.  usage: ab_ssb.py LIB [LIB ...] [--queries q,q]"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def child(queries):
    sys.path.insert(0, ROOT)
    import numpy as np
    import torch
    import datagen.ssb as gen
    from paper_conf_sigmod_shanbhagyym22_b200.ssb import QUERIES, SSBEngine
    g = json.load(open(os.path.join(ROOT, "tests", "golden", "ssb_sf20.json")))
    db = gen.generate(20, seed=5000, columns=gen.QUERY_COLUMNS)
    scheme = os.environ.get("TILEPACK_AB_SCHEME")  # "none": the uncompressed columns through the same kernel
    eng = SSBEngine(db, schemes={c: scheme for c in gen.QUERY_COLUMNS} if scheme else None)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    res = {}
    for q in (queries or QUERIES):
        prep = eng.prepare(q)
        sums = torch.zeros(prep["ngroups"], dtype=torch.int64, device="cuda")
        counts = torch.zeros_like(sums)
        ts = []
        for it in range(7):
            sums.zero_(); counts.zero_(); flush.zero_(); flush.sum()
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda._sleep(2_000_000)  # the host's launch work overlaps GPU time: not timed
            a.record()
            eng.execute(prep, sums, counts)
            b.record()
            torch.cuda.synchronize()
            if it >= 2:
                ts.append(a.elapsed_time(b))
        ok = [list(r) for r in eng.result(q, prep, sums, counts)] == g["results"][q]
        res[q] = (round(float(np.median(ts)), 4), ok)
    print("RESULT", json.dumps(res))


if __name__ == "__main__":
    if sys.argv[1] == "--child":
        child(sys.argv[2].split(",") if len(sys.argv) > 2 and sys.argv[2] else None)
        sys.exit(0)
    args = sys.argv[1:]
    qs = ""
    if "--queries" in args:
        i = args.index("--queries")
        qs = args[i + 1]
        args = args[:i] + args[i + 2:]
    for spec in args:  # LIB or LIB:VAR=VAL,VAR=VAL (tuning knobs read from the environment)
        lib, _, kv = spec.partition(":")
        env = dict(os.environ, TILEPACK_LIB_OVERRIDE=os.path.abspath(lib))
        env.update(dict(x.split("=", 1) for x in kv.split(",") if x))
        out = subprocess.run([sys.executable, __file__, "--child", qs], env=env, capture_output=True, text=True)
        line = [x for x in out.stdout.splitlines() if x.startswith("RESULT")]
        if not line:
            print(os.path.basename(spec), "FAILED", out.stderr[-800:], flush=True)
            continue
        r = json.loads(line[0][7:])
        import math
        geo = math.exp(sum(math.log(v[0]) for v in r.values()) / len(r))
        print(os.path.basename(spec), "geomean %.4f" % geo, "parity", all(v[1] for v in r.values()),
              " ".join(f"{q}:{v[0]}" for q, v in r.items()), flush=True)
