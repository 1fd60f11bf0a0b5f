#!/usr/bin/env python
"""Same-box A/B of library builds on single-column decodes, decode->sum and decode->global
(500M rows, L2 flushed before every launch, each library in its own process, alternating).

  python scripts/ab_modes.py OUT.json rfor_runs4,rfor_runs8 LIB_A.so LIB_B.so ... [--reps 2]
configs: the names of scripts/tile_sweep.py CONFIGS, or for_b<k>"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "scripts"))


def child(cfgs):
    sys.path.insert(0, ROOT)
    import numpy as np
    import torch
    from tile_sweep import CONFIGS
    from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    out = torch.empty(500_000_000, dtype=torch.int32, device="cuda")
    acc = torch.zeros(1, dtype=torch.int64, device="cuda")
    res = {}
    for cfg in cfgs:
        if cfg.startswith("for_b") and cfg not in CONFIGS:
            b = int(cfg[5:])
            scheme, gen = "for", (lambda n, b=b: __import__("datagen").uniform_bits(b, n, seed=2000 + b))
        else:
            scheme, gen = CONFIGS[cfg]
        x = gen(500_000_000)
        h = tp.encode(x, scheme)
        d = h.to_device()
        xd = torch.from_numpy(x).cuda()
        truth = int(x.astype(np.int64).sum())
        r = {"bytes": h.nbytes()}
        for mode in ("sum", "global"):
            f = (lambda: tp.tp_decode_sum(d.col, acc)) if mode == "sum" else (lambda: tp.tp_decode(d.col, out))
            for _ in range(3):
                acc.zero_()
                f()
            torch.cuda.synchronize()
            r[mode + "_ok"] = (int(acc.item()) == truth) if mode == "sum" else bool(torch.equal(out, xd))
            ts = []
            for _ in range(15):
                flush.zero_()
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                f()
                b.record()
                torch.cuda.synchronize()
                ts.append(a.elapsed_time(b))
            r[mode + "_ms"] = float(np.median(ts))
        del d, xd
        res[cfg] = r
    print("RESULT", json.dumps(res))


def main():
    if sys.argv[1] == "--child":
        child(sys.argv[2].split(","))
        return
    args = sys.argv[1:]
    reps = 2
    if "--reps" in args:
        i = args.index("--reps")
        reps = int(args[i + 1])
        del args[i:i + 2]
    outp, cfgs, libs = args[0], args[1], args[2:]
    peak = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])
    allr = {}
    for rep in range(reps):
        for lib in libs:
            name = os.path.basename(lib)
            env = dict(os.environ, TILEPACK_LIB_OVERRIDE=os.path.abspath(lib), TILEPACK_DEBUG_LAUNCH="1")
            o = subprocess.run([sys.executable, __file__, "--child", cfgs], env=env, capture_output=True, text=True)
            line = [x for x in o.stdout.splitlines() if x.startswith("RESULT")]
            if not line:
                print(name, "FAILED", o.stderr[-800:], flush=True)
                continue
            r = json.loads(line[0][7:])
            launches = [x[9:] for x in o.stderr.splitlines() if x.startswith("TPLAUNCH")]
            launches = [x for i, x in enumerate(launches) if i == 0 or x != launches[i - 1]]  # per (cfg, mode)
            print(name, "launch configs:", launches, flush=True)
            for cfg, v in r.items():
                v["global_hbm_frac"] = (v["bytes"] + 2e9) / (v["global_ms"] / 1e3) / 1e9 / peak
                allr.setdefault(name, {}).setdefault(cfg, []).append(v)
                print(rep, name, cfg, json.dumps(v), flush=True)
    summ = {lib: {cfg: {k: min(x[k] for x in vs) for k in ("sum_ms", "global_ms")} |
                  {"ok": all(x["sum_ok"] and x["global_ok"] for x in vs),
                   "global_hbm_frac": max(x["global_hbm_frac"] for x in vs)}
                  for cfg, vs in d.items()} for lib, d in allr.items()}
    for lib, d in summ.items():
        print(lib, json.dumps(d))
    json.dump({"what": __doc__.split("\n\n")[0], "runs": allr, "best": summ}, open(outp, "w"), indent=1)


if __name__ == "__main__":
    main()
