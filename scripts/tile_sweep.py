#!/usr/bin/env python
"""NEXT-4 (Fig. 5): the tiles-per-thread-block study on B200.  The paper sweeps D, the
number of 128-value blocks a thread block decodes (D = 4: 1.55 ms at 500M U[0,2^16) on V100,
P:954-956); here the corresponding knobs of the persistent TMA pipeline are swept for
decode->sum at b = 4 and b = 16 (500M rows):
  rounds  -- tiles per ring item = 8 x rounds (the single-column item; default: ~16 KB of words)
  ring_kb -- the ring's bytes per CTA (default 40)
  minb    -- CTAs per SM asked of the compiler (launch bounds; default 4)
  python scripts/tile_sweep.py --build          (CPU: one library per point into build_ab/)
  python scripts/tile_sweep.py --run OUT.json   (GPU: each library in its own process)"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
POINTS = {"default": ""}
for r in (1, 2, 4, 8):
    POINTS[f"rounds{r}"] = f"-DTP_FIXED_ROUNDS={r}"
for kb in (16, 24, 64):
    POINTS[f"ring{kb}kb"] = f"-DTP_RING_KB={kb}"
for mb in (2, 3, 5):
    POINTS[f"minb{mb}"] = f"-DTP_SUM_MINB={mb}"
# second sweep: the item-size target and the ring of the instruction-bound single-column decodes
POINTS2 = {"default": ""}
for tw in (6144, 8192, 12288):
    POINTS2[f"tw{tw}"] = f"-DTP_TARGET_WORDS={tw}u"
for kb in (40, 64):
    POINTS2[f"qring{kb}kb"] = f"-DTP_QUERY_RING_KB={kb}"
POINTS2["tw8192_qring40kb"] = "-DTP_TARGET_WORDS=8192u -DTP_QUERY_RING_KB=40"
CONFIGS = {"for_b4": ("for", lambda n: __import__("datagen").uniform_bits(4, n, seed=2004)),
           "for_b16": ("for", lambda n: __import__("datagen").uniform_bits(16, n, seed=2016)),
           "dfor_d1": ("dfor", lambda n: __import__("datagen").d1_sorted(n, 2**28)),
           "rfor_runs8": ("rfor", lambda n: __import__("datagen").runs(n, 8)),
           "rfor_runs4": ("rfor", lambda n: __import__("datagen").runs(n, 4)),
           "dfor_near": ("dfor", lambda n: __import__("datagen").near_sorted(n)),
           "dfor_sorted": ("dfor", lambda n: __import__("datagen").sorted_uniform(n)),
           "dfor_consec": ("dfor", lambda n: __import__("datagen").consecutive(n))}


def build(points=POINTS):
    for name, flags in points.items():
        subprocess.check_call([sys.executable, os.path.join(ROOT, "scripts", "build_variant.py"), f"sw_{name}", flags],
                              stdout=subprocess.DEVNULL)
        print("built", name, flags, flush=True)


def child(cfg):
    sys.path.insert(0, ROOT)
    import numpy as np
    import torch
    from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp
    if cfg.isdigit() or (cfg.startswith("for_b") and cfg not in CONFIGS):
        b = int(cfg[5:] if cfg.startswith("for_b") else cfg)
        scheme, gen = "for", (lambda n: __import__("datagen").uniform_bits(b, n, seed=2000 + b))
    else:
        scheme, gen = CONFIGS[cfg]
    x = gen(500_000_000)
    h = tp.encode(x, scheme)
    d = h.to_device()
    truth = int(x.astype(np.int64).sum())
    acc = torch.zeros(1, dtype=torch.int64, device="cuda")
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    for _ in range(3):
        acc.zero_()
        tp.tp_decode_sum(d.col, acc)
    torch.cuda.synchronize()
    ok = int(acc.item()) == truth
    ts = []
    for _ in range(15):
        flush.zero_()
        flush.sum()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        tp.tp_decode_sum(d.col, acc)
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    sms, occ = tp.tp_device_info()
    print("RESULT", json.dumps({"ms": float(np.median(ts)), "bytes": h.nbytes(), "parity": ok, "ctas_per_sm": occ}))


def run(out, points=POINTS, cfgs=("4", "16"), prefix="sw_"):
    peak = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])
    res = {"what": __doc__.split("\n\n")[0], "peak_hbm_gbs": peak, "points": {}}
    for name, flags in points.items():
        lib = os.path.join(ROOT, "build_ab", f"libtilepack_{prefix}{name}.so")
        for bits in cfgs:
            env = dict(os.environ, TILEPACK_LIB_OVERRIDE=lib)
            o = subprocess.run([sys.executable, __file__, "--child", str(bits)], env=env, capture_output=True, text=True)
            line = [x for x in o.stdout.splitlines() if x.startswith("RESULT")]
            if not line:
                print(name, bits, "FAILED", o.stderr[-500:], flush=True)
                continue
            r = json.loads(line[0][7:])
            r["flags"] = flags
            r["decoded_gbs"] = 2e9 / (r["ms"] / 1e3) / 1e9
            r["hbm_frac"] = r["bytes"] / (r["ms"] / 1e3) / 1e9 / peak
            res["points"][f"{name}_{'b' + bits if bits.isdigit() else bits}"] = r
            print(name, bits, json.dumps(r), flush=True)
    json.dump(res, open(out, "w"), indent=1)


if __name__ == "__main__":
    if sys.argv[1] == "--build":
        build()
    elif sys.argv[1] == "--build2":
        build({f"sw2_{k}": v for k, v in POINTS2.items()})
    elif sys.argv[1] == "--child":
        child(sys.argv[2])
    elif sys.argv[1] == "--ab":  # --ab OUT.json cfg1,cfg2 LIB...
        libs = sys.argv[4:]
        pts = {os.path.basename(l)[len("libtilepack_"):-3]: "" for l in libs}
        run(sys.argv[2], pts, tuple(sys.argv[3].split(",")), "")
    elif sys.argv[1] == "--run2":
        run(sys.argv[2], POINTS2, ("for_b4", "for_b16", "dfor_d1", "rfor_runs8"), "sw2_")
    else:
        run(sys.argv[2])
