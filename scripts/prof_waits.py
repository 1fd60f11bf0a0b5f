#!/usr/bin/env python
"""Cycle split of the query pipeline (build with TP_NVCC_FLAGS=-DTP_PROFILE_WAITS):
consumer data waits vs per-column work vs producer slot waits, per SSB query.
usage: prof_waits.py SF q1,q2,..."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    sf = float(sys.argv[1])
    qs = sys.argv[2].split(",")
    import torch
    import datagen.ssb as gen
    from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp
    from paper_conf_sigmod_shanbhagyym22_b200.ssb import SSBEngine
    eng = SSBEngine(gen.generate(sf, seed=5000, columns=gen.QUERY_COLUMNS))  # noqa
    for q in qs:
        prep = eng.prepare(q)
        eng.execute(prep)
        torch.cuda.synchronize()
        tp.tp_debug_counters()
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record()
        eng.execute(prep)
        ev1.record()
        torch.cuda.synchronize()
        c = tp.tp_debug_counters().astype(float)
        tot = c[0] + c[1:8].sum()
        print(q, f"ms={ev0.elapsed_time(ev1):.3f}", f"consumer: wait={c[0] / tot:.1%}",
              "cols=" + " ".join(f"{x / tot:.1%}" for x in c[1:8] if x),
              f"| producer wait/consumer total={c[8] / tot:.2f}", flush=True)


if __name__ == "__main__":
    main()
