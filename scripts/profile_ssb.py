#!/usr/bin/env python
"""Run SSB queries once each (for ncu: -k regex:k_star_query).  usage: profile_ssb.py SF q1,q2,..."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    sf = float(sys.argv[1])
    qs = sys.argv[2].split(",")
    import torch
    import datagen.ssb as gen
    from paper_conf_sigmod_shanbhagyym22_b200.ssb import SSBEngine
    eng = SSBEngine(gen.generate(sf, seed=5000))
    for q in qs:
        prep = eng.prepare(q)
        eng.execute(prep)
        torch.cuda.synchronize()
        print(q, "done", flush=True)


if __name__ == "__main__":
    main()
