#!/usr/bin/env python
"""Run ONE decode of a bench_suite configuration (for ncu: capture the last launch).

  ncu --set full -k regex:k_decode -s 2 -c 1 -o out python scripts/profile_one.py for_b4 sum
  modes: sum | global | enc (tp_gpu_encode of the column)
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))


def main():
    name, mode = sys.argv[1], sys.argv[2]
    rows = int(sys.argv[3]) if len(sys.argv) > 3 else 500_000_000
    import torch
    from bench_suite import configs
    from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp
    cfg = {c[0]: c for c in configs(rows, None, list(range(33)))}[name]
    x = cfg[2]()
    h = tp.encode(x, cfg[1])
    d = h.to_device()
    print(name, "compressed bytes", h.nbytes(), "rows", rows, flush=True)
    acc = torch.zeros(1, dtype=torch.int64, device="cuda")
    out = torch.empty(rows, dtype=torch.int32, device="cuda") if mode == "global" else None
    if mode == "enc":  # the GPU encoder on the same column
        xd = torch.from_numpy(x).cuda()
        for _ in range(3):
            tp.gpu_encode(xd, cfg[1])
        torch.cuda.synchronize()
        return
    for _ in range(3):
        if mode == "sum":
            tp.tp_decode_sum(d.col, acc)
        else:
            tp.tp_decode(d.col, out)
    torch.cuda.synchronize()


if __name__ == "__main__":
    main()
