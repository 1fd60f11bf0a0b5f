#!/usr/bin/env python
"""Fold the per-configuration ncu CSVs of scripts/issue_profile.sh into profiles/r02_issue.json:
warp instructions per launch, instructions per decoded value (32 x warp insts / rows), pipe split,
issue-active %, achieved occupancy, shared-memory bank conflicts and the top stall reasons."""
import csv
import glob
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ROWS = 500_000_000


def read(path):
    rows = [r for r in csv.reader(open(path)) if r]
    hdr_i = next(i for i, r in enumerate(rows) if "ID" in r and "Kernel Name" in r)
    hdr, vals = rows[hdr_i], rows[-1]
    out = {}
    for k, v in zip(hdr, vals):
        try:
            out[k] = float(v.replace(",", ""))
        except ValueError:
            out[k] = v
    return out


def main():
    src = sys.argv[1]
    res = {}
    for f in sorted(glob.glob(os.path.join(src, "*.csv"))):
        name = os.path.basename(f)[:-4]
        cfg, mode = name.rsplit("_", 1)
        try:
            m = read(f)
        except (StopIteration, IndexError):
            continue
        wi = m.get("smsp__inst_executed.sum")
        if not isinstance(wi, float):
            continue
        stalls = {k.split("smsp__average_warps_issue_stalled_")[1].split("_per_issue_active")[0]: v
                  for k, v in m.items() if k.startswith("smsp__average_warps_issue_stalled_")
                  and k.endswith("_per_issue_active.ratio") and isinstance(v, float)}
        top = dict(sorted(stalls.items(), key=lambda kv: -kv[1])[:6])
        r = res.setdefault(cfg, {})
        r[f"{mode}_warp_insts"] = wi
        r[f"{mode}_insts_per_value"] = 32 * wi / ROWS
        r[f"{mode}_ncu_ms"] = m.get("gpu__time_duration.sum", 0) / 1e6 if m.get("gpu__time_duration.sum") else None
        for p in ("alu", "fma", "lsu", "uniform"):
            v = m.get(f"smsp__inst_executed_pipe_{p}.sum")
            if isinstance(v, float):
                r[f"{mode}_pipe_{p}_frac"] = v / wi
        r[f"{mode}_issue_active_pct"] = m.get("smsp__issue_active.avg.pct_of_peak_sustained_active")
        r[f"{mode}_warps_active_pct"] = m.get("sm__warps_active.avg.pct_of_peak_sustained_active")
        r[f"{mode}_dram_bytes"] = (m.get("dram__bytes_read.sum", 0) or 0) + (m.get("dram__bytes_write.sum", 0) or 0)
        ld = m.get("l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum")
        if isinstance(ld, float) and ld:
            r[f"{mode}_smem_ld_conflict_frac"] = m.get("l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", 0) / ld
        r[f"{mode}_top_stalls_per_issue"] = top
    alias = {"dfor_d1_228": "dfor_d1"}
    for a, b in alias.items():
        if a in res:
            res[b] = res[a]
    path = os.path.join(ROOT, "profiles", "r02_issue.json")
    prev = json.load(open(path)).get("configs", {}) if os.path.exists(path) else {}
    prev.update(res)  # a run over some configurations refreshes those and keeps the others
    out = {"what": "ncu (--clock-control none) per decode configuration, 500M rows, one launch each: "
                   "scripts/issue_profile.sh", "configs": prev}
    json.dump(out, open(path, "w"), indent=1)
    for k, v in res.items():
        print(k, {kk: (round(vv, 3) if isinstance(vv, float) else vv) for kk, vv in v.items() if "stalls" not in kk})


if __name__ == "__main__":
    main()
