#!/usr/bin/env python
"""Summarise an ncu report (--set full) into profiles/ncu_summary.json and print key metrics.

usage: python scripts/ncu_summarize.py <report.ncu-rep> <workload-key> [--algorithmic-bytes B]
"""
import csv
import io
import json
import os
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__inst_executed.sum", "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__cycles_elapsed.avg.per_second", "launch__occupancy_limit_shared_mem",
        "launch__shared_mem_per_block_dynamic", "lts__t_bytes.sum"]
SCALE = {"Ghz": 1e9, "Mhz": 1e6, "hz": 1, "Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1, "us": 1e-6, "ms": 1e-3, "ns": 1e-9, "s": 1}


def main():
    rep, key = sys.argv[1], sys.argv[2]
    alg = None
    if "--algorithmic-bytes" in sys.argv:
        alg = int(sys.argv[sys.argv.index("--algorithmic-bytes") + 1])
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    recs = []
    for r in rows[2:]:
        d = {}
        for i, k in enumerate(hdr):
            if k in KEYS or k == "Kernel Name":
                d[k] = r[i]
                if k != "Kernel Name" and units[i]:
                    d[k + ".unit"] = units[i]
        recs.append(d)
    r = recs[-1]

    def val(k):
        v = float(r[k].replace(",", ""))
        return v * SCALE.get(r.get(k + ".unit", ""), 1)
    summ = {"kernel": r["Kernel Name"], "report": os.path.basename(rep),
            "duration_s": val("gpu__time_duration.sum"),
            "dram_bytes_read": int(val("dram__bytes_read.sum")), "dram_bytes_write": int(val("dram__bytes_write.sum")),
            "inst_executed": int(val("smsp__inst_executed.sum")),
            "issue_active_pct": val("smsp__issue_active.avg.pct_of_peak_sustained_active"),
            "warps_active_pct": val("sm__warps_active.avg.pct_of_peak_sustained_active"),
            "smem_bank_conflicts": int(val("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum")),
            "registers": int(val("launch__registers_per_thread")), "sm_clock_hz": val("sm__cycles_elapsed.avg.per_second"),
            "dram_pct_peak": val("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed") if "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed" in r else None}
    if alg:
        summ["algorithmic_bytes"] = alg
        summ["traffic_over_algorithmic"] = (summ["dram_bytes_read"] + summ["dram_bytes_write"]) / alg
    path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "ncu_summary.json")
    try:
        allp = json.load(open(path))
    except Exception:
        allp = {"_about": "ncu --set full --clock-control none captures (one launch each); per-launch DRAM bytes",
                "kernels": {}}
    allp["kernels"][key] = summ
    json.dump(allp, open(path, "w"), indent=1, sort_keys=True)
    print(json.dumps(summ, indent=1))


if __name__ == "__main__":
    main()
