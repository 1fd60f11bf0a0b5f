#!/usr/bin/env python
"""Regenerate profiles/README.md from the committed profiles/*.json (after copying a
scripts/refresh_profiles.sh run from gpurun_out/r/).  usage: python scripts/profiles_readme.py"""
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
P = os.path.join(ROOT, "profiles")


def load(name):
    path = os.path.join(P, name)
    if name.endswith(".json") and os.path.exists(path):
        txt = open(path).read().strip()
        return json.loads(txt.splitlines()[-1]) if txt.startswith('{"metric"') else json.loads(txt)
    return None


def main():
    b = load("r01_bench.json")
    r = b["roofline"]
    ncu = load("ncu_summary.json")["kernels"]["for_b16_sum"]
    s = f"""# profiles/ — measured evidence (round 1)

All numbers on one B200 (148 SMs, sm_100a, SM clock {b['clocks']['sm_mhz']:.0f} MHz under load = max, no throttle
reasons recorded), CUDA 12.9, driver 580.  Roofline denominator: `MEASURED_PEAKS.json` `hbm_gbs`
(copy, read+write; "of measured").  Every file below comes from ONE run of
`scripts/refresh_profiles.sh` (all measurements + ncu captures on one box, at the final commit of
round 1); this README is generated from them by `scripts/profiles_readme.py`.

| file | what |
|---|---|
| `r01_bench.json` | `python bench.py` (defaults: 500 steps, 5 warm-up) — the JSON line the driver reads |
| `r01_launches_bench.csv` | `ncu --metrics gpu__time_duration.sum --clock-control none -c 60 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 2` — per-launch list |
| `ncu_summary.json`, `r01_ncu_k_decode_sum_details.txt` | `ncu --set full --clock-control none --import-source on -k regex:k_decode_sum -s 3 -c 1 python bench.py --steps 3 ...` — DRAM bytes per launch (the bench's `roofline.traffic`), occupancy, issue, stall details |
| `r01_suite.json` | `scripts/bench_suite.py` — every BASELINE config 2-4 column (FOR b = 0..32, DFOR C3, RFOR C4) at 500M rows, decode→sum and decode→global, full-size parity flags |
| `r01_ssb_sf20.json`, `r01_ssb_sf20_none.json`, `r01_ssb_sf160.json` | `scripts/bench_ssb.py --sf 20 --check` (GPU-*, every result == the oracle), `--scheme none` (uncompressed through the same kernels), `--sf 160` (config 5's SF×8) |
| `r01_encode.json` | `scripts/bench_encode.py` — the tile-parallel GPU encoder at 500M rows (GPU bytes == host-encoder bytes, decode == input), the GPU-* analysis pass, the host encoder and the oracle (20M-row sample) beside it |
| `r01_random_access.json` | `scripts/bench_random_access.py` — P:1241-1262 selectivity sweep at 250M rows, compressed vs None, parity and the oracle's time at every point |
| `r01_cascaded_ablation.json` | `scripts/bench_cascaded.py` — tile-based vs cascading decode (NEXT-1, Fig. 7a) |
| `r01_waterfall_sf20.json` | `scripts/bench_waterfall.py` — SSB compression waterfall + per-column decode (NEXT-2, Fig. 9/10) |
| `r01_nomb_ablation.json` | `scripts/bench_nomb.py` — GPU-FOR with vs without miniblocks (NEXT-4, P:975-987) |

## Headline (config 2, b = 16, 500M rows, decode fused into an int64 sum)

* step {b['ms_per_step']:.4f} ms; `k_decode_sum` average {r['kernel_avg_ms'] * 1000:.1f} µs (CUDA events over 500 launches)
* achieved {r['achieved']:,.0f} GB/s on compressed bytes = **{100 * r['frac']:.1f} % of measured HBM**; {b['value'] / 1000:.1f} TB/s decoded;
  {b['vs_baseline']:.1f}× the paper's V100 number for the same workload (1.55 ms, P:954-956).  Across box
  allocations the same build measures 160.5-167 µs (96-99.6 %).
* ncu (cold, serialised, one launch): {ncu['duration_s'] * 1e6:.1f} µs, DRAM read {ncu['dram_bytes_read'] / 1e9:.4f} GB + write
  {ncu['dram_bytes_write'] / 1e6:.1f} MB = {ncu['traffic_over_algorithmic']:.3f} × the algorithmic 1.0469 GB (no re-reads),
  {ncu['inst_executed'] / 1e6:.0f} M warp instructions, issue active {ncu['issue_active_pct']:.0f} %, {ncu['registers']} registers
* launch list share: inside a bench step the only other launch is torch's 1-element zero fill (~2 µs);
  `k_plain_sum` rows are the uncompressed "None" context measurement after the timed region.
* e2e (compressed arrays copied from pinned host memory every step): {b['e2e']['value']:.0f} GB/s decoded (PCIe-bound)
* cpu_baseline (the oracle, 1 thread): {b['cpu_baseline']['value']:.2f} GB/s decoded
"""
    d = load("r01_suite.json")
    s += """
## Sweep and other schemes (r01_suite.json, 500M rows, single launches after an L2 flush)

| column | bits/int | decode→sum ms | HBM frac | decoded TB/s | decode→global ms | HBM frac (read + 2 GB write) |
|---|---|---|---|---|---|---|
"""
    for k, v in d["configs"].items():
        if k.startswith("for_b") and int(k[5:]) not in (0, 1, 4, 8, 12, 16, 24, 32):
            continue
        s += (f"| {k} | {v['bits_per_int']:.2f} | {v['sum_ms']:.3f} | {v['sum_hbm_frac']:.2f} | "
              f"{v['sum_decoded_gbs'] / 1000:.1f} | {v['global_ms']:.3f} | {v['global_hbm_frac']:.2f} |\n")
    s += """
Decode-only below b ≈ 12 and for DFOR / RFOR is instruction-bound (the compressed bytes are too few
for HBM to bind: SURVEY App. C.4); decode→global is the HBM-bound mode the ≥70 % target applies to.
"""
    e = load("r01_encode.json")
    s += """
## GPU encoder (r01_encode.json, 500M rows; NEXT-3)

| column | GPU encode ms | HBM frac (4 B/row read + compressed written) | GPU-* analysis (3 schemes) ms | host encoder s (all cores) | oracle rows/s (1 thread) |
|---|---|---|---|---|---|
"""
    for k, v in e["configs"].items():
        s += (f"| {k} | {v['gpu_encode_ms']:.3f} | {v['gpu_encode_hbm_frac']:.2f} | {v['gpu_sizes_all3_ms']:.2f} | "
              f"{v['host_encode_s']:.3f} | {v.get('oracle_encode_rows_per_s', 0) / 1e6:.0f} M |\n")
    s += """
Every GPU-encoded column is byte-identical to the host encoder's (itself pinned to the oracle) and
decodes to its input.  FOR / DFOR are bounded by the chunk look-back (ncu: half the stall samples
on the barrier after it); RFOR by the run marking + two streams at 2 CTAs/SM.  Context: the paper
encodes 250M values in 1.2 / 1.3 / 2.2 s on 6 vCPUs (P:1228-1232).
"""
    q, n, q160 = load("r01_ssb_sf20.json"), load("r01_ssb_sf20_none.json"), load("r01_ssb_sf160.json")
    s += f"""
## SSB (r01_ssb_sf20.json, r01_ssb_sf20_none.json, r01_ssb_sf160.json)

All 13 SF20 queries equal the oracle (exact int64).  GPU-* picks RFOR for lo_orderdate and
lo_custkey and FOR elsewhere (P:1916-1918, 2009-2011).  Geomean kernel time at SF20: GPU-*
{q['geomean_query_ms']:.3f} ms, None {n['geomean_query_ms']:.3f} ms (paper V100: None 1.35× faster than GPU-*; here
{q['geomean_query_ms'] / n['geomean_query_ms']:.2f}×); SF160: {q160['geomean_query_ms']:.2f} ms.

| query | SF20 GPU-* ms | SF20 None ms | SF20 HBM floor ms | SF160 GPU-* ms |
|---|---|---|---|---|
"""
    for k, v in q["queries"].items():
        s += (f"| {k} | {v['kernel_ms']:.3f} | {n['queries'][k]['kernel_ms']:.3f} | {v['hbm_floor_ms']:.3f} | "
              f"{q160['queries'][k]['kernel_ms']:.3f} |\n")
    s += """
The star kernel is instruction/latency-bound (RFOR expansion of the date / customer keys, probe
round trips, 2-3 CTAs/SM by registers and shared memory), not HBM-bound.
"""
    ra = load("r01_random_access.json")
    s += """
## Random access (r01_random_access.json, 250M rows, P:1241-1262)

| σ | FOR b=16 ms | None ms | DFOR sorted ms | RFOR runs8 ms |
|---|---|---|---|---|
"""
    pts = {}
    for p_ in ra["points"]:
        pts.setdefault(p_["sigma"], {})[p_["column"]] = p_["ms"]
    for sg, v in pts.items():
        s += f"| {sg:.3g} | {v['for_b16']:.3f} | {v['none_b16']:.3f} | {v['dfor_sorted']:.3f} | {v['rfor_runs8']:.3f} |\n"
    s += """
At σ ≥ 1/32 every FOR miniblock is read and FOR beats None (paper V100 2.1 vs 2.5 ms); below
σ ≈ 1/512 most tiles are skipped; in between None reads fewer bytes (one 128-byte line per
selected miniblock vs FOR's block_starts → header → miniblock chain).
"""
    c = load("r01_cascaded_ablation.json")
    w = load("r01_waterfall_sf20.json")
    s += f"""
## Ablations (r01_cascaded_ablation.json, r01_waterfall_sf20.json)

Tile-based vs cascading decode (250M rows, decode→global, geomean over the sweep): FOR
{c['ratio_geomean']['for']:.1f}×, DFOR {c['ratio_geomean']['dfor']:.1f}×, RFOR {c['ratio_geomean']['rfor']:.1f}× (paper V100: 2.6× / 4× / 8×).
SSB SF20 waterfall: GPU-* footprint {w['footprint_ratio_none_over_gpu*']:.2f}× below None over all lineorder columns
(paper 2.8×); tile decode vs cascading {w['decode_speedup_geomean_vs_cascaded']:.1f}× geomean per column.
"""
    nm = load("r01_nomb_ablation.json")
    if nm:
        s += """
## Miniblock ablation (r01_nomb_ablation.json, 500M rows, P:975-987)

| column | FOR bits/int | no-miniblock bits/int | FOR decode→sum ms | no-miniblock decode→sum ms | FOR →global ms | no-miniblock →global ms |
|---|---|---|---|---|---|---|
"""
        for k, v in nm["columns"].items():
            f, g = v["for"], v["fornm"]
            s += (f"| {k} | {f['bits_per_int']:.2f} | {g['bits_per_int']:.2f} | {f['sum_ms']:.3f} | {g['sum_ms']:.3f} | "
                  f"{f['global_ms']:.3f} | {g['global_ms']:.3f} |\n")
        s += """
On B200 both layouts decode b = 16 at the HBM roof (paper V100: 2.0 vs 2.1 ms, the no-miniblock
layout 5 % faster); miniblocks cost nothing there and keep skewed columns 15 % smaller.
"""
    open(os.path.join(P, "README.md"), "w").write(s)
    print("wrote profiles/README.md")


if __name__ == "__main__":
    main()
