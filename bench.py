#!/usr/bin/env python
"""bench.py -- BASELINE.json config 2 (GPU-FOR decode-only on a 500M-entry int32 column)
through the tilepack C ABI on B200, plus the oracle timed on the host as cpu_baseline.

Step = one pass of the decode hot path over the whole column: tile addressing, TMA
staging, header + miniblock offsets, bit unpack, consume in registers (fused int64 sum)
-- SURVEY.md 8(a) rows a1-a4, a7 -- plus, for N > 1, the NCCL allreduce of the
partial aggregate (row a9).  Default workload: U[0, 2^16), the paper's E1 column
(P:720-724, 500 million values), i.e. the b = 16 point of the bitwidth sweep;
--bits picks another point, --sweep adds the whole 0..32 sweep as an extra object.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--bits B] [--sweep] [--impl reference]

Multi-GPU: one process per GPU (torchrun), each rank owns its own 500M column (weak
scaling: tile-range partitions of a dataset N x larger), partial sums combined with
one NCCL allreduce per step.  Timing: CUDA events on the launch stream, barrier +
synchronize on both sides, max over ranks.  L2: the compressed column (>= 1 GB at
b=16) is 8x the 126 MB L2, so consecutive steps never hit L2 (no flush needed).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

N_ROWS = 500_000_000
PAPER_DECODED_GBS = 2e9 / 1.55e-3 / 1e9  # V100, D=16, 500M U(0,2^16): 1.55 ms -> 1290 GB/s


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=500)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--bits", type=int, default=16)
    ap.add_argument("--rows", type=int, default=N_ROWS)
    ap.add_argument("--sweep", action="store_true", help="also time every bitwidth 0..32 (extra object)")
    ap.add_argument("--impl", default="tilepack", choices=["tilepack", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=10)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    return ap.parse_args()


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


# ------------------------------------------------------------------ clocks (NVML, during the timed region)
class ClockSampler:
    def __init__(self, index: int, period: float = 0.005):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self.period, self._stop = period, threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    _NAMES = {0x8: "hw_slowdown", 0x40: "hw_thermal_slowdown", 0x20: "sw_thermal_slowdown",
              0x4: "sw_power_cap", 0x80: "hw_power_brake_slowdown", 0x2: "applications_clocks_setting",
              0x100: "display_clock_setting", 0x1: "gpu_idle", 0x10: "sync_boost"}

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self._NAMES.items():
                    if r & bit and name != "gpu_idle":
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.nv:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        if self.nv:
            self._stop.set()
            self.t.join()

    def summary(self):
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": len(self.samples),
                "source": "NVML (same counters as nvidia-smi), sampled every 5 ms during the timed steps"}


def measured_peak():
    try:
        mp = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
        return float(mp["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs: copy read+write)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


def ncu_traffic(workload: str):
    """dram bytes per launch of the dominant kernel from the committed ncu --set full summary."""
    try:
        prof = json.load(open(os.path.join(ROOT, "profiles", "ncu_summary.json")))
        t = prof["kernels"][workload]
        return int(t["dram_bytes_read"]) + int(t["dram_bytes_write"])
    except Exception:
        return None


# ------------------------------------------------------------------ workload
def make_column(bits: int, rows: int, rank: int):
    import datagen
    seed = 2000 + bits + 1000 * rank
    return datagen.uniform_bits(bits, rows, seed=seed)


def cpu_baseline(h, rows: int, budget_rows: int = N_ROWS):
    """The oracle (oracle/, single-threaded scalar C, Algorithm 1 per entry) decoding and
    summing a bounded sample: the first `budget_rows` rows of the same encoded column."""
    import oracle
    sample = min(rows, budget_rows)
    e = oracle.Encoded(scheme="for", header=h.header(), starts=h.starts0[: h.col.num_blocks + 1],
                       data=h.data0[: h.col.words0])
    t = time.perf_counter()
    y = oracle.for_decode_range(e, 0, sample, h.data0)
    s = oracle.column_sum(y)
    dt = time.perf_counter() - t
    return {"value": 4 * sample / dt / 1e9, "unit": "decoded GB/s", "cores": 1, "kind": "oracle",
            "sample": f"first {sample:,} rows of the same encoded column: Alg. 1 decode per entry + int64 sum "
                      f"(oracle/oracle.c, 1 thread), {dt:.1f} s", "checksum": int(s)}


def run_reference(args):
    """--impl reference: the oracle as it stands on the host cores, same metric/config."""
    rank, world, _ = dist_env()
    if rank != 0:
        return
    import oracle
    from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp  # host encoder only (no GPU call)
    x = make_column(args.bits, args.rows, 0)
    h = tp.encode(x, "for")
    sample = min(args.rows, 25_000_000)
    e = oracle.Encoded(scheme="for", header=h.header(), starts=h.starts0[: h.col.num_blocks + 1],
                       data=h.data0[: h.col.words0])
    for _ in range(args.warmup):
        oracle.column_sum(oracle.for_decode_range(e, 0, min(sample, 1_000_000), h.data0))
    times = []
    for _ in range(args.steps if args.steps <= 20 else 20):
        t = time.perf_counter()
        oracle.column_sum(oracle.for_decode_range(e, 0, sample, h.data0))
        times.append(time.perf_counter() - t)
    ms = 1e3 * sum(times) / len(times)
    value = 4 * sample / (ms / 1e3) / 1e9
    line = {"impl": "reference", "metric": "decoded GB/s (GPU-FOR decode-only, fused int64 sum)", "value": value,
            "unit": "GB/s", "n_gpus": world, "steps": len(times), "warmup": args.warmup, "ms_per_step": ms,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32",
            "data": "synthetic",
            "config": {"workload": f"C2 GPU-FOR b={args.bits} U[0,2^{args.bits}) {args.rows:,} rows, decode->sum",
                       "sample_rows_per_step": sample},
            "cpu_baseline": {"value": value, "unit": "GB/s", "cores": 1, "kind": "oracle",
                             "sample": f"first {sample:,} rows per step, Alg. 1 per entry, 1 thread"},
            "e2e": {"value": value, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    import torch
    import torch.distributed as dist

    rank, world, local = dist_env()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp

    # ---------------- setup (untimed): generate + encode on the host, copy once
    t_setup = time.perf_counter()
    x = make_column(args.bits, args.rows, rank)
    t_enc = time.perf_counter()
    h = tp.encode(x, "for")
    enc_s = time.perf_counter() - t_enc
    d = h.to_device(dev)
    comp_bytes = h.nbytes()
    truth = int(x.astype(np.int64).sum())
    stream = torch.cuda.current_stream(dev)
    acc = torch.zeros(1, dtype=torch.int64, device=dev)

    def step():
        acc.zero_()
        tp.tp_decode_sum(d.col, acc, stream)
        if world > 1:
            dist.all_reduce(acc)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    got = int(acc.item())
    want = truth
    if world > 1:
        tt = torch.tensor([truth], dtype=torch.int64, device=dev)
        dist.all_reduce(tt)
        want = int(tt.item())
    assert got == want, f"checksum mismatch: {got} != {want}"

    # ---------------- timed region: K steps, per-launch events for the dominant kernel
    ev_k = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    l0 = tp.tp_launch_count()
    with ClockSampler(local) as clk:
        start.record(stream)
        for i in range(args.steps):
            acc.zero_()
            ev_k[i][0].record(stream)
            tp.tp_decode_sum(d.col, acc, stream)
            ev_k[i][1].record(stream)
            if world > 1:
                dist.all_reduce(acc)
        end.record(stream)
        torch.cuda.synchronize()
    launches = tp.tp_launch_count() - l0
    if world > 1:
        dist.barrier()
    ms_total = start.elapsed_time(end)
    k_ms = [a.elapsed_time(b) for a, b in ev_k]
    tm = torch.tensor([ms_total], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tm, op=dist.ReduceOp.MAX)
    ms_step = float(tm.item()) / args.steps
    rows_all = args.rows * world
    value = 4 * rows_all / (ms_step / 1e3) / 1e9
    k_avg = sum(k_ms) / len(k_ms)
    peak, peak_src = measured_peak()
    achieved = comp_bytes / (k_avg / 1e3) / 1e9

    # ---------------- e2e: host buffers through the C ABI, H2D + decode + D2H inside the timed region
    pin = {k: torch.from_numpy(v.view(np.int32)).pin_memory() for k, v in
           (("starts0", h.starts0), ("data0", h.data0))}
    dst = {k: torch.empty_like(v, device=dev) for k, v in pin.items()}
    col = tp.tp_column()
    import ctypes
    ctypes.pointer(col)[0] = h.col
    col.starts0, col.data0 = dst["starts0"].data_ptr(), dst["data0"].data_ptr()
    host_sum = torch.zeros(1, dtype=torch.int64).pin_memory()
    h2d = sum(v.numel() * 4 for v in pin.values())

    def e2e_step():
        for k in pin:
            dst[k].copy_(pin[k], non_blocking=True)
        acc.zero_()
        tp.tp_decode_sum(col, acc, stream)
        if world > 1:
            dist.all_reduce(acc)
        host_sum.copy_(acc, non_blocking=True)

    e2e_step()
    torch.cuda.synchronize()
    assert int(host_sum.item()) == want
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(args.e2e_steps):
        e2e_step()
    e1.record(stream)
    torch.cuda.synchronize()
    te = torch.tensor([e0.elapsed_time(e1) / args.e2e_steps], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
    e2e_ms = float(te.item())

    # ---------------- the "None" roof (uncompressed int32 read of the same consumer), rank-local
    none_gbs = None
    try:
        xd = torch.from_numpy(x).to(dev)
        tp.tp_plain_sum(xd, args.rows, acc, stream)
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        for _ in range(20):
            tp.tp_plain_sum(xd, args.rows, acc, stream)
        b.record(stream)
        torch.cuda.synchronize()
        none_gbs = 4 * args.rows / (a.elapsed_time(b) / 20 / 1e3) / 1e9
        del xd
    except Exception:
        pass

    sweep = None
    if args.sweep:
        sweep = run_sweep(args, tp, dev, stream, torch)

    if rank == 0:
        sms, occ = tp.tp_device_info()
        line = {
            "metric": "decoded GB/s (GPU-FOR decode-only, fused int64 sum)",
            "value": value, "unit": "GB/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": ms_step, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": value / PAPER_DECODED_GBS if world == 1 else None,
            "dtype": "int32", "data": "synthetic",
            "config": {"workload": f"C2 GPU-FOR b={args.bits}: {args.rows:,} int32 U[0,2^{args.bits}) per GPU, "
                                   "decode fused into int64 sum (paper E1, P:720-724)",
                       "rows_per_gpu": args.rows, "bits": args.bits, "compressed_bytes_per_gpu": comp_bytes,
                       "bits_per_int": 8 * comp_bytes / args.rows,
                       "l2": "inputs larger than L2 (compressed column > 8x 126 MB), no flush",
                       "grid": f"{sms} SMs x {occ} CTAs, 160 threads (1 TMA producer warp + 4 consumer warps)",
                       "parallelism": f"tile-range partitions, {world} GPU(s), NCCL allreduce of the partial sum"},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": ncu_traffic(f"for_b{args.bits}_sum"),
                         "kernel": "k_decode_sum", "kernel_avg_ms": k_avg,
                         "algorithmic_bytes_per_launch": comp_bytes, "peak_source": peak_src},
            "e2e": {"value": 4 * rows_all / (e2e_ms / 1e3) / 1e9, "unit": "GB/s", "ms_per_step": e2e_ms,
                    "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": 8,
                    "path": "pinned host arrays -> tp_decode_sum (C ABI) -> 8-byte result to host"},
            "gpu_launches": int(launches),
            "clocks": clk.summary(),
            "context": {"paper_v100_decoded_gbs": PAPER_DECODED_GBS,
                        "none_uncompressed_read_gbs": none_gbs,
                        "host_encode_s": enc_s, "setup_s": time.perf_counter() - t_setup},
        }
        if sweep is not None:
            line["sweep"] = sweep
        if world == 1 and not args.no_cpu_baseline:
            line["cpu_baseline"] = cpu_baseline(h, args.rows)
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def run_sweep(args, tp, dev, stream, torch):
    """Bitwidth sweep 0..32 (BASELINE config 2): per-b kernel time, decoded + compressed GB/s."""
    peak, _ = measured_peak()
    out = {}
    acc = torch.zeros(1, dtype=torch.int64, device=dev)
    for b in range(33):
        x = make_column(b, args.rows, 0)
        h = tp.encode(x, "for")
        d = h.to_device(dev)
        truth = int(x.astype(np.int64).sum())
        del x
        for _ in range(3):
            acc.zero_()
            tp.tp_decode_sum(d.col, acc, stream)
        torch.cuda.synchronize()
        assert int(acc.item()) == truth
        flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
        ts = []
        for _ in range(10):
            flush.sum()  # L2 flush by reading (no dirty lines to write back)
            a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            tp.tp_decode_sum(d.col, acc, stream)
            e.record(stream)
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(e))
        ms = statistics.median(ts)
        cb = h.nbytes()
        out[str(b)] = {"ms": ms, "decoded_gbs": 4 * args.rows / ms / 1e6, "compressed_gbs": cb / ms / 1e6,
                       "hbm_frac": cb / ms / 1e6 / peak, "bits_per_int": 8 * cb / args.rows}
        del d, h, flush
        torch.cuda.empty_cache()
    return out


if __name__ == "__main__":
    main()
