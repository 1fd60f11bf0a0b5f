"""Multi-GPU plumbing: contiguous 512-row tile ranges per rank, one shard of
every encoded column per rank (rebased `block_starts`, `tp_shard`), and the combine step --
one allreduce (sum) of the per-rank partial aggregates (NCCL over NVLink on GPUs, gloo in
the CPU tests).  One process per GPU; torch.distributed supplies the process group.
"""
from __future__ import annotations

import ctypes

import numpy as np

from . import tilepack as tp

TILE = 512


def tile_range(n: int, rank: int, world: int) -> tuple[int, int]:
    """rows [lo, hi) of `rank`: tiles [T*rank/world, T*(rank+1)/world) of T = ceil(n/512)."""
    ntiles = (n + TILE - 1) // TILE
    lo = TILE * (ntiles * rank // world)
    hi = min(n, TILE * (ntiles * (rank + 1) // world))
    return lo, hi


class ShardColumn:
    """Rows [lo, hi) of a HostColumn as a self-contained host column (own arrays, guard words)."""

    def __init__(self, host: tp.HostColumn, lo: int, hi: int):
        rf = host.col.scheme == tp.TP_RFOR
        per = TILE if rf else 128
        nbv = -(-(hi - lo) // per)
        r0 = np.zeros(nbv + 1 + tp.GUARD_WORDS, np.uint32)
        r1 = np.zeros(nbv + 1 + tp.GUARD_WORDS, np.uint32) if rf else None
        view = tp.tp_shard(host.col, lo, hi, r0, r1)

        def take(ptr, words):
            a = np.zeros(words + tp.GUARD_WORDS, np.uint32)
            if words:
                a[:words] = np.ctypeslib.as_array((ctypes.c_uint32 * words).from_address(ptr))
            return a
        self.scheme = host.scheme
        self.starts0, self.data0 = r0, take(view.data0, int(view.words0))
        self.starts1 = r1
        self.data1 = take(view.data1, int(view.words1)) if rf else None
        col = tp.tp_column()
        ctypes.pointer(col)[0] = view
        col.starts0, col.data0 = self.starts0.ctypes.data, self.data0.ctypes.data
        if rf:
            col.starts1, col.data1 = self.starts1.ctypes.data, self.data1.ctypes.data
        self.col = col
        self.rows = (lo, hi)

    @property
    def n(self) -> int:
        return int(self.col.n)

    def header(self) -> np.ndarray:
        return np.array([self.col.block_size, self.col.miniblock_count, self.col.n], np.uint32)

    def to_device(self, device=None) -> tp.DeviceColumn:
        return tp.DeviceColumn(self, device)


def shard(host: tp.HostColumn, rank: int, world: int) -> ShardColumn:
    lo, hi = tile_range(host.n, rank, world)
    return ShardColumn(host, lo, hi)


def combine(tensors, group=None):
    """Sum the per-rank partial aggregates in place on every rank (one allreduce each)."""
    import torch.distributed as dist
    for t in tensors:
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return tensors
