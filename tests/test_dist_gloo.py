"""Multi-process (world size 2, gloo, CPU) coverage of the multi-GPU host logic: tile-range
partitioning, per-rank shard columns (tp_shard), and the allreduce combine of per-rank partial
aggregates.  The per-rank "kernel" here is the CPU oracle decoding the rank's shard (no GPU in
this container); the result must equal the unsharded answer."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import datagen
import oracle
from paper_conf_sigmod_shanbhagyym22_b200 import dist as tpd
from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp

WORLD = 2


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _cols(n):
    return {"for": datagen.uniform_bits(13, n, seed=1), "dfor": datagen.near_sorted(n, seed=2),
            "rfor": datagen.runs(n, 6, seed=3)}


def _oracle_decode(sc):
    h = sc.header()
    nb = int(sc.col.num_blocks)
    if sc.scheme == "rfor":
        e = oracle.Encoded(scheme="rfor", header=h, startsV=sc.starts0[:nb + 1], dataV=sc.data0[:sc.col.words0],
                           startsL=sc.starts1[:nb + 1], dataL=sc.data1[:sc.col.words1])
    else:
        e = oracle.Encoded(scheme=sc.scheme, header=h, starts=sc.starts0[:nb + 1], data=sc.data0[:sc.col.words0])
    return oracle.decode(e)


def _worker(rank, port, n, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=WORLD)
    try:
        res = {}
        cols = _cols(n)
        for scheme, x in cols.items():
            sc = tpd.shard(tp.encode(x, scheme), rank, WORLD)
            lo, hi = sc.rows
            part = _oracle_decode(sc)
            assert np.array_equal(part, x[lo:hi])
            t = torch.tensor([oracle.column_sum(part), hi - lo], dtype=torch.int64)
            tpd.combine([t])
            res[scheme] = t.tolist()
        # a fused select/project/aggregate over the shard's decoded columns, combined
        parts = [_oracle_decode(tpd.shard(tp.encode(x, s), rank, WORLD)) for s, x in cols.items()]
        q = torch.tensor([oracle.select_project_sum(parts, [0, 0, 0], [4000, 2**31 - 1, 30000], "mul", 0, 2)],
                         dtype=torch.int64)
        tpd.combine([q])
        res["query"] = int(q.item())
        out[rank] = res
    finally:
        dist.destroy_process_group()


def test_tile_ranges_partition_the_column():
    for n in (1, 511, 512, 513, 512 * 7 + 3, 10**6):
        for world in (1, 2, 3, 8):
            rs = [tpd.tile_range(n, r, world) for r in range(world)]
            assert rs[0][0] == 0 and rs[-1][1] == n
            for (a, b), (c, d) in zip(rs, rs[1:]):
                assert b == c and a % 512 == 0
            assert all(b >= a for a, b in rs)


@pytest.mark.timeout(300)
def test_two_rank_gloo_combine_equals_unsharded():
    n = 512 * 37 + 101
    out = mp.Manager().dict()
    mp.spawn(_worker, args=(_free_port(), n, out), nprocs=WORLD, join=True)
    cols = _cols(n)
    for scheme, x in cols.items():
        for r in range(WORLD):
            assert out[r][scheme] == [oracle.column_sum(x), n], (scheme, r)
    want = oracle.select_project_sum(list(cols.values()), [0, 0, 0], [4000, 2**31 - 1, 30000], "mul", 0, 2)
    assert out[0]["query"] == out[1]["query"] == want


def _ssb_worker(rank, port, sf, out):
    """bench.py's SSB leg on one rank, with the oracle as the per-rank kernel: the rank generates
    ONLY its 512-row tile range of lineorder (datagen.ssb rows=, as bench.ssb_leg does), answers
    every query on it, and the dense per-group partials are combined with one allreduce each."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=WORLD)
    try:
        import datagen.ssb as gen
        from oracle import ssb as ossb
        total = gen.num_rows(sf, seed=5000)
        r0, r1 = tpd.tile_range(total, rank, WORLD)
        db = gen.generate(sf, seed=5000, columns=gen.QUERY_COLUMNS, rows=(r0, r1))
        assert len(db["lineorder"]["lo_orderdate"]) == r1 - r0
        whole = ossb.SSB(gen.generate(sf, seed=5000, columns=gen.QUERY_COLUMNS))
        part = ossb.SSB(db)
        res = {}
        for q in ossb.QUERIES:
            want = whole.run(q)
            keys = [tuple(r[:-1]) for r in want]           # the group space, identical on every rank
            got = {tuple(r[:-1]): r[-1] for r in part.run(q)}
            assert set(got) - set(keys) <= {()}, q           # a shard never invents a group
            dense = torch.tensor([got.get(k, 0) for k in keys], dtype=torch.int64)
            tpd.combine([dense])                             # the GPU path's allreduce of partials
            res[q] = [list(k) + [int(v)] for k, v in zip(keys, dense.tolist())] == [list(r) for r in want]
        out[rank] = res
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(600)
def test_two_rank_gloo_ssb_leg_equals_unsharded():
    out = mp.Manager().dict()
    mp.spawn(_ssb_worker, args=(_free_port(), 0.05, out), nprocs=WORLD, join=True)
    for r in range(WORLD):
        assert all(out[r].values()), out[r]
