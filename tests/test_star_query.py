"""tp_star_query (the fused decode -> filter -> probe -> group -> aggregate pass, P:1179-1188,
P:1874-1888) on seeded synthetic columns of every scheme, against oracle.star_query (the
plain definition).  The GPU cases run each query with the kernel forced to evaluate every
column densely (TILEPACK_SPARSE_MAX=0), sparsely (=1024) and with the default switch, so
both evaluation modes and the RFOR per-run probe are covered.  Integer results: exact."""
import os

import numpy as np
import pytest

import datagen
import oracle

N = 512 * 37 + 77  # several CTAs' tile ranges and a ragged tail


def _inputs(seed):
    rng = np.random.default_rng(seed)
    runs = datagen.runs(N, 4, seed=seed)                        # RFOR-friendly key column
    keys = (runs % 3000).astype(np.int32)
    fk = rng.integers(0, 2000, N, dtype=np.int32)               # FOR key column
    qty = rng.integers(1, 51, N, dtype=np.int32)
    price = rng.integers(-(1 << 20), 1 << 24, N, dtype=np.int32)
    cost = rng.integers(0, 1 << 17, N, dtype=np.int32)
    srt = datagen.near_sorted(N, seed=seed + 1)                 # DFOR column
    t1 = np.where(rng.random(3000) < 0.3, rng.integers(0, 7, 3000), -1).astype(np.int32)
    t2 = np.where(rng.random(2000) < 0.5, rng.integers(0, 25, 2000), -1).astype(np.int32)
    short = (datagen.runs(N, 1, seed=seed + 2) % 3000).astype(np.int32)   # RFOR, 512 runs per block
    long_ = (datagen.runs(N, 100, seed=seed + 3) % 3000).astype(np.int32)  # RFOR, runs across many lanes
    return dict(keys=keys, fk=fk, qty=qty, price=price, cost=cost, srt=srt, t1=t1, t2=t2, short=short, long=long_)


def _cases(d):
    """(columns, schemes, roles, agg, ngroups)"""
    lo_s, hi_s = int(np.quantile(d["srt"], 0.2)), int(np.quantile(d["srt"], 0.9))
    I32 = (-(2**31), 2**31 - 1)
    probe1 = dict(role="probe", table=d["t1"], key_min=0, stride=25)
    probe2 = dict(role="probe", table=d["t2"], key_min=0, stride=1)
    meas = lambda lo=I32[0], hi=I32[1]: dict(role="measure", lo=lo, hi=hi)  # noqa: E731
    return [
        # q1-like: range on a run column, staged filtered first measure, range, product
        (["keys", "price", "qty", "cost"], ["rfor", "for", "for", "for"],
         [dict(role="range", lo=100, hi=900), meas(-5000, 1 << 23), dict(role="range", lo=1, hi=24), meas()],
         "mul", 1),
        # grouped: RFOR probe first (per-run lookups), FOR probe, DFOR range, sum
        (["keys", "fk", "srt", "price"], ["rfor", "for", "dfor", "for"],
         [probe1, probe2, dict(role="range", lo=lo_s, hi=hi_s), meas()], "sum", 7 * 25),
        # grouped SUB with the staged first measure before a probe
        (["fk", "price", "keys", "cost"], ["for", "for", "rfor", "for"],
         [probe2, meas(), probe1, meas()], "sub", 7 * 25),
        # ungrouped SUB, measures on RFOR / DFOR columns
        (["qty", "keys", "srt"], ["for", "rfor", "dfor"],
         [dict(role="range", lo=10, hi=40), meas(), meas()], "sub", 1),
        # the uncompressed baseline (None) mixed with compressed columns
        (["keys", "fk", "qty", "price"], ["none", "rfor", "none", "for"],
         [probe1, probe2, dict(role="range", lo=5, hi=30), meas()], "sum", 7 * 25),
        (["price", "qty", "cost"], ["none", "none", "none"],
         [meas(-(1 << 19), 1 << 23), dict(role="range", lo=1, hi=24), meas()], "mul", 1),
        # grouped MUL, filter-only probe, no payload probe -> single group 0 of 3
        (["fk", "qty", "cost"], ["for", "for", "for"],
         [dict(role="probe", table=d["t2"], key_min=0, stride=0), meas(), meas(0, 60000)], "mul", 3),
        # grouped, the aggregating measure GPU-DFOR (dense path, no random access)
        (["fk", "srt"], ["for", "dfor"], [probe2, meas(lo_s, hi_s)], "sum", 25),
        # grouped, the aggregating measure GPU-RFOR (per alive row through its run number)
        (["fk", "keys"], ["for", "rfor"], [probe2, meas(100, 2000)], "sum", 25),
        # the first measure GPU-RFOR (staged per row), FOR range, FOR aggregating product
        (["keys", "qty", "price"], ["rfor", "for", "for"], [meas(0, 2500), dict(role="range", lo=1, hi=30), meas()],
         "mul", 1),
        # RFOR with one-row runs (512 runs per block: two passes of 8 entries per lane) as a range,
        # RFOR with runs of up to 199 rows (spanning lanes and blocks) as a grouped probe
        (["short", "long", "price"], ["rfor", "rfor", "for"],
         [dict(role="range", lo=0, hi=2000), dict(role="probe", table=d["t1"], key_min=0, stride=25), meas()],
         "sum", 7 * 25),
        # RFOR range first, a None first measure, a FOR probe, grouped difference
        (["keys", "price", "fk", "cost"], ["rfor", "none", "for", "for"],
         [dict(role="range", lo=0, hi=1500), meas(), probe2, meas()], "sub", 25),
        # ungrouped RFOR probe (filter only) on one-row runs, FOR first measure, product
        (["short", "cost", "price"], ["rfor", "for", "for"],
         [dict(role="probe", table=d["t1"], key_min=0, stride=0), meas(0, 90000), meas()], "mul", 1),
        # a selective FOR filter first (~20 of a warp's 1024 rows), then RFOR columns in every role
        # with few alive rows (the sparse RFOR path: run lengths + a binary search per row):
        # a grouped payload probe, a range, an RFOR first measure and an RFOR aggregating one
        (["qty", "keys", "short", "long", "keys"], ["for", "rfor", "rfor", "rfor", "rfor"],
         [dict(role="range", lo=7, hi=7), probe1, dict(role="range", lo=0, hi=2500), meas(), meas(0, 2900)],
         "sub", 7 * 25),
        (["qty", "long", "keys"], ["for", "rfor", "rfor"],
         [dict(role="range", lo=3, hi=3), dict(role="probe", table=d["t1"], key_min=0, stride=0), meas()],
         "sum", 1),
    ]


def test_oracle_star_query_brute_force():
    """pin the oracle's star_query against a per-row Python loop on a tiny input"""
    rng = np.random.default_rng(5)
    n = 300
    a = rng.integers(0, 40, n)
    b = rng.integers(-50, 50, n)
    c = rng.integers(0, 9, n)
    t = np.where(rng.random(40) < 0.6, rng.integers(0, 4, 40), -1)
    roles = [dict(role="probe", table=t, key_min=0, stride=3), dict(role="measure", lo=-20, hi=49),
             dict(role="range", lo=2, hi=7), dict(role="measure", lo=-(2**31), hi=2**31 - 1)]
    cols = [a, b, c, b * 2 + 1]
    for agg in ("sum", "mul", "sub"):
        sums = [0] * 12
        cnts = [0] * 12
        for i in range(n):
            if t[a[i]] < 0 or not (-20 <= b[i] <= 49) or not (2 <= c[i] <= 7):
                continue
            m0, m1 = int(b[i]), int(b[i] * 2 + 1)
            y = m1 if agg == "sum" else (m0 * m1 if agg == "mul" else m0 - m1)
            g = int(t[a[i]]) * 3
            sums[g] += y
            cnts[g] += 1
        s, k = oracle.star_query(cols, roles, agg, 12)
        assert list(s) == sums and list(k) == cnts, agg


@pytest.mark.gpu
@pytest.mark.parametrize("mode", ["dense", "sparse", "sparse64", "auto"])
def test_gpu_star_query_modes(mode, monkeypatch):
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp
    if mode != "auto":
        monkeypatch.setenv("TILEPACK_SPARSE_MAX", "0" if mode == "dense" else "1024")
        monkeypatch.setenv("TILEPACK_SPARSE_LANE_MAX", "0" if mode == "dense" else "32")
        # sparse64: up to two alive rows per lane in the sparse GPU-RFOR path
        monkeypatch.setenv("TILEPACK_RFOR_SPARSE_MAX", {"dense": "0", "sparse": "32", "sparse64": "64"}[mode])
    _run_cases(torch, tp, N, (1, 2), mode)


@pytest.mark.gpu
@pytest.mark.parametrize("ring", ["default", "tight"])
def test_gpu_star_query_long_columns(ring, monkeypatch):
    """20M rows: every CTA runs tens of rounds, so the byte ring wraps many times with items of
    very different sizes (RFOR 6-bit keys next to 25-bit FOR prices);
    'tight': the smallest ring the host allows (the largest item + the slack)."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp
    if ring == "tight":
        monkeypatch.setenv("TILEPACK_QUERY_RING_WORDS", "0")
    _run_cases(torch, tp, 20_000_000 + 333, (3,), "auto")
    assert tp.tp_device_errors() == 0


def _run_cases(torch, tp, n, seeds, mode):
    global N
    n0, N = N, n
    try:
        _run_cases_n(torch, tp, seeds, mode)
    finally:
        N = n0


def _run_cases_n(torch, tp, seeds, mode):
    for seed in seeds:
        d = _inputs(seed)
        dev = {}
        for ci, (names, schemes, roles, agg, G) in enumerate(_cases(d)):
            dcols, croles, keep = [], [], []
            for nm, sc, r in zip(names, schemes, roles):
                key = (nm, sc)
                if key not in dev:
                    dev[key] = tp.encode(d[nm], sc).to_device()
                dcols.append(dev[key].col)
                cr = tp.tp_star_col()
                cr.role = {"range": tp.TP_ROLE_RANGE, "probe": tp.TP_ROLE_PROBE, "measure": tp.TP_ROLE_MEASURE}[r["role"]]
                if r["role"] == "probe":
                    t = torch.from_numpy(r["table"]).cuda()
                    keep.append(t)
                    cr.table, cr.key_min, cr.table_len, cr.stride = t.data_ptr(), r["key_min"], len(r["table"]), r["stride"]
                else:
                    cr.lo, cr.hi = r["lo"], r["hi"]
                croles.append(cr)
            sums = torch.zeros(G, dtype=torch.int64, device="cuda")
            cnts = torch.zeros(G, dtype=torch.int64, device="cuda")
            tp.tp_star_query(dcols, croles, tp.TP_AGG[agg], sums, cnts, G)
            torch.cuda.synchronize()
            want_s, want_c = oracle.star_query([d[nm] for nm in names], roles, agg, G)
            assert np.array_equal(sums.cpu().numpy(), want_s), (mode, seed, ci)
            assert np.array_equal(cnts.cpu().numpy(), want_c), (mode, seed, ci)
    assert tp.tp_device_errors() == 0
