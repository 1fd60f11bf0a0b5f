"""SSB: the oracle's SQL semantics pinned by a row-at-a-time brute force and by
subset invariants; the GPU star-join kernel vs the oracle (exact int64 results)."""
import numpy as np
import pytest

import datagen.ssb as gen
from oracle import ssb as ossb

QUERIES = ossb.QUERIES


@pytest.fixture(scope="module")
def tiny():
    return gen.generate(0.01, seed=11)


def _brute(db, qid):
    """row-at-a-time SQL with dict joins (independent of the vectorised oracle)."""
    lo, d, c, s, p = db["lineorder"], db["date"], db["customer"], db["supplier"], db["part"]
    D = {int(k): i for i, k in enumerate(d["d_datekey"])}
    C = {int(k): i for i, k in enumerate(c["c_custkey"])}
    S = {int(k): i for i, k in enumerate(s["s_suppkey"])}
    Pk = {int(k): i for i, k in enumerate(p["p_partkey"])}
    out = {}
    n = len(lo["lo_orderdate"])
    for r in range(n):
        di = D[int(lo["lo_orderdate"][r])]
        year, ym, wk = int(d["d_year"][di]), int(d["d_yearmonthnum"][di]), int(d["d_weeknuminyear"][di])
        disc, qty = int(lo["lo_discount"][r]), int(lo["lo_quantity"][r])
        rev, cost, ext = int(lo["lo_revenue"][r]), int(lo["lo_supplycost"][r]), int(lo["lo_extendedprice"][r])
        ci, si, pi = C[int(lo["lo_custkey"][r])], S[int(lo["lo_suppkey"][r])], Pk[int(lo["lo_partkey"][r])]
        cr, cn, cc = int(c["c_region"][ci]), int(c["c_nation"][ci]), int(c["c_city"][ci])
        sr, sn, sc = int(s["s_region"][si]), int(s["s_nation"][si]), int(s["s_city"][si])
        mf, cat, br = int(p["p_mfgr"][pi]), int(p["p_category"][pi]), int(p["p_brand1"][pi])
        key, val = None, None
        if qid == "1.1" and year == 1993 and 1 <= disc <= 3 and qty < 25:
            key, val = (), ext * disc
        elif qid == "1.2" and ym == 199401 and 4 <= disc <= 6 and 26 <= qty <= 35:
            key, val = (), ext * disc
        elif qid == "1.3" and wk == 6 and year == 1994 and 5 <= disc <= 7 and 26 <= qty <= 35:
            key, val = (), ext * disc
        elif qid == "2.1" and cat == 12 and sr == 1:
            key, val = (year, br), rev
        elif qid == "2.2" and 2221 <= br <= 2228 and sr == 2:
            key, val = (year, br), rev
        elif qid == "2.3" and br == 2239 and sr == 3:
            key, val = (year, br), rev
        elif qid == "3.1" and cr == 2 and sr == 2 and 1992 <= year <= 1997:
            key, val = (cn, sn, year), rev
        elif qid == "3.2" and cn == 24 and sn == 24 and 1992 <= year <= 1997:
            key, val = (cc, sc, year), rev
        elif qid == "3.3" and cc in (231, 235) and sc in (231, 235) and 1992 <= year <= 1997:
            key, val = (cc, sc, year), rev
        elif qid == "3.4" and cc in (231, 235) and sc in (231, 235) and ym == 199712:
            key, val = (cc, sc, year), rev
        elif qid == "4.1" and cr == 1 and sr == 1 and mf in (1, 2):
            key, val = (year, cn), rev - cost
        elif qid == "4.2" and cr == 1 and sr == 1 and year in (1997, 1998) and mf in (1, 2):
            key, val = (year, sn, cat), rev - cost
        elif qid == "4.3" and cr == 1 and sn == 24 and year in (1997, 1998) and cat == 14:
            key, val = (year, sc, br), rev - cost
        if key is not None:
            out[key] = out.get(key, 0) + val
    if qid.startswith("1."):
        return [(out.get((), 0),)]
    rows = [(*k, v) for k, v in out.items()]
    if qid.startswith("3."):
        return sorted(rows, key=lambda r: (r[2], -r[3], r[0], r[1]))
    return sorted(rows)


@pytest.mark.parametrize("qid", QUERIES)
def test_oracle_matches_row_at_a_time_sql(tiny, qid):
    assert ossb.SSB(tiny).run(qid) == _brute(tiny, qid)


def test_oracle_subset_invariants():
    db = gen.generate(0.05, seed=3)
    o = ossb.SSB(db)
    q33 = {r[:3]: r[3] for r in o.q33()}
    for r in o.q34():            # q3.4 rows are q3.3 rows restricted to Dec 1997
        assert 0 < r[3] <= q33[r[:3]]
    q42 = {r[:3]: r[3] for r in o.q42()}
    by_year = {}
    for y, city, brand, v in o.q43():  # q4.3 = q4.2 restricted to s_nation US, category 14
        by_year[y] = by_year.get(y, 0) + v
    for y, v in by_year.items():
        assert q42[(y, 24, 14)] == v
    # q1.1's revenue over the whole year 1993 == the sum of the per-week q1.3-style slices
    assert o.q11()[0][0] > 0


def test_generator_shape():
    db = gen.generate(1, seed=5000)
    lo = db["lineorder"]
    n = len(lo["lo_orderdate"])
    assert 5_900_000 < n < 6_100_000                      # ~6M rows per SF
    runs = np.count_nonzero(np.diff(lo["lo_orderdate"])) + 1
    assert 3.5 < n / runs < 4.5                             # orders of 1..7 lines
    assert lo["lo_quantity"].min() == 1 and lo["lo_quantity"].max() == 50
    assert lo["lo_discount"].min() == 0 and lo["lo_discount"].max() == 10


@pytest.mark.gpu
@pytest.mark.parametrize("sf", [0.05, 1])
def test_gpu_star_queries_match_oracle(sf):
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sigmod_shanbhagyym22_b200.ssb import SSBEngine
    db = gen.generate(sf, seed=5000)
    o = ossb.SSB(db)
    eng = SSBEngine(db)
    for qid in QUERIES:
        assert eng.run(qid) == o.run(qid), qid


@pytest.mark.gpu
def test_gpu_star_queries_sharded_sum_equals_whole():
    """tile-range shards: per-shard group arrays add up to the unsharded ones."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sigmod_shanbhagyym22_b200.ssb import SSBEngine
    db = gen.generate(0.2, seed=8)
    n = len(db["lineorder"]["lo_orderdate"])
    cuts = [0, 512 * 301, 512 * 777, n]
    whole = SSBEngine(db)
    parts = [SSBEngine(db, rows=(cuts[i], cuts[i + 1])) for i in range(3)]
    for qid in ("1.1", "2.1", "3.2", "4.3"):
        pw = whole.prepare(qid)
        sw, cw = whole.execute(pw)
        acc_s = torch.zeros_like(sw)
        acc_c = torch.zeros_like(cw)
        for e in parts:
            pp = e.prepare(qid)
            e.execute(pp, acc_s, acc_c)
        assert torch.equal(acc_s, sw) and torch.equal(acc_c, cw), qid


def test_generator_rank_slices_concatenate():
    """Rank-local generation (bench / multi-GPU): the row slices of the chunked generator are the
    rows of the whole table, for ragged 512-row tile-range cuts."""
    from paper_conf_sigmod_shanbhagyym22_b200.dist import tile_range
    whole = gen.generate(0.3, seed=9)
    n = whole["lineorder_rows"]
    assert n == len(whole["lineorder"]["lo_orderdate"]) == gen.num_rows(0.3, seed=9)
    for world in (3, 8):
        parts = [gen.generate(0.3, seed=9, rows=tile_range(n, r, world)) for r in range(world)]
        for c in ("lo_orderdate", "lo_custkey", "lo_revenue", "lo_supplycost"):
            assert np.array_equal(np.concatenate([p["lineorder"][c] for p in parts]), whole["lineorder"][c])


@pytest.mark.gpu
@pytest.mark.slow
def test_gpu_star_queries_sf20_match_golden():
    """BASELINE config 5 at the bench's size (SF 20, 120M rows, GPU-* columns, the bench's launch
    configuration): every query == the oracle's answer stored by scripts/make_ssb_golden.py
    (oracle/ssb.py over the uncompressed columns)."""
    import json
    import os
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sigmod_shanbhagyym22_b200.ssb import SSBEngine
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "ssb_sf20.json")))
    db = gen.generate(20, seed=g["seed"], columns=gen.QUERY_COLUMNS)
    assert db["lineorder_rows"] == g["rows"]
    eng = SSBEngine(db)
    for qid in QUERIES:
        assert [list(r) for r in eng.run(qid)] == g["results"][qid], qid
