"""Seeded SSB-shaped data (Star Schema Benchmark [35], used at SF 20 in P:1874-1888).

Holds no compression arithmetic.  String attributes are emitted directly as dictionary
codes with the mapping of SURVEY.md Appendix B:
  region 0..4 (AFRICA, AMERICA, ASIA, EUROPE, MIDDLE EAST); nation 0..24 (TPC-H order,
  NATION_REGION below); city = nation*10 + digit ('UNITED KI1' = 231);
  p_mfgr m in 1..5; p_category = 10m + c, c in 1..5 ('MFGR#12' = 12);
  p_brand1 = 100*category + k, k in 1..40 ('MFGR#2221' = 2221);
  d_datekey = yyyymmdd, d_yearmonthnum = d_yearmonth = yyyymm, d_weeknuminyear = (doy-1)//7 + 1.
Lineorder keeps the dbgen run structure that decides GPU-* (P:1916-1918): orders of 1..7
lines, orderdate / custkey / orderpriority constant per order.
"""
from __future__ import annotations

import datetime as _dt
import math

import numpy as np

REGIONS = ["AFRICA", "AMERICA", "ASIA", "EUROPE", "MIDDLE EAST"]
NATIONS = ["ALGERIA", "ARGENTINA", "BRAZIL", "CANADA", "EGYPT", "ETHIOPIA", "FRANCE", "GERMANY", "INDIA",
           "INDONESIA", "IRAN", "IRAQ", "JAPAN", "JORDAN", "KENYA", "MOROCCO", "MOZAMBIQUE", "PERU", "CHINA",
           "ROMANIA", "SAUDI ARABIA", "VIETNAM", "RUSSIA", "UNITED KINGDOM", "UNITED STATES"]
NATION_REGION = np.array([0, 1, 1, 1, 4, 0, 3, 3, 2, 2, 4, 4, 2, 4, 0, 0, 0, 1, 2, 3, 4, 2, 3, 3, 1], np.int32)
AMERICA, ASIA, EUROPE = 1, 2, 3
UNITED_STATES, UNITED_KINGDOM = 24, 23

LINEORDER_COLUMNS = ("lo_orderkey", "lo_linenumber", "lo_custkey", "lo_partkey", "lo_suppkey", "lo_orderdate",
                     "lo_orderpriority", "lo_quantity", "lo_extendedprice", "lo_ordtotalprice", "lo_discount",
                     "lo_revenue", "lo_supplycost", "lo_tax", "lo_commitdate")
QUERY_COLUMNS = ("lo_orderdate", "lo_quantity", "lo_discount", "lo_extendedprice", "lo_partkey", "lo_suppkey",
                 "lo_revenue", "lo_custkey", "lo_supplycost")


def sizes(sf: float) -> dict:
    return {"customer": int(30_000 * sf), "supplier": int(2_000 * sf),
            "part": int(200_000 * math.floor(1 + math.log2(sf))) if sf >= 1 else int(200_000 * sf),
            "orders": int(1_500_000 * sf)}


def date_dim() -> dict:
    """1992-01-01 .. 1998-12-31 (the SSB date dimension, 7 years)."""
    d0 = _dt.date(1992, 1, 1)
    days = (_dt.date(1998, 12, 31) - d0).days + 1
    keys, year, ym, week = [], [], [], []
    for i in range(days):
        d = d0 + _dt.timedelta(days=i)
        keys.append(d.year * 10000 + d.month * 100 + d.day)
        year.append(d.year)
        ym.append(d.year * 100 + d.month)
        week.append((d.timetuple().tm_yday - 1) // 7 + 1)
    a = lambda v: np.array(v, np.int32)  # noqa: E731
    return {"d_datekey": a(keys), "d_year": a(year), "d_yearmonthnum": a(ym), "d_yearmonth": a(ym),
            "d_weeknuminyear": a(week)}


ORDER_CHUNK = 1 << 20  # orders per independently seeded chunk (rank-local generation)


def _dims(sf: float, seed: int) -> dict:
    rng = np.random.default_rng(seed)
    z = sizes(sf)
    C, S, P = z["customer"], z["supplier"], z["part"]
    date = date_dim()
    # dimensions (keys are dense 1..N; attributes uniform like dbgen)
    c_nation = rng.integers(0, 25, C, dtype=np.int32)
    customer = {"c_custkey": np.arange(1, C + 1, dtype=np.int32), "c_nation": c_nation,
                "c_region": NATION_REGION[c_nation], "c_city": c_nation * 10 + rng.integers(0, 10, C, dtype=np.int32)}
    s_nation = rng.integers(0, 25, S, dtype=np.int32)
    supplier = {"s_suppkey": np.arange(1, S + 1, dtype=np.int32), "s_nation": s_nation,
                "s_region": NATION_REGION[s_nation], "s_city": s_nation * 10 + rng.integers(0, 10, S, dtype=np.int32)}
    mfgr = rng.integers(1, 6, P, dtype=np.int32)
    cat = mfgr * 10 + rng.integers(1, 6, P, dtype=np.int32)
    brand = cat * 100 + rng.integers(1, 41, P, dtype=np.int32)
    pk = np.arange(1, P + 1, dtype=np.int64)
    retail = (90000 + (pk // 10) % 20001 + 100 * (pk % 1000)).astype(np.int32)  # TPC-H p_retailprice (cents)
    part = {"p_partkey": pk.astype(np.int32), "p_mfgr": mfgr, "p_category": cat, "p_brand1": brand}
    return {"date": date, "customer": customer, "supplier": supplier, "part": part, "retail": retail}


def _chunk_lines(seed: int, k: int, count: int) -> np.ndarray:
    """lines per order (1..7) of order chunk k: the first draw of the chunk's order stream."""
    return np.random.default_rng([seed, 1, k]).integers(1, 8, count, dtype=np.int64)


def _chunks(sf: float):
    O = sizes(sf)["orders"]
    return [(k, k * ORDER_CHUNK, min(O, (k + 1) * ORDER_CHUNK)) for k in range((O + ORDER_CHUNK - 1) // ORDER_CHUNK)]


def chunk_rows(sf: float, seed: int = 5000) -> np.ndarray:
    """lineorder rows of every order chunk (lines are drawn chunk by chunk, so this is cheap)."""
    return np.array([int(_chunk_lines(seed, k, o1 - o0).sum()) for k, o0, o1 in _chunks(sf)], np.int64)


def num_rows(sf: float, seed: int = 5000) -> int:
    return int(chunk_rows(sf, seed).sum())


def _gen_chunk(sf, seed, k, o0, o1, dims, want):
    z = sizes(sf)
    C, S, P = z["customer"], z["supplier"], z["part"]
    date = dims["date"]
    cnt = o1 - o0
    ro = np.random.default_rng([seed, 1, k])    # per-order stream (lines first, see _chunk_lines)
    lines = ro.integers(1, 8, cnt, dtype=np.int64)
    n = int(lines.sum())
    last = int(np.searchsorted(date["d_datekey"], 19980802)) + 1
    odate = date["d_datekey"][ro.integers(0, last, cnt)]   # orders dated 1992-01-01 .. 1998-08-02
    ocust = ro.integers(1, C + 1, cnt, dtype=np.int32)
    oprio = ro.integers(1, 6, cnt, dtype=np.int32)
    rl = np.random.default_rng([seed, 2, k])    # per-line stream
    okey = np.arange(o0 + 1, o1 + 1, dtype=np.int64)
    okey = (okey // 8) * 32 + okey % 8                      # sparse TPC-H-style order keys
    rep = lambda v: np.repeat(v, lines)  # noqa: E731
    lo = {}
    if "lo_orderkey" in want:
        lo["lo_orderkey"] = rep(okey).astype(np.int32)
    if "lo_linenumber" in want:
        starts = np.cumsum(lines) - lines
        lo["lo_linenumber"] = (np.arange(n, dtype=np.int64) - rep(starts) + 1).astype(np.int32)
    qty = rl.integers(1, 51, n, dtype=np.int32)
    disc = rl.integers(0, 11, n, dtype=np.int32)
    tax = rl.integers(0, 9, n, dtype=np.int32)
    lo_partkey = rl.integers(1, P + 1, n, dtype=np.int32)
    lo_suppkey = rl.integers(1, S + 1, n, dtype=np.int32)
    ext = qty * dims["retail"][lo_partkey - 1]              # < 50 * 2.1e6: fits int32
    rev = (ext.astype(np.int64) * (100 - disc) // 100).astype(np.int32)
    supplycost = rl.integers(100, 100_001, n, dtype=np.int32)
    commit_off = rl.integers(30, 91, n)
    if "lo_ordtotalprice" in want:
        otot = np.bincount(np.repeat(np.arange(cnt), lines), weights=rev, minlength=cnt).astype(np.int64)
        lo["lo_ordtotalprice"] = np.minimum(rep(otot), 2**31 - 1).astype(np.int32)
    lo_orderdate = rep(odate).astype(np.int32)
    if "lo_commitdate" in want:
        dayidx = np.searchsorted(date["d_datekey"], lo_orderdate)
        lo["lo_commitdate"] = date["d_datekey"][np.minimum(dayidx + commit_off,
                                                           len(date["d_datekey"]) - 1)].astype(np.int32)
    full = {"lo_custkey": lambda: rep(ocust).astype(np.int32), "lo_partkey": lambda: lo_partkey,
            "lo_suppkey": lambda: lo_suppkey, "lo_orderdate": lambda: lo_orderdate,
            "lo_orderpriority": lambda: rep(oprio).astype(np.int32), "lo_quantity": lambda: qty,
            "lo_extendedprice": lambda: ext, "lo_discount": lambda: disc, "lo_revenue": lambda: rev,
            "lo_supplycost": lambda: supplycost, "lo_tax": lambda: tax}
    for key, f in full.items():
        if key in want:
            lo[key] = f()
    return lo


def generate(sf: float, seed: int = 5000, columns=None, rows: tuple | None = None) -> dict:
    """Returns {'lineorder': {col: int32 array}, 'date': ..., 'customer': ..., 'supplier': ..., 'part': ...}.
    `columns` restricts the lineorder columns returned; `rows` = (r0, r1) returns only lineorder
    rows [r0, r1) (a rank's tile range) and generates only the order chunks that
    overlap them -- every chunk has its own seeded streams, so the values do not depend on
    `columns` or `rows`.  'lineorder_rows' is the whole table's row count either way."""
    dims = _dims(sf, seed)
    want = set(columns) if columns is not None else set(LINEORDER_COLUMNS)
    counts = chunk_rows(sf, seed)
    bounds = np.concatenate([[0], np.cumsum(counts)])
    total = int(bounds[-1])
    r0, r1 = rows if rows is not None else (0, total)
    assert 0 <= r0 <= r1 <= total
    parts = []
    for k, o0, o1 in _chunks(sf):
        c0, c1 = int(bounds[k]), int(bounds[k + 1])
        if c1 <= r0 or c0 >= r1:
            continue
        lo = _gen_chunk(sf, seed, k, o0, o1, dims, want)
        a, b = max(r0, c0) - c0, min(r1, c1) - c0
        parts.append({key: v[a:b] for key, v in lo.items()})
    cols = [c for c in LINEORDER_COLUMNS if c in want]
    lineorder = {c: (np.ascontiguousarray(np.concatenate([p[c] for p in parts])) if parts
                     else np.zeros(0, np.int32)) for c in cols}
    return {"sf": sf, "lineorder": lineorder, "lineorder_rows": total, "rows": (r0, r1), "date": dims["date"],
            "customer": dims["customer"], "supplier": dims["supplier"], "part": dims["part"]}
