"""TEST INFRASTRUCTURE ONLY -- SSB query semantics over UNCOMPRESSED columns.

The 13 Star Schema Benchmark queries (SSB spec [35], used in P:1874-1888; query text as
listed in SURVEY.md Appendix B) evaluated literally: equi-joins of lineorder foreign keys
with the dimension primary keys, the WHERE predicates on dimension attributes (date
predicates through the date dimension, not rewritten to key ranges), GROUP BY with int64
sums (R24) and ORDER BY (ties by group key ascending, R23).  String attributes are the
dictionary codes of datagen.ssb.  No compression code is involved: the
paper's invariant is that GPU-* and None give the same answers.

Each query returns a list of tuples: group attributes in SELECT order, then the aggregate.
"""
from __future__ import annotations

import numpy as np

AMERICA, ASIA, EUROPE = 1, 2, 3
UNITED_STATES = 24
UKI1, UKI5 = 231, 235  # 'UNITED KI1', 'UNITED KI5'


def _join(fk: np.ndarray, pk: np.ndarray) -> np.ndarray:
    """row index in the dimension of each foreign key (equi-join on a unique key)."""
    order = np.argsort(pk, kind="stable")
    pos = np.searchsorted(pk[order], fk)
    pos = np.minimum(pos, len(pk) - 1)
    idx = order[pos]
    assert np.array_equal(pk[idx], fk), "dangling foreign key"
    return idx


def _group_sum(keys: list, vals: np.ndarray) -> dict:
    """GROUP BY keys (list of int arrays) -> {tuple: int64 sum}."""
    if len(vals) == 0:
        return {}
    stacked = np.stack([k.astype(np.int64) for k in keys], axis=1)
    uniq, inv = np.unique(stacked, axis=0, return_inverse=True)
    sums = np.zeros(len(uniq), np.int64)
    np.add.at(sums, inv.reshape(-1), vals.astype(np.int64))
    return {tuple(int(x) for x in u): int(s) for u, s in zip(uniq, sums)}


class SSB:
    def __init__(self, db: dict):
        self.db = db
        lo = db["lineorder"]
        self.lo = lo
        self.d = db["date"]
        self.c = db["customer"]
        self.s = db["supplier"]
        self.p = db["part"]
        self.di = _join(lo["lo_orderdate"], self.d["d_datekey"])
        self._ci = self._si = self._pi = None

    @property
    def ci(self):
        if self._ci is None:
            self._ci = _join(self.lo["lo_custkey"], self.c["c_custkey"])
        return self._ci

    @property
    def si(self):
        if self._si is None:
            self._si = _join(self.lo["lo_suppkey"], self.s["s_suppkey"])
        return self._si

    @property
    def pi(self):
        if self._pi is None:
            self._pi = _join(self.lo["lo_partkey"], self.p["p_partkey"])
        return self._pi

    # ---------------------------------------------------------------- flight 1
    def _q1(self, date_pred, dlo, dhi, qlo, qhi):
        lo = self.lo
        m = date_pred & (lo["lo_discount"] >= dlo) & (lo["lo_discount"] <= dhi) & \
            (lo["lo_quantity"] >= qlo) & (lo["lo_quantity"] <= qhi)
        rev = (lo["lo_extendedprice"][m].astype(np.int64) * lo["lo_discount"][m].astype(np.int64)).sum()
        return [(int(rev),)]

    def q11(self):
        # where lo_orderdate = d_datekey and d_year = 1993 and lo_discount between 1 and 3 and lo_quantity < 25
        return self._q1(self.d["d_year"][self.di] == 1993, 1, 3, -2**31, 24)

    def q12(self):
        # d_yearmonthnum = 199401, lo_discount between 4 and 6, lo_quantity between 26 and 35
        return self._q1(self.d["d_yearmonthnum"][self.di] == 199401, 4, 6, 26, 35)

    def q13(self):
        # d_weeknuminyear = 6 and d_year = 1994, lo_discount between 5 and 7, lo_quantity between 26 and 35
        dp = (self.d["d_weeknuminyear"][self.di] == 6) & (self.d["d_year"][self.di] == 1994)
        return self._q1(dp, 5, 7, 26, 35)

    # ---------------------------------------------------------------- flight 2
    def _q2(self, part_pred, region):
        lo = self.lo
        m = part_pred & (self.s["s_region"][self.si] == region)
        g = _group_sum([self.d["d_year"][self.di][m], self.p["p_brand1"][self.pi][m]], lo["lo_revenue"][m])
        return sorted((k[0], k[1], v) for k, v in g.items())  # order by d_year, p_brand1

    def q21(self):
        return self._q2(self.p["p_category"][self.pi] == 12, AMERICA)   # 'MFGR#12', 'AMERICA'

    def q22(self):
        b = self.p["p_brand1"][self.pi]
        return self._q2((b >= 2221) & (b <= 2228), ASIA)                # between 'MFGR#2221' and 'MFGR#2228'

    def q23(self):
        return self._q2(self.p["p_brand1"][self.pi] == 2239, EUROPE)     # 'MFGR#2239', 'EUROPE'

    # ---------------------------------------------------------------- flight 3
    def _q3(self, m, ckey, skey):
        lo = self.lo
        g = _group_sum([ckey[m], skey[m], self.d["d_year"][self.di][m]], lo["lo_revenue"][m])
        rows = [(k[0], k[1], k[2], v) for k, v in g.items()]
        return sorted(rows, key=lambda r: (r[2], -r[3], r[0], r[1]))  # d_year asc, revenue desc (R23)

    def q31(self):
        y = self.d["d_year"][self.di]
        m = (self.c["c_region"][self.ci] == ASIA) & (self.s["s_region"][self.si] == ASIA) & (y >= 1992) & (y <= 1997)
        return self._q3(m, self.c["c_nation"][self.ci], self.s["s_nation"][self.si])

    def q32(self):
        y = self.d["d_year"][self.di]
        m = (self.c["c_nation"][self.ci] == UNITED_STATES) & (self.s["s_nation"][self.si] == UNITED_STATES) & \
            (y >= 1992) & (y <= 1997)
        return self._q3(m, self.c["c_city"][self.ci], self.s["s_city"][self.si])

    def _cities(self):
        cc, sc = self.c["c_city"][self.ci], self.s["s_city"][self.si]
        return ((cc == UKI1) | (cc == UKI5)) & ((sc == UKI1) | (sc == UKI5)), cc, sc

    def q33(self):
        y = self.d["d_year"][self.di]
        m, cc, sc = self._cities()
        return self._q3(m & (y >= 1992) & (y <= 1997), cc, sc)

    def q34(self):
        m, cc, sc = self._cities()
        return self._q3(m & (self.d["d_yearmonth"][self.di] == 199712), cc, sc)   # d_yearmonth = 'Dec1997'

    # ---------------------------------------------------------------- flight 4
    def _profit(self, m):
        return self.lo["lo_revenue"][m].astype(np.int64) - self.lo["lo_supplycost"][m].astype(np.int64)

    def q41(self):
        mf = self.p["p_mfgr"][self.pi]
        m = (self.c["c_region"][self.ci] == AMERICA) & (self.s["s_region"][self.si] == AMERICA) & \
            ((mf == 1) | (mf == 2))
        g = _group_sum([self.d["d_year"][self.di][m], self.c["c_nation"][self.ci][m]], self._profit(m))
        return sorted((k[0], k[1], v) for k, v in g.items())

    def q42(self):
        mf = self.p["p_mfgr"][self.pi]
        y = self.d["d_year"][self.di]
        m = (self.c["c_region"][self.ci] == AMERICA) & (self.s["s_region"][self.si] == AMERICA) & \
            ((y == 1997) | (y == 1998)) & ((mf == 1) | (mf == 2))
        g = _group_sum([y[m], self.s["s_nation"][self.si][m], self.p["p_category"][self.pi][m]], self._profit(m))
        return sorted((k[0], k[1], k[2], v) for k, v in g.items())

    def q43(self):
        y = self.d["d_year"][self.di]
        m = (self.c["c_region"][self.ci] == AMERICA) & (self.s["s_nation"][self.si] == UNITED_STATES) & \
            ((y == 1997) | (y == 1998)) & (self.p["p_category"][self.pi] == 14)
        g = _group_sum([y[m], self.s["s_city"][self.si][m], self.p["p_brand1"][self.pi][m]], self._profit(m))
        return sorted((k[0], k[1], k[2], v) for k, v in g.items())

    def run(self, qid: str):
        return getattr(self, "q" + qid.replace(".", ""))()


QUERIES = ("1.1", "1.2", "1.3", "2.1", "2.2", "2.3", "3.1", "3.2", "3.3", "3.4", "4.1", "4.2", "4.3")
