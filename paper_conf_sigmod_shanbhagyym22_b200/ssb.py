"""SSB (Star Schema Benchmark) on compressed lineorder columns -- P:1874-1888, Fig. 11.

Declarative query plans for the 13 queries (SSB spec [35]; text in SURVEY.md App. B),
marshalled to the C ABI: `tp_lookup_build` builds the per-query dimension lookup tables on
the GPU (Crystal's perfect-hash build), `tp_star_query` runs the whole query in one tile
kernel over the GPU-*-encoded lineorder columns (decode -> filter -> probe -> group ->
aggregate).  The host only (a) dictionary-encodes dimension attributes to
dense codes before loading, (b) turns date predicates of flight 1 into
lo_orderdate key ranges read off the date dimension (the survey's allowed rewrite), and
(c) turns the few non-empty groups of the result into ORDER BY-sorted tuples.
"""
from __future__ import annotations

import numpy as np

from . import tilepack as tp

QUERIES = ("1.1", "1.2", "1.3", "2.1", "2.2", "2.3", "3.1", "3.2", "3.3", "3.4", "4.1", "4.2", "4.3")
QUERY_COLUMNS = ("lo_orderdate", "lo_quantity", "lo_discount", "lo_extendedprice", "lo_partkey", "lo_suppkey",
                 "lo_revenue", "lo_custkey", "lo_supplycost")
AMERICA, ASIA, EUROPE = 1, 2, 3
UNITED_STATES, UKI1, UKI5 = 24, 231, 235
I32MIN, I32MAX = -(2**31), 2**31 - 1
DATE_MIN, DATE_MAX = 19920101, 19981231


def brand_index(brand1):
    """p_brand1 = 100*(10m + c) + k  ->  dense 0..999 (dictionary code)."""
    b = np.asarray(brand1)
    cat, k = b // 100, b % 100
    return ((cat // 10 - 1) * 200 + (cat % 10 - 1) * 40 + (k - 1)).astype(np.int32)


def brand_from_index(i):
    m, rem = divmod(int(i), 200)
    c, k = divmod(rem, 40)
    return 100 * (10 * (m + 1) + (c + 1)) + (k + 1)


def category_index(cat):
    c = np.asarray(cat)
    return ((c // 10 - 1) * 5 + (c % 10 - 1)).astype(np.int32)


def category_from_index(i):
    m, c = divmod(int(i), 5)
    return 10 * (m + 1) + (c + 1)


class SSBEngine:
    """Dimension tables + GPU-*-encoded lineorder columns on one device.

    rows: optional (lo, hi) range of lineorder rows (512-row aligned lo) for tile-range
    sharding across GPUs; dimensions are replicated.
    """

    def __init__(self, db: dict, device=None, schemes: dict | None = None, rows: tuple | None = None):
        import torch
        self.torch = torch
        self.device = device if device is not None else torch.device("cuda", torch.cuda.current_device())
        dev = lambda a: torch.from_numpy(np.ascontiguousarray(a, np.int32)).to(self.device)  # noqa: E731
        d, c, s, p = db["date"], db["customer"], db["supplier"], db["part"]
        self.date_keys = np.asarray(d["d_datekey"])
        self._dd = {k: np.asarray(d[k]) for k in ("d_year", "d_yearmonthnum", "d_yearmonth", "d_weeknuminyear")}
        self.dims = {
            "date": {"keys": dev(d["d_datekey"]), "key_min": DATE_MIN, "len": DATE_MAX - DATE_MIN + 1,
                     "d_year": dev(d["d_year"]), "d_yearmonthnum": dev(d["d_yearmonthnum"]),
                     "d_yearmonth": dev(d["d_yearmonth"]), "year_idx": dev(np.asarray(d["d_year"]) - 1992)},
            "customer": {"keys": dev(c["c_custkey"]), "key_min": 1, "len": len(c["c_custkey"]),
                         "c_region": dev(c["c_region"]), "c_nation": dev(c["c_nation"]), "c_city": dev(c["c_city"])},
            "supplier": {"keys": dev(s["s_suppkey"]), "key_min": 1, "len": len(s["s_suppkey"]),
                         "s_region": dev(s["s_region"]), "s_nation": dev(s["s_nation"]), "s_city": dev(s["s_city"])},
            "part": {"keys": dev(p["p_partkey"]), "key_min": 1, "len": len(p["p_partkey"]),
                     "p_mfgr": dev(p["p_mfgr"]), "p_category": dev(p["p_category"]), "p_brand1": dev(p["p_brand1"]),
                     "brand_idx": dev(brand_index(p["p_brand1"])), "cat_idx": dev(category_index(p["p_category"]))},
        }
        lo = db["lineorder"]
        r0, r1 = rows if rows is not None else (0, len(lo["lo_orderdate"]))
        self.rows = (r0, r1)
        self.n = r1 - r0
        self.host = {}
        self.cols = {}
        for name in QUERY_COLUMNS:
            x = np.ascontiguousarray(lo[name][r0:r1], np.int32)
            scheme = (schemes or {}).get(name, "auto")
            h = tp.encode(x, scheme)
            self.host[name] = h
            self.cols[name] = h.to_device(self.device)
        self.tables = {}

    def footprint(self) -> dict:
        return {k: (h.scheme, h.nbytes()) for k, h in self.host.items()}

    # ------------------------------------------------------------ plans
    def _date_range(self, mask) -> tuple:
        """lo_orderdate key range of the date rows selected by `mask` (must be contiguous)."""
        keys = self.date_keys[np.asarray(mask)]
        first, last = int(keys.min()), int(keys.max())
        span = np.flatnonzero((self.date_keys >= first) & (self.date_keys <= last))
        assert len(span) == len(keys), "date predicate is not a contiguous key range"
        return first, last

    def _table(self, dim: str, preds: list, payload: str | None):
        D = self.dims[dim]
        t = self.torch.empty(D["len"], dtype=self.torch.int32, device=self.device)
        tp.tp_lookup_build(D["keys"], len(D["keys"]), D["key_min"], D["len"],
                           [(D[a], *rng) for a, rng in preds], D[payload] if payload else None, t)
        return t, D["key_min"], D["len"]

    def plan(self, qid: str) -> dict:
        """columns in evaluation order with their roles, aggregate, group layout and decoder."""
        d = np.asarray
        date = self.date_keys
        if qid.startswith("1."):
            dd = self._dates()
            if qid == "1.1":
                r = self._date_range(dd["d_year"] == 1993)
                q, dl = (I32MIN, 24), (1, 3)
            elif qid == "1.2":
                r = self._date_range(dd["d_yearmonthnum"] == 199401)
                q, dl = (26, 35), (4, 6)
            else:
                r = self._date_range((dd["d_weeknuminyear"] == 6) & (dd["d_year"] == 1994))
                q, dl = (26, 35), (5, 7)
            # most selective first: the date range (RFOR, decoded whole), then the discount
            # (the staged first measure with its filter), the quantity, the price
            cols = [("lo_orderdate", "range", r), ("lo_discount", "measure", dl),
                    ("lo_quantity", "range", q), ("lo_extendedprice", "measure", None)]
            return {"cols": cols, "agg": "mul", "radix": [], "decode": lambda g: ()}
        year_all = ("date", [("d_year", (1992, 1998))], "year_idx")
        if qid.startswith("2."):
            part_pred = {"2.1": [("p_category", (12, 12))], "2.2": [("p_brand1", (2221, 2228))],
                         "2.3": [("p_brand1", (2239, 2239))]}[qid]
            region = {"2.1": AMERICA, "2.2": ASIA, "2.3": EUROPE}[qid]
            cols = [("lo_partkey", "probe", ("part", part_pred, "brand_idx"), 1),
                    ("lo_suppkey", "probe", ("supplier", [("s_region", (region, region))], None), 0),
                    ("lo_orderdate", "probe", year_all, 1000),
                    ("lo_revenue", "measure", None)]
            return {"cols": cols, "agg": "sum", "radix": [7, 1000],
                    "decode": lambda g: (1992 + g // 1000, brand_from_index(g % 1000))}
        if qid.startswith("3."):
            years = ("date", [("d_year", (1992, 1997))], "year_idx")
            if qid == "3.1":
                c = ("customer", [("c_region", (ASIA, ASIA))], "c_nation")
                s = ("supplier", [("s_region", (ASIA, ASIA))], "s_nation")
                rad = 25
            elif qid == "3.2":
                c = ("customer", [("c_nation", (UNITED_STATES, UNITED_STATES))], "c_city")
                s = ("supplier", [("s_nation", (UNITED_STATES, UNITED_STATES))], "s_city")
                rad = 250
            else:
                c = ("customer", [("c_city", (UKI1, UKI1, UKI5, UKI5))], "c_city")
                s = ("supplier", [("s_city", (UKI1, UKI1, UKI5, UKI5))], "s_city")
                rad = 250
                if qid == "3.4":
                    years = ("date", [("d_yearmonth", (199712, 199712))], "year_idx")
            cols = [("lo_custkey", "probe", c, rad * 7), ("lo_suppkey", "probe", s, 7),
                    ("lo_orderdate", "probe", years, 1), ("lo_revenue", "measure", None)]
            return {"cols": cols, "agg": "sum", "radix": [rad, rad, 7],
                    "decode": lambda g, rad=rad: (g // (rad * 7), (g // 7) % rad, 1992 + g % 7),
                    "order": "q3"}
        # flight 4: profit = revenue - supplycost
        y9798 = ("date", [("d_year", (1997, 1998))], "year_idx")
        mfgr12 = ("part", [("p_mfgr", (1, 2))], None)
        if qid == "4.1":
            cols = [("lo_custkey", "probe", ("customer", [("c_region", (AMERICA, AMERICA))], "c_nation"), 1),
                    ("lo_suppkey", "probe", ("supplier", [("s_region", (AMERICA, AMERICA))], None), 0),
                    ("lo_partkey", "probe", mfgr12, 0),
                    ("lo_orderdate", "probe", year_all, 25)]
            radix, dec = [7, 25], (lambda g: (1992 + g // 25, g % 25))
        elif qid == "4.2":
            cols = [("lo_custkey", "probe", ("customer", [("c_region", (AMERICA, AMERICA))], None), 0),
                    ("lo_suppkey", "probe", ("supplier", [("s_region", (AMERICA, AMERICA))], "s_nation"), 25),
                    ("lo_partkey", "probe", ("part", [("p_mfgr", (1, 2))], "cat_idx"), 1),
                    ("lo_orderdate", "probe", y9798, 625)]
            radix = [7, 25, 25]
            dec = lambda g: (1992 + g // 625, (g // 25) % 25, category_from_index(g % 25))  # noqa: E731
        else:
            cols = [("lo_suppkey", "probe", ("supplier", [("s_nation", (UNITED_STATES, UNITED_STATES))], "s_city"),
                     1000),
                    ("lo_partkey", "probe", ("part", [("p_category", (14, 14))], "brand_idx"), 1),
                    ("lo_custkey", "probe", ("customer", [("c_region", (AMERICA, AMERICA))], None), 0),
                    ("lo_orderdate", "probe", y9798, 250_000)]
            radix = [7, 250, 1000]
            dec = lambda g: (1992 + g // 250_000, (g // 1000) % 250, brand_from_index(g % 1000))  # noqa: E731
        cols = cols + [("lo_revenue", "measure", None), ("lo_supplycost", "measure", None)]
        return {"cols": cols, "agg": "sub", "radix": radix, "decode": dec}

    def _dates(self):
        return self._dd

    def prepare(self, qid: str) -> dict:
        """Build the query's lookup tables (GPU) and marshal its column roles."""
        pl = self.plan(qid)
        dcols, roles, keep = [], [], []
        for spec in pl["cols"]:
            name, role = spec[0], spec[1]
            r = tp.tp_star_col()
            if role == "range":
                r.role, (r.lo, r.hi) = tp.TP_ROLE_RANGE, spec[2]
            elif role == "measure":
                r.role = tp.TP_ROLE_MEASURE
                r.lo, r.hi = spec[2] if spec[2] else (I32MIN, I32MAX)
            else:
                dim, preds, payload = spec[2]
                preds2 = [(a, rng if len(rng) == 4 else (rng[0], rng[1], 1, 0)) for a, rng in preds]
                t, kmin, tlen = self._table(dim, preds2, payload)
                keep.append(t)
                r.role, r.table, r.key_min, r.table_len, r.stride = tp.TP_ROLE_PROBE, t.data_ptr(), kmin, tlen, spec[3]
            dcols.append(self.cols[name].col)
            roles.append(r)
        ngroups = int(np.prod(pl["radix"])) if pl["radix"] else 1
        return {"plan": pl, "dcols": dcols, "roles": roles, "tables": keep, "ngroups": ngroups}

    def execute(self, prep: dict, sums=None, counts=None, stream=None):
        torch = self.torch
        G = prep["ngroups"]
        if sums is None:
            sums = torch.zeros(G, dtype=torch.int64, device=self.device)
            counts = torch.zeros(G, dtype=torch.int64, device=self.device)
        tp.tp_star_query(prep["dcols"], prep["roles"], tp.TP_AGG[prep["plan"]["agg"]], sums, counts, G, stream)
        return sums, counts

    def run(self, qid: str):
        prep = self.prepare(qid)
        sums, counts = self.execute(prep)
        return self.result(qid, prep, sums, counts)

    @staticmethod
    def result(qid: str, prep: dict, sums, counts) -> list:
        """non-empty groups -> tuples in SELECT order, sorted per the query's ORDER BY."""
        s = sums.cpu().numpy()
        c = counts.cpu().numpy()
        pl = prep["plan"]
        if not pl["radix"]:
            return [(int(s[0]),)]
        rows = [(*pl["decode"](int(g)), int(s[g])) for g in np.flatnonzero(c)]
        if pl.get("order") == "q3":
            return sorted(rows, key=lambda r: (r[2], -r[3], r[0], r[1]))
        return sorted(rows)
