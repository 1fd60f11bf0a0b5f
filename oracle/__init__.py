"""TEST INFRASTRUCTURE ONLY -- the CPU oracle for the GPU-FOR / GPU-DFOR / GPU-RFOR
formats of Shanbhag et al., SIGMOD '22 (/root/reference/PAPER.md, ``P:<line>``).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  It shares no code with the
product package ``paper_conf_sigmod_shanbhagyym22_b200`` and imports nothing from it.

The arithmetic lives in ``oracle.c`` (plain scalar C, one entry at a time, written
in the paper's order); this module only marshals numpy arrays through ctypes.
``ssb.py`` holds the SSB query semantics (plain SQL over uncompressed columns).
"""
from __future__ import annotations

import ctypes
import hashlib
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
GUARD_WORDS = 4  # [R9]: Alg. 1 line 15 reads data[s+1]; zero words after every data array

_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c with plain gcc (no intrinsics, -O2)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-fPIC", "-shared", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        u64, i64, i32, u32 = ctypes.c_uint64, ctypes.c_int64, ctypes.c_int32, ctypes.c_uint32
        vp = ctypes.c_void_p
        L.orc_for_size.restype = u64
        L.orc_for_size.argtypes = [vp, u64, u32, u32]
        L.orc_for_encode.argtypes = [vp, u64, u32, u32, vp, vp, vp]
        L.orc_for_decode.argtypes = [vp, vp, vp, vp]
        L.orc_for_decode_range.argtypes = [vp, vp, vp, u64, u64, vp]
        L.orc_dfor_size.restype = u64
        L.orc_dfor_size.argtypes = [vp, u64]
        L.orc_dfor_encode.argtypes = [vp, u64, vp, vp, vp]
        L.orc_dfor_decode.argtypes = [vp, vp, vp, vp]
        L.orc_rfor_size.argtypes = [vp, u64, vp, vp]
        L.orc_rfor_encode.argtypes = [vp, u64, vp, vp, vp, vp, vp]
        L.orc_rfor_decode.argtypes = [vp, vp, vp, vp, vp, vp]
        L.orc_select_project_sum.restype = i64
        L.orc_select_project_sum.argtypes = [vp, ctypes.c_int, vp, vp, u64, ctypes.c_int, ctypes.c_int, ctypes.c_int]
        L.orc_sum.restype = i64
        L.orc_sum.argtypes = [vp, u64]
        for f in ("orc_for_encode", "orc_for_decode", "orc_for_decode_range", "orc_dfor_encode",
                  "orc_dfor_decode", "orc_rfor_size", "orc_rfor_encode", "orc_rfor_decode"):
            getattr(L, f).restype = ctypes.c_int
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _col(x) -> np.ndarray:
    x = np.ascontiguousarray(x, dtype=np.int32)
    return x


def _check(rc: int, what: str):
    if rc != 0:
        raise ValueError(f"oracle {what} failed with status {rc}")


class Encoded(dict):
    """scheme, header (3 u32), arrays without guard words; ``guarded(name)`` adds them."""

    def guarded(self, name: str) -> np.ndarray:
        a = self[name]
        return np.concatenate([a, np.zeros(GUARD_WORDS, np.uint32)])

    def nbytes(self) -> int:
        """Compressed size: header + block_starts + data."""
        if self["scheme"] == "rfor":
            return 4 * (3 + len(self["startsV"]) + len(self["dataV"]) + len(self["startsL"]) + len(self["dataL"]))
        return 4 * (3 + len(self["starts"]) + len(self["data"]))

    def serialize(self) -> bytes:
        """header || starts || data (FOR/DFOR); header || startsV || dataV || startsL || dataL (RFOR)."""
        if self["scheme"] == "rfor":
            parts = [self["header"], self["startsV"], self["dataV"], self["startsL"], self["dataL"]]
        else:
            parts = [self["header"], self["starts"], self["data"]]
        return b"".join(np.ascontiguousarray(p, dtype="<u4").tobytes() for p in parts)

    def digest(self) -> str:
        return hashlib.sha256(self.serialize()).hexdigest()[:16]


# ---------------------------------------------------------------- GPU-FOR
def for_encode(x, block_size: int = 128, mb_count: int = 4) -> Encoded:
    """GPU-FOR encoding, P:614-711 (defaults 128-entry blocks, 4 miniblocks of 32)."""
    x = _col(x)
    n = len(x)
    L = lib()
    words = L.orc_for_size(_p(x), n, block_size, mb_count)
    nb = (n + block_size - 1) // block_size
    header = np.zeros(3, np.uint32)
    starts = np.zeros(nb + 1, np.uint32)
    data = np.zeros(words + GUARD_WORDS, np.uint32)
    _check(L.orc_for_encode(_p(x), n, block_size, mb_count, _p(header), _p(starts), _p(data)), "for_encode")
    return Encoded(scheme="for", header=header, starts=starts, data=data[:words])


def for_decode(enc: Encoded) -> np.ndarray:
    """Algorithm 1, one entry at a time."""
    n = int(enc["header"][2])
    out = np.zeros(n, np.int32)
    data = enc.guarded("data")
    _check(lib().orc_for_decode(_p(enc["header"]), _p(enc["starts"]), _p(data), _p(out)), "for_decode")
    return out


def for_decode_range(enc: Encoded, lo: int, hi: int, data_guarded: np.ndarray | None = None) -> np.ndarray:
    out = np.zeros(hi - lo, np.int32)
    data = enc.guarded("data") if data_guarded is None else data_guarded
    _check(lib().orc_for_decode_range(_p(enc["header"]), _p(enc["starts"]), _p(data), lo, hi, _p(out)),
           "for_decode_range")
    return out


# ---------------------------------------------------------------- GPU-DFOR
def dfor_encode(x) -> Encoded:
    """GPU-DFOR encoding, P:1060-1083 (D = 4 blocks of 128 per tile)."""
    x = _col(x)
    n = len(x)
    L = lib()
    words = L.orc_dfor_size(_p(x), n)
    nb = (n + 127) // 128
    header = np.zeros(3, np.uint32)
    starts = np.zeros(nb + 1, np.uint32)
    data = np.zeros(words + GUARD_WORDS, np.uint32)
    _check(L.orc_dfor_encode(_p(x), n, _p(header), _p(starts), _p(data)), "dfor_encode")
    return Encoded(scheme="dfor", header=header, starts=starts, data=data[:words])


def dfor_decode(enc: Encoded) -> np.ndarray:
    """Algorithm-1 unpack of the deltas, then the in-tile prefix sum."""
    n = int(enc["header"][2])
    out = np.zeros(n, np.int32)
    data = enc.guarded("data")
    _check(lib().orc_dfor_decode(_p(enc["header"]), _p(enc["starts"]), _p(data), _p(out)), "dfor_decode")
    return out


# ---------------------------------------------------------------- GPU-RFOR
def rfor_encode(x) -> Encoded:
    """GPU-RFOR encoding, P:1128-1137 (layout B, reading R17)."""
    x = _col(x)
    n = len(x)
    L = lib()
    wv = np.zeros(1, np.uint64)
    wl = np.zeros(1, np.uint64)
    _check(L.orc_rfor_size(_p(x), n, _p(wv), _p(wl)), "rfor_size")
    wv, wl = int(wv[0]), int(wl[0])
    nrb = (n + 511) // 512
    header = np.zeros(3, np.uint32)
    sV = np.zeros(nrb + 1, np.uint32)
    sL = np.zeros(nrb + 1, np.uint32)
    dV = np.zeros(wv + GUARD_WORDS, np.uint32)
    dL = np.zeros(wl + GUARD_WORDS, np.uint32)
    _check(L.orc_rfor_encode(_p(x), n, _p(header), _p(sV), _p(dV), _p(sL), _p(dL)), "rfor_encode")
    return Encoded(scheme="rfor", header=header, startsV=sV, dataV=dV[:wv], startsL=sL, dataL=dL[:wl])


def rfor_decode(enc: Encoded) -> np.ndarray:
    """unpack values and run lengths, expand the runs."""
    n = int(enc["header"][2])
    out = np.zeros(n, np.int32)
    dV = enc.guarded("dataV")
    dL = enc.guarded("dataL")
    _check(lib().orc_rfor_decode(_p(enc["header"]), _p(enc["startsV"]), _p(dV), _p(enc["startsL"]), _p(dL),
                                 _p(out)), "rfor_decode")
    return out


ENCODERS = {"for": for_encode, "dfor": dfor_encode, "rfor": rfor_encode,
            # GPU-FOR without miniblocks: one 128-entry miniblock per block
            "fornm": lambda x: for_encode(x, 128, 1)}
DECODERS = {"for": for_decode, "dfor": dfor_decode, "rfor": rfor_decode}


def encode(scheme: str, x) -> Encoded:
    return ENCODERS[scheme](x)


def decode(enc: Encoded) -> np.ndarray:
    return DECODERS[enc["scheme"]](enc)


def choose_scheme(x) -> tuple[str, Encoded]:
    """GPU-* (P:1206-1217): the scheme with the lowest storage footprint;
    ties -> FOR < DFOR < RFOR (reading R20)."""
    best = None
    for s in ("for", "dfor", "rfor"):
        e = encode(s, x)
        if best is None or e.nbytes() < best[1].nbytes():
            best = (s, e)
    return best


# ---------------------------------------------------------------- queries
PROJ = {"col": 0, "mul": 1, "sub": 2, "count": 3}


def select_project_sum(cols, lo, hi, proj: str = "col", a: int = 0, b: int = 0) -> int:
    """sum over rows passing every inclusive range predicate of proj(row), int64."""
    cols = [_col(c) for c in cols]
    n = len(cols[0]) if cols else 0
    ptrs = (ctypes.c_void_p * max(1, len(cols)))(*[c.ctypes.data for c in cols])
    lo = np.ascontiguousarray(lo, np.int32)
    hi = np.ascontiguousarray(hi, np.int32)
    return int(lib().orc_select_project_sum(ptrs, len(cols), _p(lo), _p(hi), n, PROJ[proj], a, b))


def bitmap_sum(x, bitmap) -> int:
    """Random access under a predicate bitvector, by its plain definition:
    the int64 sum of x[i] over rows i whose bit is set (bit i = bit i % 32 of word i // 32)."""
    x = _col(x)
    n = len(x)
    bits = np.unpackbits(np.ascontiguousarray(bitmap, np.uint32).view(np.uint8), bitorder="little")[:n]
    return int(x[bits.astype(bool)].astype(np.int64).sum())


def column_sum(x) -> int:
    x = _col(x)
    return int(lib().orc_sum(_p(x), len(x)))


def star_query(cols, roles, agg: str, ngroups: int):
    """One star-join pass by its plain definition (include/tilepack.h tp_star_query; SSB
    star joins P:1874-1888): rows survive every RANGE (lo <= v <= hi), every PROBE
    (p = table[v - key_min] >= 0, group += p * stride) and every MEASURE's own range;
    the last column is the aggregating measure m_last, an earlier measure is m_first;
    aggregate = m_last (sum) | m_first * m_last (mul) | m_first - m_last (sub), int64.
    roles: dicts {role: "range"|"probe"|"measure", lo, hi, table (np int32), key_min, stride}.
    Returns (sums[ngroups] int64, counts[ngroups] int64).  Plain numpy, row-parallel."""
    cols = [np.asarray(c, np.int64) for c in cols]
    n = len(cols[0])
    alive = np.ones(n, bool)
    group = np.zeros(n, np.int64)
    meas = []
    for x, r in zip(cols, roles):
        if r["role"] == "probe":
            t = np.asarray(r["table"], np.int64)
            k = x - r["key_min"]
            inside = (k >= 0) & (k < len(t))
            p = np.full(n, -1, np.int64)
            p[inside] = t[k[inside]]
            alive &= p >= 0
            group += np.where(p >= 0, p, 0) * r.get("stride", 0)
        else:
            alive &= (x >= r["lo"]) & (x <= r["hi"])
            if r["role"] == "measure":
                meas.append(x)
    if agg == "sum":
        y = meas[-1]
    elif agg == "mul":
        y = meas[0] * meas[1]
    else:
        y = meas[0] - meas[1]
    g = group[alive] if ngroups > 1 else np.zeros(int(alive.sum()), np.int64)
    sums = np.zeros(ngroups, np.int64)
    np.add.at(sums, g, y[alive])
    counts = np.bincount(g, minlength=ngroups).astype(np.int64)
    return sums, counts
