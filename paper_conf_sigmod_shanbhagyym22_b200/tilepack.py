"""Thin ctypes binding of the tilepack C ABI (include/tilepack.h).

Argument marshalling only: every step of encode/decode/query runs in the native
library (host encoder in C++, decoders and fused operators as sm_100a CUDA
kernels).  PyTorch provides device memory and streams.  There is no CPU or
Python fallback: if ``libtilepack.so`` is missing this module raises at import.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("TILEPACK_LIB_OVERRIDE") or os.path.join(_HERE, "libtilepack.so")  # override: A/B builds
GUARD_WORDS = 4

TP_FOR, TP_DFOR, TP_RFOR, TP_NONE, TP_FORNM = 1, 2, 3, 4, 5
# "fornm": GPU-FOR without miniblocks, the miniblock ablation (decode / decode_sum only)
SCHEMES = {"for": TP_FOR, "dfor": TP_DFOR, "rfor": TP_RFOR, "none": TP_NONE, "fornm": TP_FORNM}
SCHEME_NAMES = {v: k for k, v in SCHEMES.items()}
TP_PROJ = {"col": 0, "mul": 1, "sub": 2, "count": 3}
TP_MAX_COLS = 6


class TilepackError(RuntimeError):
    pass


class tp_column(ctypes.Structure):
    _fields_ = [
        ("scheme", ctypes.c_uint32),
        ("block_size", ctypes.c_uint32),
        ("miniblock_count", ctypes.c_uint32),
        ("tile_blocks", ctypes.c_uint32),
        ("n", ctypes.c_uint64),
        ("num_blocks", ctypes.c_uint64),
        ("starts0", ctypes.c_void_p),
        ("data0", ctypes.c_void_p),
        ("words0", ctypes.c_uint64),
        ("starts1", ctypes.c_void_p),
        ("data1", ctypes.c_void_p),
        ("words1", ctypes.c_uint64),
        ("max_tile_words0", ctypes.c_uint32),
        ("max_tile_words1", ctypes.c_uint32),
    ]


class tp_dim_pred(ctypes.Structure):
    _fields_ = [("attr", ctypes.c_void_p), ("lo1", ctypes.c_int32), ("hi1", ctypes.c_int32),
                ("lo2", ctypes.c_int32), ("hi2", ctypes.c_int32)]


class tp_star_col(ctypes.Structure):
    _fields_ = [("role", ctypes.c_int32), ("lo", ctypes.c_int32), ("hi", ctypes.c_int32),
                ("table", ctypes.c_void_p), ("key_min", ctypes.c_int32), ("table_len", ctypes.c_uint32),
                ("stride", ctypes.c_uint32)]


TP_ROLE_RANGE, TP_ROLE_PROBE, TP_ROLE_MEASURE = 0, 1, 2
TP_AGG = {"sum": 0, "mul": 1, "sub": 2}


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(
            f"tilepack native library not built: {LIB_PATH} is missing "
            "(run `python -c 'import __graft_entry__ as g; g.build()'`)")
    L = ctypes.CDLL(LIB_PATH)
    vp, u64, i32, u32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_uint32
    colp = ctypes.POINTER(tp_column)
    sig = {
        "tp_encode_size": (i32, [i32, vp, u64, vp, vp, vp]),
        "tp_encode": (i32, [i32, vp, u64, vp, vp, vp, vp, colp]),
        "tp_choose_scheme": (i32, [vp, u64, vp, vp]),
        "tp_compressed_bytes": (u64, [colp]),
        "tp_shard": (i32, [colp, u64, u64, vp, vp, colp]),
        "tp_validate": (i32, [colp, vp, vp]),
        "tp_device_errors": (i32, [vp, vp]),
        "tp_decode": (i32, [colp, vp, vp]),
        "tp_decode_sum": (i32, [colp, vp, vp]),
        "tp_select_project_sum": (i32, [colp, i32, vp, vp, i32, i32, i32, vp, vp]),
        "tp_plain_sum": (i32, [vp, u64, vp, vp]),
        "tp_bitmap_sum": (i32, [colp, vp, vp, vp]),
        "tp_cascaded_workspace_words": (u64, [colp]),
        "tp_decode_cascaded": (i32, [colp, vp, vp, vp]),
        "tp_lookup_build": (i32, [vp, u64, ctypes.c_int32, u32, ctypes.POINTER(tp_dim_pred), i32, vp, vp, vp]),
        "tp_star_query": (i32, [colp, ctypes.POINTER(tp_star_col), i32, i32, vp, vp, u32, vp]),
        "tp_gpu_encode_workspace_bytes": (u64, [u64]),
        "tp_gpu_encode_bound": (i32, [i32, u64, vp, vp, vp]),
        "tp_gpu_encode_sizes": (i32, [vp, u64, vp, vp, vp]),
        "tp_gpu_choose_scheme": (i32, [vp, u64, vp, vp, vp, vp]),
        "tp_gpu_encode_launch": (i32, [i32, vp, u64, vp, vp, u64, vp, vp, u64, vp, vp]),
        "tp_gpu_encode_result": (i32, [i32, u64, vp, vp, vp, vp, vp, colp, vp]),
        "tp_gpu_encode": (i32, [i32, vp, u64, vp, vp, u64, vp, vp, u64, vp, colp, vp]),
        "tp_bench_int_roof": (i32, [i32, u32, vp, vp, vp]),
        "tp_status_string": (ctypes.c_char_p, [i32]),
        "tp_launch_count": (u64, []),
        "tp_debug_counters": (i32, [vp]),
        "tp_device_info": (i32, [vp, vp]),
    }
    for name, (res, args) in sig.items():
        if os.environ.get("TILEPACK_LIB_OVERRIDE") and not hasattr(L, name):
            continue  # A/B experiments with older builds
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    return L


_lib = _load()


def lib():
    return _lib


def _check(rc: int, what: str):
    if rc != 0:
        raise TilepackError(f"{what}: {_lib.tp_status_string(rc).decode()} (status {rc})")


def _ptr(a) -> int | None:
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        return a.ctypes.data
    return a.data_ptr()  # torch tensor


def _stream(stream=None):
    import torch
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


# ------------------------------------------------------------------ C ABI, same names
def tp_encode_size(scheme: int, x: np.ndarray):
    nb, w0, w1 = ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_uint64()
    _check(_lib.tp_encode_size(scheme, _ptr(x), len(x), ctypes.byref(nb), ctypes.byref(w0), ctypes.byref(w1)),
           "tp_encode_size")
    return nb.value, w0.value, w1.value


def tp_encode(scheme: int, x: np.ndarray, starts0, data0, starts1=None, data1=None) -> tp_column:
    col = tp_column()
    _check(_lib.tp_encode(scheme, _ptr(x), len(x), _ptr(starts0), _ptr(data0), _ptr(starts1), _ptr(data1),
                          ctypes.byref(col)), "tp_encode")
    return col


def tp_choose_scheme(x: np.ndarray):
    s, b = ctypes.c_int(), ctypes.c_uint64()
    _check(_lib.tp_choose_scheme(_ptr(x), len(x), ctypes.byref(s), ctypes.byref(b)), "tp_choose_scheme")
    return s.value, b.value


def tp_compressed_bytes(col: tp_column) -> int:
    return int(_lib.tp_compressed_bytes(ctypes.byref(col)))


def tp_shard(col: tp_column, row_lo: int, row_hi: int, rebased0, rebased1=None) -> tp_column:
    view = tp_column()
    _check(_lib.tp_shard(ctypes.byref(col), row_lo, row_hi, _ptr(rebased0), _ptr(rebased1), ctypes.byref(view)),
           "tp_shard")
    return view


def tp_validate(col: tp_column):
    """Format check of a HOST column; returns (max_tile_words0, max_tile_words1)."""
    m0, m1 = ctypes.c_uint32(), ctypes.c_uint32()
    _check(_lib.tp_validate(ctypes.byref(col), ctypes.byref(m0), ctypes.byref(m1)), "tp_validate")
    return m0.value, m1.value


TP_DEVERR_TILE_WORDS, TP_DEVERR_RUNS = 2, 4


def tp_device_errors(stream=None) -> int:
    """Format-violation flags seen by the device calls since the last read (cleared); syncs."""
    f = ctypes.c_uint32()
    _check(_lib.tp_device_errors(ctypes.byref(f), _stream(stream)), "tp_device_errors")
    return f.value


def tp_decode(dcol: tp_column, d_out, stream=None):
    _check(_lib.tp_decode(ctypes.byref(dcol), _ptr(d_out), _stream(stream)), "tp_decode")


def tp_decode_sum(dcol: tp_column, d_sum, stream=None):
    _check(_lib.tp_decode_sum(ctypes.byref(dcol), _ptr(d_sum), _stream(stream)), "tp_decode_sum")


def tp_select_project_sum(dcols, lo, hi, proj_op: int, a: int, b: int, d_result, stream=None):
    n = len(dcols)
    arr = (tp_column * n)(*dcols)
    lo = np.ascontiguousarray(lo, np.int32)
    hi = np.ascontiguousarray(hi, np.int32)
    _check(_lib.tp_select_project_sum(arr, n, _ptr(lo), _ptr(hi), proj_op, a, b, _ptr(d_result), _stream(stream)),
           "tp_select_project_sum")


def tp_lookup_build(d_keys, nrows: int, key_min: int, table_len: int, preds, d_payload, d_table, stream=None):
    """preds: list of (attr_tensor, lo1, hi1[, lo2, hi2])"""
    arr = (tp_dim_pred * max(1, len(preds)))()
    for i, p in enumerate(preds):
        lo2, hi2 = (p[3], p[4]) if len(p) > 3 else (1, 0)
        arr[i] = tp_dim_pred(_ptr(p[0]), p[1], p[2], lo2, hi2)
    _check(_lib.tp_lookup_build(_ptr(d_keys), nrows, key_min, table_len, arr, len(preds), _ptr(d_payload),
                                _ptr(d_table), _stream(stream)), "tp_lookup_build")


def tp_star_query(dcols, roles, agg: int, d_sums, d_counts, ngroups: int, stream=None):
    n = len(dcols)
    carr = (tp_column * n)(*dcols)
    rarr = (tp_star_col * n)(*roles)
    _check(_lib.tp_star_query(carr, rarr, n, agg, _ptr(d_sums), _ptr(d_counts), ngroups, _stream(stream)),
           "tp_star_query")


def tp_cascaded_workspace_words(col: tp_column) -> int:
    return int(_lib.tp_cascaded_workspace_words(ctypes.byref(col)))


def tp_decode_cascaded(dcol: tp_column, d_out, d_work, stream=None):
    _check(_lib.tp_decode_cascaded(ctypes.byref(dcol), _ptr(d_out), _ptr(d_work), _stream(stream)),
           "tp_decode_cascaded")


def decode_cascaded(dcol: "DeviceColumn", out=None, work=None, stream=None):
    """The cascading-decompression baseline (one kernel per layer)."""
    import torch
    dev = dcol.data0.device
    if out is None:
        out = torch.empty(dcol.n, dtype=torch.int32, device=dev)
    if work is None:
        work = torch.empty(max(1, tp_cascaded_workspace_words(dcol.col)), dtype=torch.int32, device=dev)
    tp_decode_cascaded(dcol.col, out, work, stream)
    return out


# ---- GPU encoder (tile-parallel, one pass; include/tilepack.h "GPU encoder")
def tp_gpu_encode_workspace_bytes(n: int) -> int:
    return int(_lib.tp_gpu_encode_workspace_bytes(n))


def tp_gpu_encode_bound(scheme: int, n: int):
    nb, w0, w1 = ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_uint64()
    _check(_lib.tp_gpu_encode_bound(scheme, n, ctypes.byref(nb), ctypes.byref(w0), ctypes.byref(w1)),
           "tp_gpu_encode_bound")
    return nb.value, w0.value, w1.value


def tp_gpu_encode_sizes(d_x, n: int, d_work, stream=None):
    w = (ctypes.c_uint64 * 4)()
    _check(_lib.tp_gpu_encode_sizes(_ptr(d_x), n, _ptr(d_work), w, _stream(stream)), "tp_gpu_encode_sizes")
    return [int(v) for v in w]


def tp_gpu_choose_scheme(d_x, n: int, d_work, stream=None):
    s, b = ctypes.c_int(), ctypes.c_uint64()
    _check(_lib.tp_gpu_choose_scheme(_ptr(d_x), n, _ptr(d_work), ctypes.byref(s), ctypes.byref(b), _stream(stream)),
           "tp_gpu_choose_scheme")
    return s.value, b.value


def tp_gpu_encode_launch(scheme: int, d_x, n: int, starts0, data0, cap0: int, starts1, data1, cap1: int, d_work,
                         stream=None):
    _check(_lib.tp_gpu_encode_launch(scheme, _ptr(d_x), n, _ptr(starts0), _ptr(data0), cap0, _ptr(starts1),
                                     _ptr(data1), cap1, _ptr(d_work), _stream(stream)), "tp_gpu_encode_launch")


def tp_gpu_encode_result(scheme: int, n: int, starts0, data0, starts1, data1, d_work, stream=None) -> tp_column:
    col = tp_column()
    _check(_lib.tp_gpu_encode_result(scheme, n, _ptr(starts0), _ptr(data0), _ptr(starts1), _ptr(data1),
                                     _ptr(d_work), ctypes.byref(col), _stream(stream)), "tp_gpu_encode_result")
    return col


def tp_gpu_encode(scheme: int, d_x, n: int, starts0, data0, cap0: int, starts1, data1, cap1: int, d_work,
                  stream=None) -> tp_column:
    col = tp_column()
    _check(_lib.tp_gpu_encode(scheme, _ptr(d_x), n, _ptr(starts0), _ptr(data0), cap0, _ptr(starts1), _ptr(data1),
                              cap1, _ptr(d_work), ctypes.byref(col), _stream(stream)), "tp_gpu_encode")
    return col


def tp_bitmap_sum(dcol: tp_column, d_bitmap, d_sum, stream=None):
    _check(_lib.tp_bitmap_sum(ctypes.byref(dcol), _ptr(d_bitmap), _ptr(d_sum), _stream(stream)), "tp_bitmap_sum")


def bitmap_sum(dcol, d_bitmap, out=None, stream=None):
    """Random access: sum of the rows selected by a device bitvector."""
    import torch
    if out is None:
        out = torch.zeros(1, dtype=torch.int64, device=dcol.data0.device)
    tp_bitmap_sum(dcol.col, d_bitmap, out, stream)
    return out


def tp_plain_sum(d_x, n: int, d_sum, stream=None):
    _check(_lib.tp_plain_sum(_ptr(d_x), n, _ptr(d_sum), _stream(stream)), "tp_plain_sum")


def tp_bench_int_roof(kind: int, iters: int, d_sink, stream=None) -> int:
    """Launch the INT32 issue-roof microbenchmark; returns the warp instructions it executes."""
    w = ctypes.c_uint64()
    _check(_lib.tp_bench_int_roof(kind, iters, _ptr(d_sink), ctypes.byref(w), _stream(stream)), "tp_bench_int_roof")
    return w.value


INT_ROOF_KINDS = {0: "SHF", 1: "LOP3", 2: "IADD3", 3: "IMAD", 4: "SHF+LOP3+IADD3 (ALU pipe)",
                  5: "LOP3+IMAD (ALU+FMA pipes)", 6: "SHF imm", 7: "LOP3 imm", 8: "IMAD imm",
                  9: "LOP3+SHF+IMAD imm (ALU+FMA pipes)"}


def measure_int_roof(iters: int = 4000, reps: int = 5, stream=None) -> dict:
    """The measured INT32 issue roof: warp instructions / s over all SMs per
    kind, best of `reps` CUDA-event-timed launches after a warm-up."""
    import torch
    sink = torch.zeros(1, dtype=torch.int32, device="cuda")
    s = stream if stream is not None else torch.cuda.current_stream()
    out = {}
    for kind, name in INT_ROOF_KINDS.items():
        tp_bench_int_roof(kind, 64, sink, s)
        best = None
        for _ in range(reps):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            w = tp_bench_int_roof(kind, iters, sink, s)
            b.record(s)
            torch.cuda.synchronize()
            ms = a.elapsed_time(b)
            best = ms if best is None or ms < best else best
        out[name] = {"warp_insts": w, "ms": best, "warp_insts_per_s": w / (best / 1e3),
                     "lane_ops_per_s": 32 * w / (best / 1e3)}
    out["roof_warp_insts_per_s"] = max(v["warp_insts_per_s"] for v in out.values())
    return out


def tp_debug_counters():
    """16 cycle counters of a -DTP_PROFILE_WAITS build (zeros otherwise); resets them."""
    import numpy as np
    out = np.zeros(16, np.uint64)
    _check(_lib.tp_debug_counters(out.ctypes.data), "tp_debug_counters")
    return out


def tp_launch_count() -> int:
    return int(_lib.tp_launch_count())


def tp_device_info():
    sms, occ = ctypes.c_int(), ctypes.c_int()
    _check(_lib.tp_device_info(ctypes.byref(sms), ctypes.byref(occ)), "tp_device_info")
    return sms.value, occ.value


# ------------------------------------------------------------------ convenience objects
class HostColumn:
    """An encoded column in host memory (numpy arrays with guard words) + its tp_column."""

    def __init__(self, scheme: str, x: np.ndarray):
        x = np.ascontiguousarray(x, dtype=np.int32)
        sc = SCHEMES[scheme]
        nb, w0, w1 = tp_encode_size(sc, x)
        self.scheme = scheme
        self.starts0 = np.zeros(nb + 1 + GUARD_WORDS, np.uint32)
        self.data0 = np.zeros(w0 + GUARD_WORDS, np.uint32)
        self.starts1 = np.zeros(nb + 1 + GUARD_WORDS, np.uint32) if sc == TP_RFOR else None
        self.data1 = np.zeros(w1 + GUARD_WORDS, np.uint32) if sc == TP_RFOR else None
        self.col = tp_encode(sc, x, self.starts0, self.data0, self.starts1, self.data1)

    @property
    def n(self) -> int:
        return int(self.col.n)

    def nbytes(self) -> int:
        return tp_compressed_bytes(self.col)

    def header(self) -> np.ndarray:
        return np.array([self.col.block_size, self.col.miniblock_count, self.col.n], np.uint32)

    def arrays(self) -> dict:
        """Used words only (no guard words): the oracle's layout for byte comparison."""
        nb = int(self.col.num_blocks)
        d = {"header": self.header(), "starts0": self.starts0[:nb + 1], "data0": self.data0[:self.col.words0]}
        if self.starts1 is not None:
            d["starts1"] = self.starts1[:nb + 1]
            d["data1"] = self.data1[:self.col.words1]
        return d

    def to_device(self, device=None) -> "DeviceColumn":
        return DeviceColumn(self, device)


def _to_dev(a: np.ndarray | None, device, pinned: bool = False):
    import torch
    if a is None:
        return None
    t = torch.from_numpy(a.view(np.int32))
    if pinned:
        t = t.pin_memory()
    return t.to(device, non_blocking=pinned)


class DeviceColumn:
    """Device copies (torch int32 storage) of an encoded column + a tp_column of device pointers."""

    def __init__(self, host: HostColumn, device=None):
        import torch
        device = device if device is not None else torch.device("cuda", torch.cuda.current_device())
        self.host = host
        self.starts0 = _to_dev(host.starts0, device)
        self.data0 = _to_dev(host.data0, device)
        self.starts1 = _to_dev(host.starts1, device)
        self.data1 = _to_dev(host.data1, device)
        c = tp_column()
        ctypes.pointer(c)[0] = host.col
        c.starts0, c.data0 = self.starts0.data_ptr(), self.data0.data_ptr()
        if self.starts1 is not None:
            c.starts1, c.data1 = self.starts1.data_ptr(), self.data1.data_ptr()
        self.col = c

    @property
    def n(self) -> int:
        return int(self.col.n)

    def nbytes(self) -> int:
        return tp_compressed_bytes(self.col)


class GpuColumn:
    """A column encoded ON THE DEVICE by the tile-parallel encoder (tp_gpu_encode): torch int32
    storage (capacity = the bound, or exact sizes with exact=True) + its tp_column of device
    pointers.  Same interface as DeviceColumn."""

    def __init__(self, x, scheme: str = "for", exact: bool = False, work=None, stream=None):
        import torch
        assert x.is_cuda and x.dtype == torch.int32 and x.is_contiguous()
        n = x.numel()
        dev = x.device
        if work is None:
            work = torch.empty((tp_gpu_encode_workspace_bytes(n) + 7) // 8, dtype=torch.int64, device=dev)
        if scheme == "auto":
            s, _ = tp_gpu_choose_scheme(x, n, work, stream)
            scheme = SCHEME_NAMES[s]
        sc = SCHEMES[scheme]
        nb, w0, w1 = tp_gpu_encode_bound(sc, n)
        if exact and sc != TP_NONE:
            w = tp_gpu_encode_sizes(x, n, work, stream)
            w0, w1 = {TP_FOR: (w[0], 0), TP_DFOR: (w[1], 0), TP_RFOR: (w[2], w[3])}[sc]
        self.scheme = scheme
        self.starts0 = torch.empty(nb + 1 + GUARD_WORDS, dtype=torch.int32, device=dev)
        self.data0 = torch.empty(w0 + GUARD_WORDS, dtype=torch.int32, device=dev)
        rf = sc == TP_RFOR
        self.starts1 = torch.empty(nb + 1 + GUARD_WORDS, dtype=torch.int32, device=dev) if rf else None
        self.data1 = torch.empty(w1 + GUARD_WORDS, dtype=torch.int32, device=dev) if rf else None
        self.col = tp_gpu_encode(sc, x, n, self.starts0, self.data0, w0, self.starts1, self.data1, w1, work, stream)

    @property
    def n(self) -> int:
        return int(self.col.n)

    def nbytes(self) -> int:
        return tp_compressed_bytes(self.col)

    def arrays(self) -> dict:
        """Used words only, copied to the host (the oracle's layout for byte comparison)."""
        nb = int(self.col.num_blocks)
        hdr = np.array([self.col.block_size, self.col.miniblock_count, self.col.n], np.uint32)
        d = {"header": hdr, "starts0": self.starts0[:nb + 1].cpu().numpy().view(np.uint32),
             "data0": self.data0[:self.col.words0].cpu().numpy().view(np.uint32)}
        if self.starts1 is not None:
            d["starts1"] = self.starts1[:nb + 1].cpu().numpy().view(np.uint32)
            d["data1"] = self.data1[:self.col.words1].cpu().numpy().view(np.uint32)
        return d


def gpu_encode(x, scheme: str = "for", exact: bool = False, stream=None) -> GpuColumn:
    """Encode a DEVICE int32 tensor on the GPU (scheme 'for' | 'dfor' | 'rfor' | 'none' | 'auto')."""
    return GpuColumn(x, scheme, exact=exact, stream=stream)


def encode(x: np.ndarray, scheme: str = "for") -> HostColumn:
    """Encode a host int32 column (scheme 'for' | 'dfor' | 'rfor' | 'auto' = GPU-*)."""
    if scheme == "auto":
        s, _ = tp_choose_scheme(np.ascontiguousarray(x, np.int32))
        scheme = SCHEME_NAMES[s]
    return HostColumn(scheme, x)


def decode(dcol: DeviceColumn, out=None, stream=None):
    import torch
    if out is None:
        out = torch.empty(dcol.n, dtype=torch.int32, device=dcol.data0.device)
    tp_decode(dcol.col, out, stream)
    return out


def decode_sum(dcol: DeviceColumn, out=None, stream=None):
    import torch
    if out is None:
        out = torch.zeros(1, dtype=torch.int64, device=dcol.data0.device)
    tp_decode_sum(dcol.col, out, stream)
    return out


def select_project_sum(dcols, lo, hi, proj: str = "col", a: int = 0, b: int = 0, out=None, stream=None):
    import torch
    if out is None:
        out = torch.zeros(1, dtype=torch.int64, device=dcols[0].data0.device)
    tp_select_project_sum([d.col for d in dcols], lo, hi, TP_PROJ[proj], a, b, out, stream)
    return out


def tp_status_string(status: int) -> str:
    return _lib.tp_status_string(status).decode()
