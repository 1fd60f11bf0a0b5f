"""The device-side API (include/tilepack/device.cuh): the paper's LoadBitPack / LoadDBitPack /
LoadRBitPack used inside a USER kernel.  tests/device_api/user_kernels.cu
includes only the public headers (no libtilepack.so); its kernels decode whole columns and run a
three-column select-sum, checked against the oracle."""
import ctypes
import os

import numpy as np
import pytest

import datagen
import oracle
from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp

HERE = os.path.dirname(os.path.abspath(__file__))
SO = os.path.join(HERE, "device_api", "libuser_kernels.so")
I32 = (-(2**31), 2**31 - 1)


def _lib():
    L = ctypes.CDLL(SO)
    colp = ctypes.POINTER(tp.tp_column)
    L.user_decode_launch.argtypes = [colp, ctypes.c_void_p, ctypes.c_void_p]
    L.user_select_sum_launch.argtypes = [colp, colp, colp, ctypes.c_int32, ctypes.c_int32, ctypes.c_void_p,
                                         ctypes.c_void_p]
    return L


def test_user_kernel_library_built_without_tilepack():
    """the user library exports its launchers and does not link libtilepack.so"""
    import subprocess
    L = _lib()
    assert hasattr(L, "user_decode_launch") and hasattr(L, "user_select_sum_launch")
    deps = subprocess.run(["ldd", SO], capture_output=True, text=True).stdout
    assert "libtilepack" not in deps
    hdr = open(os.path.join(os.path.dirname(HERE), "include", "tilepack", "device.cuh")).read()
    for f in ("tp_load_for", "tp_load_dfor", "tp_load_rfor"):
        assert f"__device__ void {f}(" in hdr


def _columns(n, seed):
    return {"for": datagen.uniform_bits(19, n, seed=seed),
            "dfor": datagen.near_sorted(n, seed=seed + 1),
            "rfor": datagen.runs(n, 6, seed=seed + 2)}


@pytest.mark.gpu
@pytest.mark.parametrize("scheme", ["for", "dfor", "rfor"])
def test_user_kernel_decodes_columns(scheme):
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    L = _lib()
    cols = [x for _, x in datagen.mixed_columns(seed=17) if len(x)] + [_columns(3_000_017, 5)[scheme]]
    for x in cols:
        d = tp.encode(x, scheme).to_device()
        out = torch.full((len(x),), -7, dtype=torch.int32, device="cuda")
        s = torch.cuda.current_stream()
        assert L.user_decode_launch(ctypes.byref(d.col), ctypes.c_void_p(out.data_ptr()),
                                    ctypes.c_void_p(s.cuda_stream)) == 0
        want = oracle.decode(oracle.encode(scheme, x))
        assert np.array_equal(out.cpu().numpy(), want), (scheme, len(x))


@pytest.mark.gpu
def test_user_kernel_select_sum():
    """SELECT SUM(a * b) WHERE lo <= c <= hi over a GPU-FOR, a GPU-DFOR and a GPU-RFOR column,
    decoded by the device API inside one user kernel == the oracle's select_project_sum."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    L = _lib()
    for n, seed in ((512 * 37 + 77, 1), (2_000_003, 2)):
        c = _columns(n, seed)
        a = (c["for"] & 0xffff).astype(np.int32)
        da = tp.encode(a, "for").to_device()
        db = tp.encode(c["dfor"], "dfor").to_device()
        dc = tp.encode(c["rfor"], "rfor").to_device()
        lo, hi = 1000, 40000
        out = torch.zeros(1, dtype=torch.int64, device="cuda")
        s = torch.cuda.current_stream()
        assert L.user_select_sum_launch(ctypes.byref(da.col), ctypes.byref(db.col), ctypes.byref(dc.col), lo, hi,
                                        ctypes.c_void_p(out.data_ptr()), ctypes.c_void_p(s.cuda_stream)) == 0
        want = oracle.select_project_sum([a, c["dfor"], c["rfor"]], [I32[0], I32[0], lo], [I32[1], I32[1], hi],
                                         "mul", 0, 1)
        assert int(out.item()) == want
