"""The C-ABI library loads and exports every symbol include/tilepack.h declares (no GPU calls)."""
import ctypes
import os
import re

from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "tilepack.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(tp_[a-z_0-9]+)\s*\(", src)))


def test_every_declared_symbol_is_exported():
    L = ctypes.CDLL(tp.LIB_PATH)
    syms = declared_symbols()
    assert len(syms) >= 12
    for s in syms:
        assert hasattr(L, s), s


def test_binding_has_same_names():
    for s in declared_symbols():
        assert hasattr(tp, s), s


def test_status_strings_and_launch_counter():
    assert tp.lib().tp_status_string(0) == b"ok"
    assert b"unsupported" in tp.lib().tp_status_string(5)
    assert tp.tp_launch_count() >= 0


def test_sm100a_code_only():
    """The library carries sm_100a SASS (cuobjdump lists the kernels)."""
    import shutil
    import subprocess
    cu = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    out = subprocess.run([cu, "--list-elf", tp.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out
