"""B200-native (sm_100a) tile-based lightweight integer compression
(GPU-FOR / GPU-DFOR / GPU-RFOR, Shanbhag et al., SIGMOD '22).

The compute path is the native library ``libtilepack.so`` (include/tilepack.h);
``tilepack`` is its ctypes binding.  Importing raises if the library is missing.
"""
from . import tilepack  # noqa: F401
from .tilepack import (DeviceColumn, HostColumn, decode, decode_sum, encode,  # noqa: F401
                       select_project_sum)

__all__ = ["tilepack", "encode", "decode", "decode_sum", "select_project_sum", "HostColumn", "DeviceColumn"]
