"""Tuned parallel CPU C2R: a stronger CPU baseline reported by bench.py.

Not a product path (the library has no CPU fallback) and not the oracle (oracle/ is the
plain checker).  Built with gcc -O3 -fopenmp from ipt_cpu.c."""
import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ipt_cpu.c")
_LIB = os.path.join(_HERE, "libipt_cpu.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-fopenmp", "-std=gnu11", "-Wall", "-shared", "-fPIC",
                               _SRC, "-o", tmp])
        os.replace(tmp, _LIB)
    return _LIB


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        _lib.ipt_cpu_c2r.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64, ctypes.c_int]
        _lib.ipt_cpu_c2r.restype = ctypes.c_int
    return _lib


def c2r(A: np.ndarray, m: int, n: int) -> None:
    """In place: the row-major m x n buffer A (uint32/uint64/float32/float64) becomes its transpose."""
    assert A.flags.c_contiguous and A.size == m * n and A.itemsize in (4, 8)
    rc = lib().ipt_cpu_c2r(A.ctypes.data_as(ctypes.c_void_p), m, n, A.itemsize)
    if rc != 0:
        raise RuntimeError(f"ipt_cpu_c2r failed: {rc}")


def threads() -> int:
    return int(lib().ipt_cpu_threads())
