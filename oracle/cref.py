"""ctypes wrapper of the plain-C fp64 oracle (oracle/c/spmv_ref.c).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "c", "spmv_ref.c")
_SO = os.path.join(_HERE, "c", "libspmvref.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-o", _SO,
                               _SRC, "-lm"])
    return _SO


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        vp, i64 = ctypes.c_void_p, ctypes.c_int64
        L.spmv_ref_f64.argtypes = [i64, vp, vp, vp, vp, vp]
        L.spmv_ref_neumaier.argtypes = [i64, vp, vp, vp, vp, vp, vp]
        L.spmv_ref_threads.argtypes = [ctypes.c_int]
        L.spmv_ref_threads.restype = ctypes.c_int
        _lib = L
    return _lib


def _c(a, dt):
    a = np.ascontiguousarray(a, dtype=dt)
    return a, a.ctypes.data


def threads(want: int = 0) -> int:
    return lib().spmv_ref_threads(want)


def spmv_f64(row_ptr, col, val, x) -> np.ndarray:
    rp, prp = _c(row_ptr, np.int64)
    c, pc = _c(col, np.int32)
    v, pv = _c(val, np.float32)
    xx, px = _c(x, np.float32)
    n = len(rp) - 1
    y = np.empty(n, np.float64)
    lib().spmv_ref_f64(n, prp, pc, pv, px, y.ctypes.data)
    return y


def spmv_neumaier(row_ptr, col, val, x):
    """(y fp64 compensated, sum|a x| per row)."""
    rp, prp = _c(row_ptr, np.int64)
    c, pc = _c(col, np.int32)
    v, pv = _c(val, np.float32)
    xx, px = _c(x, np.float32)
    n = len(rp) - 1
    y = np.empty(n, np.float64)
    a = np.empty(n, np.float64)
    lib().spmv_ref_neumaier(n, prp, pc, pv, px, y.ctypes.data, a.ctypes.data)
    return y, a
