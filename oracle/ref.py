"""O1 — reference matvec y = A·x by its plain definition
(TEST INFRASTRUCTURE ONLY, see oracle/__init__).

Thin ctypes wrapper over ``oracle/ref_csr.c`` (compensated fp64 Dot2 per row, plus the
tolerance scale bound[i] = sum_j |a_ij||x_j|).  The library is compiled here with gcc
(``build()`` in __graft_entry__ also builds it); it shares nothing with the product.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libref.so")
_LIB = None


def build() -> str:
    src = os.path.join(_HERE, "ref_csr.c")
    if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math",
                               "-fPIC", "-shared", "-o", _SO, src, "-lm"])
    return _SO


def _lib():
    global _LIB
    if _LIB is None:
        _LIB = ctypes.CDLL(build())
        _LIB.ref_spmv_dot2.restype = ctypes.c_int
        _LIB.ref_spmv_rows.restype = ctypes.c_int
        _LIB.ref_num_threads.restype = ctypes.c_int
    return _LIB


def _p(a):
    return a.ctypes.data_as(ctypes.c_void_p)


def _prep(row_ptr, col, val, x):
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int32)
    val = np.ascontiguousarray(val)
    if val.dtype not in (np.float32, np.float64):
        val = val.astype(np.float64)
    x = np.ascontiguousarray(x, dtype=val.dtype)
    return row_ptr, col, val, x, (0 if val.dtype == np.float32 else 1)


def spmv(row_ptr, col, val, x, with_bound: bool = True):
    """Return (y, bound) in fp64 for CSR (row_ptr, col, val) and x (same dtype as val)."""
    row_ptr, col, val, x, dt = _prep(row_ptr, col, val, x)
    m = row_ptr.size - 1
    y = np.empty(m, dtype=np.float64)
    b = np.empty(m, dtype=np.float64) if with_bound else None
    rc = _lib().ref_spmv_dot2(ctypes.c_int64(m), _p(row_ptr), _p(col), _p(val), _p(x), dt, _p(y),
                              _p(b) if b is not None else None)
    if rc:
        raise RuntimeError("ref_spmv_dot2 failed")
    return y, b


def spmv_rows(rows, row_ptr, col, val, x):
    """Reference values (y, bound) for the listed rows only."""
    rows = np.ascontiguousarray(rows, dtype=np.int64)
    row_ptr, col, val, x, dt = _prep(row_ptr, col, val, x)
    y = np.empty(rows.size, dtype=np.float64)
    b = np.empty(rows.size, dtype=np.float64)
    _lib().ref_spmv_rows(ctypes.c_int64(rows.size), _p(rows), _p(row_ptr), _p(col), _p(val), _p(x), dt,
                         _p(y), _p(b))
    return y, b


def num_threads() -> int:
    return int(_lib().ref_num_threads())


def check_tolerance(y, y_ref, bound, dtype) -> tuple[bool, float]:
    """BASELINE.json north_star: fp64 |y - y_ref| <= 1e-12 * bound, fp32 <= 1e-5 * bound,
    per row.  Returns (ok, worst ratio err / (tol * bound))."""
    tol = 1e-12 if np.dtype(dtype) == np.float64 else 1e-5
    err = np.abs(np.asarray(y, dtype=np.float64) - y_ref)
    lim = tol * bound
    ratio = np.where(lim > 0, err / np.where(lim > 0, lim, 1), np.where(err > 0, np.inf, 0.0))
    return bool(np.all(err <= lim)), float(ratio.max()) if ratio.size else 0.0
