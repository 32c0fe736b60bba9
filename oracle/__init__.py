"""CPU oracle for the TurboBC hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product package
(``paper_conf_icppw_artiless21_b200``) never imports it and shares no code with it.

Contents
  * ``brandes.c``  -- textbook Brandes (Eq. 2-4) in plain C / fp64,
    exposed here as :func:`bc`, :func:`bfs`, :func:`delta`; and the same algorithm in C long
    double (extended exponent range, NEXT-2) as :func:`bc_ld`, :func:`bfs_ld`.
  * ``brute.py``   -- exact brute force of Freeman's Eq. 1 with rationals
    for graphs of <= 12 vertices (a second, independent oracle used to pin the first).

Every function is pinned by ``tests/test_oracle.py`` (brute force, closed forms,
invariants, networkx); there is no "parity unpinned" function in this package.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "brandes.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile ``brandes.c`` into ``liboracle.so`` with gcc (-O3, pthreads)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-march=native", "-std=c11", "-fPIC", "-shared",
                               "-o", tmp, _SRC, "-lpthread", "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        i64, i32, dbl = ctypes.c_int64, ctypes.c_int32, ctypes.c_double
        P = ctypes.POINTER
        lib.oracle_bc.argtypes = [i64, P(i64), P(i32), ctypes.c_int, P(i32), i64, ctypes.c_int, P(dbl)]
        lib.oracle_bc.restype = ctypes.c_int
        lib.oracle_bc_timed.argtypes = [i64, P(i64), P(i32), ctypes.c_int, P(i32), i64, ctypes.c_int, P(dbl),
                                        P(dbl)]
        lib.oracle_bc_timed.restype = ctypes.c_int
        lib.oracle_bfs.argtypes = [i64, P(i64), P(i32), i32, P(i32), P(dbl)]
        lib.oracle_bfs.restype = ctypes.c_int
        lib.oracle_delta.argtypes = [i64, P(i64), P(i32), i32, P(dbl)]
        lib.oracle_delta.restype = ctypes.c_int
        lib.oracle_bfs_ld.argtypes = [i64, P(i64), P(i32), i32, P(i32), P(dbl), P(i32)]
        lib.oracle_bfs_ld.restype = ctypes.c_int
        lib.oracle_bc_ld.argtypes = [i64, P(i64), P(i32), ctypes.c_int, P(i32), i64, P(dbl)]
        lib.oracle_bc_ld.restype = ctypes.c_int
        _lib = lib
    return _lib


def _ptr(a, ct):
    return a.ctypes.data_as(ctypes.POINTER(ct))


def _csc(col_ptr, row_idx):
    cp = np.ascontiguousarray(col_ptr, dtype=np.int64)
    ri = np.ascontiguousarray(row_idx, dtype=np.int32)
    if ri.size == 0:
        ri = np.zeros(1, dtype=np.int32)
    return cp, ri


def bc(col_ptr, row_idx, directed: bool, sources, nthreads: int | None = None) -> np.ndarray:
    """bc(v) = sum over the source list of delta_s(v) (Eq. 3), halved if undirected."""
    lib = _load()
    cp, ri = _csc(col_ptr, row_idx)
    n = cp.size - 1
    src = np.ascontiguousarray(sources, dtype=np.int32)
    k = src.size
    if k == 0:
        return np.zeros(n, dtype=np.float64)
    out = np.zeros(n, dtype=np.float64)
    nt = nthreads if nthreads else (os.cpu_count() or 1)
    rc = lib.oracle_bc(n, _ptr(cp, ctypes.c_int64), _ptr(ri, ctypes.c_int32), int(bool(directed)),
                       _ptr(src, ctypes.c_int32), k, int(nt), _ptr(out, ctypes.c_double))
    if rc != 0:
        raise ValueError("oracle_bc: invalid input")
    return out


def bc_timed(col_ptr, row_idx, directed: bool, sources, nthreads: int):
    """(bc, seconds of the source loop alone, graph build excluded) -- bench cpu_baseline hook."""
    lib = _load()
    cp, ri = _csc(col_ptr, row_idx)
    n = cp.size - 1
    src = np.ascontiguousarray(sources, dtype=np.int32)
    out = np.zeros(n, dtype=np.float64)
    secs = ctypes.c_double(0.0)
    rc = lib.oracle_bc_timed(n, _ptr(cp, ctypes.c_int64), _ptr(ri, ctypes.c_int32), int(bool(directed)),
                             _ptr(src, ctypes.c_int32), src.size, int(nthreads), _ptr(out, ctypes.c_double),
                             ctypes.byref(secs))
    if rc != 0:
        raise ValueError("oracle_bc_timed: invalid input")
    return out, secs.value


def bfs(col_ptr, row_idx, source: int):
    """(depth int32[n], sigma float64[n]) from one source: depth(s)=0, unreachable -1."""
    lib = _load()
    cp, ri = _csc(col_ptr, row_idx)
    n = cp.size - 1
    depth = np.empty(n, dtype=np.int32)
    sigma = np.empty(n, dtype=np.float64)
    rc = lib.oracle_bfs(n, _ptr(cp, ctypes.c_int64), _ptr(ri, ctypes.c_int32), int(source),
                        _ptr(depth, ctypes.c_int32), _ptr(sigma, ctypes.c_double))
    if rc != 0:
        raise ValueError("oracle_bfs: invalid input")
    return depth, sigma


def delta(col_ptr, row_idx, source: int) -> np.ndarray:
    """One-sided dependencies delta_s(v) (Eq. 2), unhalved; 0 at s and unreachable v."""
    lib = _load()
    cp, ri = _csc(col_ptr, row_idx)
    n = cp.size - 1
    out = np.empty(n, dtype=np.float64)
    rc = lib.oracle_delta(n, _ptr(cp, ctypes.c_int64), _ptr(ri, ctypes.c_int32), int(source),
                          _ptr(out, ctypes.c_double))
    if rc != 0:
        raise ValueError("oracle_delta: invalid input")
    return out


def bfs_ld(col_ptr, row_idx, source: int):
    """Extended range (C long double, NEXT-2): (depth int32[n], sigma mantissa float64[n] in [0.5, 1),
    sigma binary exponent int32[n]); sigma = mantissa * 2**exponent, also beyond fp64's range."""
    lib = _load()
    cp, ri = _csc(col_ptr, row_idx)
    n = cp.size - 1
    depth = np.empty(n, dtype=np.int32)
    mant = np.empty(n, dtype=np.float64)
    expo = np.empty(n, dtype=np.int32)
    rc = lib.oracle_bfs_ld(n, _ptr(cp, ctypes.c_int64), _ptr(ri, ctypes.c_int32), int(source),
                           _ptr(depth, ctypes.c_int32), _ptr(mant, ctypes.c_double), _ptr(expo, ctypes.c_int32))
    if rc != 0:
        raise ValueError("oracle_bfs_ld: invalid input")
    return depth, mant, expo


def bc_ld(col_ptr, row_idx, directed: bool, sources) -> np.ndarray:
    """bc with long double sigma / delta / accumulation (single thread), rounded to float64."""
    lib = _load()
    cp, ri = _csc(col_ptr, row_idx)
    n = cp.size - 1
    src = np.ascontiguousarray(sources, dtype=np.int32)
    out = np.zeros(n, dtype=np.float64)
    if src.size == 0:
        return out
    rc = lib.oracle_bc_ld(n, _ptr(cp, ctypes.c_int64), _ptr(ri, ctypes.c_int32), int(bool(directed)),
                          _ptr(src, ctypes.c_int32), src.size, _ptr(out, ctypes.c_double))
    if rc != 0:
        raise ValueError("oracle_bc_ld: invalid input")
    return out
