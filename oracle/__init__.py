"""CPU oracle for TileSpMSpV / TileBFS (Ji et al., ICPP '22).

TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
cpu_baseline / --impl reference legs of bench.py may import this package.  The
product package (paper_conf_icpp_jisl0t022_b200) never imports it, and it shares
no code with the product: the arithmetic is in oracle.c (plain C, single
thread, fp64), this file only builds it and marshals numpy arrays.

Functions (each cites its passage in oracle.c):
  csr_to_csc, spmspv (Alg 2), bfs_queue, bfs_alg3 (Alg 3), tile_vector (Fig 3),
  tile_census (Sec 3.2.1), bitmask_tiles (Sec 3.2.3 / Fig 5).
Pins: tests/test_oracle_*.py.  No function is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

PLUS_TIMES, OR_AND, MIN_SECOND = 0, 1, 2


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (plain -O2, no OpenMP, no -ffast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-fPIC", "-shared", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def _L():
    global _lib
    if _lib is None:
        build()
        _lib = ctypes.CDLL(_LIB)
    return _lib


def _p(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None else ctypes.c_void_p(0)


def _np(t, dtype):
    if t is None:
        return None
    if hasattr(t, "detach"):
        t = t.detach().cpu().numpy()
    return np.ascontiguousarray(np.asarray(t), dtype=dtype)


def _chk(rc, what):
    if rc == -1:
        raise ValueError(f"oracle.{what}: invalid input")
    if rc != 0:
        raise MemoryError(f"oracle.{what}: rc={rc}")


class CSC:
    """Column-compressed copy of A owned by the oracle (its own format conversion)."""

    def __init__(self, m, n, col_ptr, row_idx, val):
        self.m, self.n, self.col_ptr, self.row_idx, self.val = m, n, col_ptr, row_idx, val


def csr_to_csc(m, n, row_ptr, col_idx, values=None) -> CSC:
    row_ptr = _np(row_ptr, np.int64)
    col_idx = _np(col_idx, np.int32)
    vals = _np(values, np.float64)
    nnz = int(row_ptr[-1])
    col_ptr = np.zeros(n + 1, np.int64)
    row_idx = np.zeros(max(nnz, 1), np.int32)
    cval = np.zeros(max(nnz, 1), np.float64) if vals is not None else None
    f = _L().oracle_csr_to_csc
    f.restype = ctypes.c_int
    _chk(f(ctypes.c_int64(m), ctypes.c_int64(n), _p(row_ptr), _p(col_idx), _p(vals),
           _p(col_ptr), _p(row_idx), _p(cval)), "csr_to_csc")
    return CSC(m, n, col_ptr, row_idx[:nnz], None if cval is None else cval[:nnz])


def csc_of(A) -> CSC:
    """A: synth.CSR (torch tensors) -> oracle CSC (fp64 values)."""
    return csr_to_csc(A.m, A.n, A.row_ptr, A.col_idx, A.values)


def spmspv(C: CSC, x_idx, x_val=None, semiring=PLUS_TIMES):
    """Algorithm 2.  Returns (y_idx int32 ascending, y_val float64)."""
    x_idx = _np(x_idx, np.int32)
    x_val = _np(x_val, np.float64)
    k = x_idx.size
    y_idx = np.zeros(max(C.m, 1), np.int32)
    y_val = np.zeros(max(C.m, 1), np.float64)
    ynnz = ctypes.c_int64(0)
    f = _L().oracle_spmspv
    f.restype = ctypes.c_int
    _chk(f(ctypes.c_int64(C.m), ctypes.c_int64(C.n), _p(C.col_ptr), _p(C.row_idx), _p(C.val),
           ctypes.c_int(semiring), ctypes.c_int64(k), _p(x_idx), _p(x_val), _p(y_idx), _p(y_val),
           ctypes.byref(ynnz)), "spmspv")
    q = ynnz.value
    return y_idx[:q].copy(), y_val[:q].copy()


def bfs_queue(C: CSC, source: int) -> np.ndarray:
    levels = np.zeros(max(C.n, 1), np.int32)
    f = _L().oracle_bfs_queue
    f.restype = ctypes.c_int
    _chk(f(ctypes.c_int64(C.n), _p(C.col_ptr), _p(C.row_idx), ctypes.c_int64(source), _p(levels)),
         "bfs_queue")
    return levels[:C.n]


def bfs_alg3(C: CSC, source: int) -> np.ndarray:
    levels = np.zeros(max(C.n, 1), np.int32)
    f = _L().oracle_bfs_alg3
    f.restype = ctypes.c_int
    _chk(f(ctypes.c_int64(C.n), _p(C.col_ptr), _p(C.row_idx), ctypes.c_int64(source), _p(levels)),
         "bfs_alg3")
    return levels[:C.n]


def bfs_parents(C: CSC, source: int):
    """Alg 3 over MIN_SECOND: (levels, min-id parents)."""
    levels = np.zeros(max(C.n, 1), np.int32)
    parents = np.zeros(max(C.n, 1), np.int32)
    f = _L().oracle_bfs_parents
    f.restype = ctypes.c_int
    _chk(f(ctypes.c_int64(C.n), _p(C.col_ptr), _p(C.row_idx), ctypes.c_int64(source), _p(levels), _p(parents)),
         "bfs_parents")
    return levels[:C.n], parents[:C.n]


def tile_vector(n, nt, x_idx, x_val):
    """Fig 3 tiled sparse vector: returns (x_ptr int64[ceil(n/nt)], x_tile float64)."""
    x_idx = _np(x_idx, np.int32)
    x_val = _np(x_val, np.float64)
    T = (n + nt - 1) // nt
    x_ptr = np.zeros(max(T, 1), np.int64)
    x_tile = np.zeros(max(T * nt, 1), np.float64)
    cnt = ctypes.c_int64(0)
    f = _L().oracle_tile_vector
    f.restype = ctypes.c_int
    _chk(f(ctypes.c_int64(n), ctypes.c_int32(nt), ctypes.c_int64(x_idx.size), _p(x_idx), _p(x_val),
           _p(x_ptr), _p(x_tile), ctypes.byref(cnt)), "tile_vector")
    return x_ptr[:T], x_tile[:cnt.value * nt]


def tile_census(m, n, row_ptr, col_idx, nt, thr):
    """(non-empty tiles, tiles with > thr nnz, nnz moved to the side matrix)."""
    row_ptr = _np(row_ptr, np.int64)
    col_idx = _np(col_idx, np.int32)
    a, b, c = ctypes.c_int64(0), ctypes.c_int64(0), ctypes.c_int64(0)
    f = _L().oracle_tile_census
    f.restype = ctypes.c_int
    _chk(f(ctypes.c_int64(m), ctypes.c_int64(n), _p(row_ptr), _p(col_idx), ctypes.c_int32(nt),
           ctypes.c_int32(thr), ctypes.byref(a), ctypes.byref(b), ctypes.byref(c)), "tile_census")
    return a.value, b.value, c.value


def bitmask_tiles(m, n, row_ptr, col_idx, nt, orient, max_tiles=4096):
    """Sec 3.2.3 bitmask tiles (MSB-first).  orient 0 = A1 (column words),
    1 = A2 (row words).  Returns list of (I, J, [nt words])."""
    row_ptr = _np(row_ptr, np.int64)
    col_idx = _np(col_idx, np.int32)
    tI = np.zeros(max_tiles, np.int64)
    tJ = np.zeros(max_tiles, np.int64)
    words = np.zeros(max_tiles * nt, np.uint64)
    cnt = ctypes.c_int64(0)
    f = _L().oracle_bitmask_tiles
    f.restype = ctypes.c_int
    _chk(f(ctypes.c_int64(m), ctypes.c_int64(n), _p(row_ptr), _p(col_idx), ctypes.c_int32(nt),
           ctypes.c_int32(orient), ctypes.c_int64(max_tiles), _p(tI), _p(tJ), _p(words),
           ctypes.byref(cnt)), "bitmask_tiles")
    return [(int(tI[t]), int(tJ[t]), [int(w) for w in words[t * nt:(t + 1) * nt]])
            for t in range(cnt.value)]
