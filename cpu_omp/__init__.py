"""CPU speed baseline: OpenMP column-merge SpMSpV ("bucket"
form) and level-synchronous BFS on all host cores, timed by bench.py beside
the single-thread oracle.  Not the oracle (oracle/ checks; this only measures),
not the product path (no GPU code, nothing shared with libtsmv).  The
computation is in omp_baseline.c; this file builds it and marshals arrays.
Checked against the oracle by tests/test_cpu_omp.py."""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "omp_baseline.c")
_LIB = os.path.join(_HERE, "libomp_baseline.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-fopenmp", "-std=gnu99", "-fPIC", "-shared", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _L():
    global _lib
    if _lib is None:
        build()
        _lib = ctypes.CDLL(_LIB)
    return _lib


def _p(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None else ctypes.c_void_p(0)


def threads() -> int:
    return int(_L().omp_max_threads())


def cpu_model() -> str:
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


class CSC:
    def __init__(self, m, n, col_ptr, row_idx, val):
        self.m, self.n, self.col_ptr, self.row_idx, self.val = m, n, col_ptr, row_idx, val


def csc_of(A) -> CSC:
    """CSC of a synth.CSR (host copy), built by this module's own counting sort."""
    rp = np.ascontiguousarray(A.row_ptr.cpu().numpy(), np.int64)
    ci = np.ascontiguousarray(A.col_idx.cpu().numpy(), np.int32)
    vv = None if A.values is None else np.ascontiguousarray(A.values.cpu().numpy(), np.float64)
    nnz = int(rp[-1])
    cp = np.zeros(A.n + 1, np.int64)
    ri = np.empty(max(nnz, 1), np.int32)
    cv = np.empty(max(nnz, 1), np.float64) if vv is not None else None
    rc = _L().omp_csr_to_csc(ctypes.c_int64(A.m), ctypes.c_int64(A.n), _p(rp), _p(ci), _p(vv), _p(cp), _p(ri), _p(cv))
    if rc:
        raise MemoryError("omp_csr_to_csc")
    return CSC(A.m, A.n, cp, ri, cv)


def spmspv(C: CSC, x_idx, x_val, nthreads: int = 0):
    xi = np.ascontiguousarray(np.asarray(x_idx), np.int32)
    xv = None if x_val is None else np.ascontiguousarray(np.asarray(x_val), np.float64)
    yi = np.empty(max(C.m, 1), np.int32)
    yv = np.empty(max(C.m, 1), np.float64)
    yn = ctypes.c_int64(0)
    rc = _L().omp_spmspv(ctypes.c_int64(C.m), ctypes.c_int64(C.n), _p(C.col_ptr), _p(C.row_idx), _p(C.val),
                         ctypes.c_int64(xi.size), _p(xi), _p(xv), _p(yi), _p(yv), ctypes.byref(yn),
                         ctypes.c_int(nthreads))
    if rc:
        raise MemoryError("omp_spmspv")
    return yi[:yn.value], yv[:yn.value]


def bfs(C: CSC, source: int, nthreads: int = 0) -> np.ndarray:
    lv = np.empty(max(C.n, 1), np.int32)
    rc = _L().omp_bfs(ctypes.c_int64(C.n), _p(C.col_ptr), _p(C.row_idx), ctypes.c_int64(source), _p(lv),
                      ctypes.c_int(nthreads))
    if rc:
        raise MemoryError("omp_bfs")
    return lv[:C.n]
