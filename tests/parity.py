"""Comparison helpers for GPU-vs-oracle parity.

Bar (BASELINE.json north_star; reading R2):
  * y index set: bit-exact;
  * values: |y_gpu - y_ref| <= tol * sum_j |a_ij x_j|, tol = 1e-12 (fp64) and,
    for fp32 (fp32 storage, fp64 accumulation, one rounding; R3), the GPU value
    must be within 1e-5 * sum|a x| of the oracle's fp64 sum rounded to fp32;
  * MIN_SECOND / OR_AND / integer-valued inputs: bit-exact.
"""
import numpy as np
import torch

import oracle


def abs_csc(C):
    return oracle.CSC(C.m, C.n, C.col_ptr, C.row_idx, None if C.val is None else np.abs(C.val))


def check_spmspv(C, yi, yv, xi, xv, semiring=oracle.PLUS_TIMES, dtype="f64", exact=False, Cabs=None):
    xi_np = xi.detach().cpu().numpy() if hasattr(xi, "detach") else np.asarray(xi)
    xv_np = None if xv is None else (xv.detach().cpu().numpy().astype(np.float64) if hasattr(xv, "detach")
                                     else np.asarray(xv, np.float64))
    ri, rv = oracle.spmspv(C, xi_np, xv_np, semiring)
    gi = yi.detach().cpu().numpy()
    assert gi.shape == ri.shape, f"y_nnz {gi.size} vs oracle {ri.size}"
    assert np.array_equal(gi, ri), "y index set differs"
    if semiring == oracle.OR_AND or yv is None:
        return ri, rv
    gv = yv.detach().cpu().numpy().astype(np.float64)
    if semiring == oracle.MIN_SECOND:
        ref = rv.astype(np.float32).astype(np.float64) if dtype == "f32" else rv
        assert np.array_equal(gv, ref), "MIN_SECOND values differ"
        return ri, rv
    if dtype == "f32":
        ref = rv.astype(np.float32).astype(np.float64)
    else:
        ref = rv
    if exact:
        assert np.array_equal(gv, ref), f"values differ (max abs {np.max(np.abs(gv - ref)) if gv.size else 0})"
        return ri, rv
    Cabs = Cabs or abs_csc(C)
    _, mag = oracle.spmspv(Cabs, xi_np, None if xv_np is None else np.abs(xv_np), semiring)
    tol = 1e-12 if dtype == "f64" else 1e-5
    slack = tol * mag + (np.abs(ref) * 2.0 ** -24 if dtype == "f32" else 0.0)
    bad = np.abs(gv - ref) > slack
    assert not bad.any(), f"{bad.sum()} values out of tolerance; worst idx {ri[np.argmax(np.abs(gv - ref) - slack)]}"
    return ri, rv
