"""The bucketed column-driven TileSpMSpV kernel (propagation blocking, spmspv_flat.cu
PB variant) forced on (TSMV_SPMSPV_KERNEL=pb) against the oracle:
integer-exact over thresholds and densities, the BASELINE shapes, fp32, the three
semirings, ragged / rectangular / tiny matrices, every bucket width, staging
buffers forced to overflow into the global accumulator (TSMV_PB_CAP), hot-row
privatisation off, invalid x, y capacity, and calls alternating with the plain
flat kernel (separate counter parities)."""
import os

import numpy as np
import pytest
import torch

import oracle
import synth
from parity import check_spmspv

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


@pytest.fixture(scope="module")
def tsmv():
    from paper_conf_icpp_jisl0t022_b200 import tsmv as t
    return t


@pytest.fixture
def pb_env():
    """Sets environment switches for the test (read at create / per call)."""
    keys = []

    def set_(**kv):
        for k, v in kv.items():
            os.environ[k] = str(v)
            keys.append(k)
    os.environ["TSMV_SPMSPV_KERNEL"] = "pb"
    keys.append("TSMV_SPMSPV_KERNEL")
    yield set_
    for k in keys:
        os.environ.pop(k, None)


def _run(tsmv, A, dens, seed=7, dtype="f64", integer=False, semiring="plus_times", **opt):
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype=dtype, build_bfs=0, **opt)
    sr = {"plus_times": oracle.PLUS_TIMES, "or_and": oracle.OR_AND, "min_second": oracle.MIN_SECOND}[semiring]
    for d in dens:
        xi, xv = synth.sample_x(A.n, max(1, synth.density_k(A.n, d)), seed=seed, integer=integer, dtype=dtype)
        yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV), semiring=semiring)
        check_spmspv(C, yi, yv, xi, xv, semiring=sr, dtype=dtype, exact=integer)
    M.close()


@pytest.mark.parametrize("thr", [0, 2, 8])
@pytest.mark.parametrize("cap", [None, 64])
def test_pb_integer_exact(tsmv, pb_env, thr, cap):
    if cap:
        pb_env(TSMV_PB_CAP=cap)
    A = synth.attach_values(synth.rmat(14, 16, seed=4), seed=2, integer=True)
    _run(tsmv, A, (0.0005, 0.01, 0.1, 1.0), integer=True, sparse_tile_max_nnz=thr)


@pytest.mark.parametrize("bl", [10, 12, 14])
def test_pb_bucket_widths(tsmv, pb_env, bl):
    pb_env(TSMV_PB_BL=bl)
    A = synth.attach_values(synth.rmat(16, 16, seed=5), seed=3, integer=True)
    _run(tsmv, A, (0.001, 0.01, 0.05), integer=True)


@pytest.mark.parametrize("gen", ["stencil2d", "stencil3d", "banded", "uniform"])
@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_pb_shapes(tsmv, pb_env, gen, dtype):
    A = {"stencil2d": lambda: synth.stencil2d(70, 45), "stencil3d": lambda: synth.stencil3d(24),
         "banded": lambda: synth.banded(5000, 40), "uniform": lambda: synth.uniform(3000, 3000, 9, seed=2)}[gen]()
    _run(tsmv, synth.attach_values(A, seed=3, dtype=dtype), (0.002, 0.05, 0.5), seed=11, dtype=dtype)


@pytest.mark.parametrize("semiring", ["or_and", "min_second"])
@pytest.mark.parametrize("cap", [None, 32])
def test_pb_semirings(tsmv, pb_env, semiring, cap):
    if cap:
        pb_env(TSMV_PB_CAP=cap)
    _run(tsmv, synth.attach_values(synth.rmat(13, 16, seed=6), seed=5), (0.01, 0.2), seed=2, semiring=semiring)
    _run(tsmv, synth.attach_values(synth.stencil3d(20), seed=5), (0.05,), seed=2, semiring=semiring)


@pytest.mark.parametrize("shape", [(1000, 3000), (3000, 1000), (17, 5000), (4099, 4099), (70000, 300)])
def test_pb_ragged_rectangular(tsmv, pb_env, shape):
    m, n = shape
    A = synth.attach_values(synth.uniform(m, n, 6, seed=3), seed=4)
    _run(tsmv, A, (0.01, 0.3, 1.0), seed=6)


def test_pb_hot_rows(tsmv, pb_env):
    """With the (opt-in) hot-row privatisation: hot partials reduced over the CTAs."""
    pb_env(TSMV_HOT=1)
    A = synth.attach_values(synth.rmat(14, 16, seed=8), seed=1, integer=True)
    _run(tsmv, A, (0.01, 0.1), integer=True)


def test_pb_errors_capacity_and_alternation(tsmv, pb_env):
    A = synth.attach_values(synth.rmat(13, 16, seed=9), seed=1)
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), build_bfs=0)
    for xi in (torch.tensor([5, 5], dtype=torch.int32), torch.tensor([A.n], dtype=torch.int32)):
        with pytest.raises(tsmv.TsmvError):
            M.spmspv(xi.to(DEV), torch.ones(xi.numel(), dtype=torch.float64, device=DEV))
    # alternate the bucketed and the plain flat kernel on one context
    for s in range(6):
        os.environ["TSMV_SPMSPV_KERNEL"] = "pb" if s % 3 else "flat"
        xi, xv = synth.sample_x(A.n, 80 + 40 * s, seed=20 + s)
        yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
        check_spmspv(C, yi, yv, xi, xv)
    os.environ["TSMV_SPMSPV_KERNEL"] = "pb"
    # too small a y: ECAPACITY with the required size; the next call is clean
    xi, xv = synth.sample_x(A.n, 200, seed=3)
    ri, _ = oracle.spmspv(C, xi.numpy(), xv.numpy(), oracle.PLUS_TIMES)
    yi = torch.empty(max(1, ri.size // 2), dtype=torch.int32, device=DEV)
    yv = torch.empty(yi.numel(), dtype=torch.float64, device=DEV)
    with pytest.raises(tsmv.TsmvError) as e:
        M.spmspv(xi.to(DEV), xv.to(DEV), y_idx=yi, y_val=yv)
    assert e.value.status == tsmv.ECAPACITY
    yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
    check_spmspv(C, yi, yv, xi, xv)
    M.close()


def test_pb_full_size_T(tsmv, pb_env):
    """T (R-MAT s22 directed, fp64, x 1 %) through the bucketed kernel, every row
    against the oracle, three x samples (the bench's launch configuration)."""
    A = synth.attach_values(synth.rmat(22, 16, seed=1, device=DEV), seed=1)
    M = tsmv.TiledMatrix.from_csr(A, build_bfs=0)
    C = oracle.csc_of(A.to("cpu"))
    for s in (1, 2, 3):
        xi, xv = synth.sample_x(A.n, synth.density_k(A.n, 0.01), seed=s)
        yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
        check_spmspv(C, yi, yv, xi, xv)
    M.close()
