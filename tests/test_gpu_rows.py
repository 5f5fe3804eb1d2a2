"""The row-driven TileSpMSpV kernel (Alg 4; spmspv_rows.cu) forced on
(TSMV_SPMSPV_KERNEL=rows) against the oracle on the inputs the column-driven
kernel is checked on: integer-exact over thresholds, the BASELINE shapes, the
three semirings, fp32, ragged and rectangular matrices, empty rows / columns,
invalid x; plus the density switch choosing each kernel where DESIGN.md §6 says."""
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
def rows_forced():
    os.environ["TSMV_SPMSPV_KERNEL"] = "rows"
    yield
    os.environ.pop("TSMV_SPMSPV_KERNEL", None)


@pytest.mark.parametrize("thr", [0, 2, 8])
def test_rows_integer_exact(tsmv, rows_forced, thr):
    A = synth.attach_values(synth.rmat(12, 16, seed=4), seed=2, integer=True)
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), sparse_tile_max_nnz=thr, build_bfs=0)
    for d in (0.001, 0.01, 0.1, 1.0):
        xi, xv = synth.sample_x(A.n, max(1, synth.density_k(A.n, d)), seed=7, integer=True)
        yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
        check_spmspv(C, yi, yv, xi, xv, exact=True)
    M.close()


@pytest.mark.parametrize("gen", ["stencil2d", "stencil3d", "banded", "uniform"])
@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_rows_shapes(tsmv, rows_forced, gen, dtype):
    A = {"stencil2d": lambda: synth.stencil2d(70, 45), "stencil3d": lambda: synth.stencil3d(24),
         "banded": lambda: synth.banded(5000, 40), "uniform": lambda: synth.uniform(3000, 3000, 9, seed=2)}[gen]()
    A = synth.attach_values(A, seed=3, dtype=dtype)
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype=dtype, build_bfs=0)
    for d in (0.002, 0.05, 0.5):
        xi, xv = synth.sample_x(A.n, max(1, synth.density_k(A.n, d)), seed=11, dtype=dtype)
        yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
        check_spmspv(C, yi, yv, xi, xv, dtype=dtype)
    # all-ones x on the Laplacian: cancellation zeros stay in y (R1)
    if gen == "stencil2d" and dtype == "f64":
        A0 = synth.stencil2d(70, 45)
        M0 = tsmv.TiledMatrix.from_csr(A0.to(DEV), build_bfs=0)
        xi = torch.arange(A0.n, dtype=torch.int32)
        yi, yv = M0.spmspv(xi.to(DEV), torch.ones(A0.n, dtype=torch.float64, device=DEV))
        check_spmspv(oracle.csc_of(A0), yi, yv, xi, torch.ones(A0.n, dtype=torch.float64), exact=True)
        M0.close()
    M.close()


@pytest.mark.parametrize("semiring", ["or_and", "min_second"])
def test_rows_semirings(tsmv, rows_forced, semiring):
    A = synth.attach_values(synth.stencil3d(20), seed=5)
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), build_bfs=0)
    xi, xv = synth.sample_x(A.n, 600, seed=2)
    yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV), semiring=semiring)
    check_spmspv(C, yi, yv, xi, xv, semiring={"or_and": oracle.OR_AND, "min_second": oracle.MIN_SECOND}[semiring])
    M.close()


@pytest.mark.parametrize("shape", [(1000, 3000), (3000, 1000), (17, 5000), (4099, 4099)])
def test_rows_ragged_rectangular(tsmv, rows_forced, shape):
    m, n = shape
    A = synth.attach_values(synth.uniform(m, n, 6, seed=3), seed=4)
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), build_bfs=0)
    for d in (0.01, 0.3):
        xi, xv = synth.sample_x(n, max(1, synth.density_k(n, d)), seed=6)
        yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
        check_spmspv(C, yi, yv, xi, xv)
    M.close()


def test_rows_errors_keep_workspace_clean(tsmv, rows_forced):
    A = synth.attach_values(synth.stencil2d(40, 40), seed=1)
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), build_bfs=0)
    for xi in (torch.tensor([5, 5], dtype=torch.int32), torch.tensor([A.n], dtype=torch.int32)):
        with pytest.raises(tsmv.TsmvError):
            M.spmspv(xi.to(DEV), torch.ones(xi.numel(), dtype=torch.float64, device=DEV))
    xi, xv = synth.sample_x(A.n, 300, seed=2)
    yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
    check_spmspv(C, yi, yv, xi, xv)
    M.close()


def test_density_switch_choice(tsmv):
    """Which kernel tsmv_spmspv runs (read from the call statistics: the row-driven
    kernel visits every dense tile): C1 (small) and a 3D stencil at 10 % go
    row-driven; a 3D stencil at 1 %, R-MAT (side-matrix heavy) and a dense band go
    column-driven; row_driven_density = 0 switches the row kernel off."""
    def tiles_visited(A, d, **opt):
        M = tsmv.TiledMatrix.from_csr(A.to(DEV), build_bfs=0, **opt)
        xi, xv = synth.sample_x(A.n, max(1, synth.density_k(A.n, d)), seed=1)
        M.spmspv(xi.to(DEV), xv.to(DEV))
        st, info = M.last_call_stats(), M.info()
        M.close()
        return st["tile_items"], info["n_dense_tiles"]
    for A, d, rows in ((synth.stencil2d(64, 64), 0.01, True), (synth.stencil3d(48), 0.1, True),
                       (synth.stencil3d(128), 0.01, False), (synth.rmat(14, 16, seed=1), 0.1, False),
                       (synth.banded(1 << 14, 64), 0.1, False)):
        items, T = tiles_visited(synth.attach_values(A, seed=1), d)
        assert (items == T) == rows, (A.name, d, items, T)
    items, T = tiles_visited(synth.attach_values(synth.stencil2d(64, 64), seed=1), 0.01, row_driven_density=0.0)
    assert items < T
