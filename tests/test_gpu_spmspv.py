"""GPU parity of tsmv_spmspv (through the C ABI) against the CPU oracle
(Algorithm 2) on seeded synthetic inputs: the BASELINE configs,
tile sizes x extraction thresholds x semirings, ragged/edge cases, errors."""
import numpy as np
import pytest
import torch

import oracle
import synth
from parity import abs_csc, check_spmspv

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


@pytest.fixture(scope="module")
def tsmv():
    from paper_conf_icpp_jisl0t022_b200 import tsmv as t
    return t


def _mk(tsmv, A, dtype="f64", **opts):
    Ad = A.to(DEV)
    return tsmv.TiledMatrix.from_csr(Ad, dtype=dtype, **opts)


def test_c1_laplacian_fp64(tsmv):
    A = synth.stencil2d(64, 64)
    C = oracle.csc_of(A)
    M = _mk(tsmv, A)
    for seed in (1, 2, 3):
        xi, xv = synth.sample_x(A.n, 41, seed=seed)
        yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
        check_spmspv(C, yi, yv, xi, xv)
    # all-ones x: interior rows cancel to exactly 0 and must be present (R1)
    xi = torch.arange(A.n, dtype=torch.int32)
    yi, yv = M.spmspv(xi.to(DEV), torch.ones(A.n, dtype=torch.float64, device=DEV))
    check_spmspv(C, yi, yv, xi, torch.ones(A.n, dtype=torch.float64), exact=True)
    assert yi.numel() == A.n


@pytest.mark.parametrize("nt", [16, 32, 64])
@pytest.mark.parametrize("thr", [0, 2, 8])
def test_tiles_thresholds_integer_exact(tsmv, nt, thr):
    A = synth.attach_values(synth.rmat(12, 16, seed=4), seed=2, integer=True)
    C = oracle.csc_of(A)
    M = _mk(tsmv, A, tile_dim=nt, sparse_tile_max_nnz=thr)
    info = M.info()
    assert (info["n_tiles"], info["n_dense_tiles"], info["side_nnz"]) == \
        oracle.tile_census(A.m, A.n, A.row_ptr, A.col_idx, nt, thr)
    for d in (0.001, 0.01, 0.1, 1.0):
        xi, xv = synth.sample_x(A.n, max(1, synth.density_k(A.n, d)), seed=7, integer=True)
        yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
        check_spmspv(C, yi, yv, xi, xv, exact=True)


@pytest.mark.parametrize("dtype", ["f64", "f32"])
@pytest.mark.parametrize("density", [0.0001, 0.001, 0.01, 0.1])
def test_c2_rmat_s20_sweep(tsmv, dtype, density, rmat20):
    A, C, Cabs = rmat20[dtype]
    M = rmat20["M_" + dtype]
    xi, xv = synth.sample_x(A.n, synth.density_k(A.n, density), seed=1, dtype=dtype)
    yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
    check_spmspv(C, yi, yv, xi, xv, dtype=dtype, Cabs=Cabs)


@pytest.fixture(scope="module")
def rmat20(tsmv):
    base = synth.rmat(20, 16, seed=1, device=DEV).to("cpu")
    out = {}
    for dt in ("f64", "f32"):
        A = synth.attach_values(base, seed=1, dtype=dt)
        C = oracle.csc_of(A)
        out[dt] = (A, C, abs_csc(C))
        out["M_" + dt] = _mk(tsmv, A, dtype=dt)
    return out


@pytest.mark.parametrize("semiring", ["or_and", "min_second"])
@pytest.mark.parametrize("dtype", ["f64", "f32", "pattern"])
def test_semirings(tsmv, semiring, dtype):
    A = synth.attach_values(synth.rmat(11, 8, seed=9), seed=3, dtype="f32" if dtype == "f32" else "f64")
    C = oracle.csc_of(A)
    M = _mk(tsmv, A, dtype=dtype)
    sr = {"or_and": oracle.OR_AND, "min_second": oracle.MIN_SECOND}[semiring]
    vdt = torch.float32 if dtype == "f32" else torch.float64
    for d in (0.01, 0.3):
        xi, _ = synth.sample_x(A.n, synth.density_k(A.n, d), seed=5)
        xv = (xi.to(torch.float64) * 0.5 - 77.0).to(vdt)   # signed values exercise the ordered-key min
        yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV), semiring=semiring)
        check_spmspv(C, yi, yv, xi, xv, semiring=sr, dtype="f32" if dtype == "f32" else "f64")


def test_pattern_plus_times_counts(tsmv):
    A = synth.rmat(11, 8, seed=2)
    C = oracle.csc_of(A)
    M = _mk(tsmv, A, dtype="pattern")
    xi, _ = synth.sample_x(A.n, 200, seed=3)
    xv = torch.ones(xi.numel(), dtype=torch.float64)
    yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
    check_spmspv(C, yi, yv, xi, xv, exact=True)


@pytest.mark.parametrize("shape", [(1, 1), (1000, 1000), (4097, 4097), (300, 5000), (5000, 300), (17, 33)])
def test_ragged_and_rectangular(tsmv, shape):
    m, n = shape
    A = synth.attach_values(synth.uniform(m, n, 3, seed=m + n), seed=4)
    C = oracle.csc_of(A)
    for nt in (16, 64):
        M = _mk(tsmv, A, tile_dim=nt)
        for k in sorted({0, 1, max(1, n // 10), n}):
            xi, xv = synth.sample_x(n, k, seed=k + 1)
            yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
            check_spmspv(C, yi, yv, xi, xv)


def test_empty_rows_and_columns(tsmv):
    D = torch.zeros(70, 90, dtype=torch.float64)
    D[3, 5] = 2.0
    D[3, 80] = -1.0
    D[64, 5] = 4.0
    D[69, 89] = 8.0
    A = synth.from_dense_pattern(D)
    C = oracle.csc_of(A)
    M = _mk(tsmv, A)
    for idx in ([5], [80, 89], [0, 1, 2], list(range(90))):
        xi = torch.tensor(idx, dtype=torch.int32)
        xv = torch.arange(1, len(idx) + 1, dtype=torch.float64)
        yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
        check_spmspv(C, yi, yv, xi, xv, exact=True)


def test_errors_keep_workspace_clean(tsmv):
    A = synth.attach_values(synth.rmat(10, 8, seed=1), seed=1)
    C = oracle.csc_of(A)
    M = _mk(tsmv, A)
    # duplicates (also unsorted ones), out of range (R21: any order of unique indices is valid)
    bad = [torch.tensor([5, 5], dtype=torch.int32), torch.tensor([9, 3, 9], dtype=torch.int32),
           torch.tensor([A.n], dtype=torch.int32), torch.tensor([-1], dtype=torch.int32)]
    for xi in bad:
        with pytest.raises(tsmv.TsmvError) as e:
            M.spmspv(xi.to(DEV), torch.ones(xi.numel(), dtype=torch.float64, device=DEV))
        assert e.value.status == tsmv.EINVAL
    xi = torch.tensor([9, 3], dtype=torch.int32)                    # unsorted, unique: accepted
    yi, yv = M.spmspv(xi.to(DEV), torch.ones(2, dtype=torch.float64, device=DEV))
    check_spmspv(C, yi, yv, torch.tensor([3, 9]), torch.ones(2, dtype=torch.float64))
    xi, xv = synth.sample_x(A.n, 100, seed=2)
    yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
    check_spmspv(C, yi, yv, xi, xv)
    # capacity
    ri, _ = oracle.spmspv(C, xi.numpy(), xv.numpy())
    with pytest.raises(tsmv.TsmvError) as e:
        M.spmspv(xi.to(DEV), xv.to(DEV), y_idx=torch.empty(3, dtype=torch.int32, device=DEV),
                 y_val=torch.empty(3, dtype=torch.float64, device=DEV))
    assert e.value.status == tsmv.ECAPACITY
    yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))   # still clean afterwards
    check_spmspv(C, yi, yv, xi, xv)
    assert yi.numel() == ri.size


@pytest.mark.parametrize("mode", ["phase_c_copy", "copy_kernel", "direct"])
def test_host_buffers_e2e(tsmv, mode, monkeypatch):
    """Host x / y through the synchronous C ABI: pinned (zero-copy x; y copied by each
    CTA of the flat kernel's phase C once its pieces are emitted, by the r2 copy
    kernel with TSMV_Y_COPY_KERNEL=1, or written by the compaction itself with
    TSMV_Y_DIRECT=1) and pageable."""
    if mode == "direct":
        monkeypatch.setenv("TSMV_Y_DIRECT", "1")
    if mode == "copy_kernel":
        monkeypatch.setenv("TSMV_Y_COPY_KERNEL", "1")
    A = synth.attach_values(synth.rmat(12, 16, seed=3), seed=3)
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A)   # host CSR -> deep copy to device
    xi, xv = synth.sample_x(A.n, 400, seed=8)
    yi, yv = M.spmspv(xi.pin_memory(), xv.pin_memory())   # host x and host y
    assert yi.device.type == "cpu"
    check_spmspv(C, yi, yv, xi, xv)
    yi2, yv2 = M.spmspv(xi, xv)                             # pageable host
    assert torch.equal(yi, yi2)                             # values: atomic order may differ
    check_spmspv(C, yi2, yv2, xi, xv)


def test_builder_round_trip(tsmv):
    for A in (synth.attach_values(synth.rmat(11, 16, seed=5), seed=1), synth.stencil2d(40, 40),
              synth.attach_values(synth.uniform(333, 1234, 7, seed=2), seed=2, dtype="f32")):
        for nt, thr in ((16, 2), (32, 0), (64, 8)):
            M = _mk(tsmv, A, dtype="f32" if A.values.dtype == torch.float32 else "f64", tile_dim=nt,
                    sparse_tile_max_nnz=thr)
            rp, ci, v = M.export_csr()
            assert torch.equal(rp, A.row_ptr) and torch.equal(ci, A.col_idx) and torch.equal(v, A.values)


def test_builder_rejects_bad_csr(tsmv):
    rp = torch.tensor([0, 2, 3], dtype=torch.int64)
    ci = torch.tensor([1, 1, 0], dtype=torch.int32)        # duplicate column in row 0
    with pytest.raises(tsmv.TsmvError):
        tsmv.TiledMatrix(2, 2, rp.to(DEV), ci.to(DEV), None, dtype="pattern")
    ci = torch.tensor([0, 2, 0], dtype=torch.int32)        # out of range
    with pytest.raises(tsmv.TsmvError):
        tsmv.TiledMatrix(2, 2, rp.to(DEV), ci.to(DEV), None, dtype="pattern")


@pytest.mark.slow
def test_target_rmat_s22_full(tsmv):
    """Config T (north_star roofline target): R-MAT s22 @ 1 %, fp64, full compare."""
    base = synth.rmat(22, 16, seed=1, device=DEV)
    A = synth.attach_values(base, seed=1).to("cpu")
    C = oracle.csc_of(A)
    M = _mk(tsmv, A)
    xi, xv = synth.sample_x(A.n, synth.density_k(A.n, 0.01), seed=1)
    yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
    check_spmspv(C, yi, yv, xi, xv)


@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_pinned_host_buffers_zero_copy(dtype):
    """Pinned host x is read in place by the kernel and pinned host y is filled by
    the device-sized copy kernel; pageable host buffers go through staging.  All
    three must equal the device-resident call: the index set exactly, the values to
    the summation-order tolerance (fp64 atomics commit in any order; positive
    values, no cancellation)."""
    from paper_conf_icpp_jisl0t022_b200 import tsmv
    A = synth.attach_values(synth.rmat(14, 16, seed=9), seed=2, dtype=dtype)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype=dtype)
    xi, xv = synth.sample_x(A.n, synth.density_k(A.n, 0.02), seed=5, dtype=dtype)
    di, dv = M.spmspv(xi.to(DEV), xv.to(DEV))
    di, dv = di.cpu(), dv.cpu()
    vt = dv.dtype
    tol = 1e-12 if dtype == "f64" else 1e-6

    def same(yi, yv):
        return torch.equal(yi, di) and torch.allclose(yv, dv, rtol=tol, atol=0.0)

    # pinned, 16-byte aligned
    pi, pv = xi.pin_memory(), xv.pin_memory()
    hyi, hyv = torch.empty(A.m, dtype=torch.int32).pin_memory(), torch.empty(A.m, dtype=vt).pin_memory()
    yi, yv = M.spmspv(pi, pv, y_idx=hyi, y_val=hyv)
    assert same(yi, yv)
    # pinned but not 16-byte aligned outputs (offset views)
    big_i, big_v = torch.empty(A.m + 3, dtype=torch.int32).pin_memory(), torch.empty(A.m + 3, dtype=vt).pin_memory()
    yi, yv = M.spmspv(pi, pv, y_idx=big_i[1:], y_val=big_v[3:])
    assert same(yi, yv)
    # pageable
    yi, yv = M.spmspv(xi.clone(), xv.clone(), y_idx=torch.empty(A.m, dtype=torch.int32),
                      y_val=torch.empty(A.m, dtype=vt))
    assert same(yi, yv)
    # capacity error reports the size
    with pytest.raises(tsmv.TsmvError):
        M.spmspv(pi, pv, y_idx=hyi[:5], y_val=hyv[:5])
    M.close()


def test_permuted_rmat_spmspv(tsmv):
    A = synth.attach_values(synth.rmat(13, 16, seed=8, permute=True), seed=3)
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV))
    for d in (0.001, 0.01, 0.1):
        xi, xv = synth.sample_x(A.n, synth.density_k(A.n, d), seed=4)
        yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
        check_spmspv(C, yi, yv, xi, xv, Cabs=abs_csc(C))
    M.close()


def test_opt_in_l2_window(tsmv, monkeypatch):
    """TSMV_PERSIST=1 (opt-in since r2 session 5): the accumulator's persisting
    L2 window changes no result; two contexts alive at once, then destroyed."""
    monkeypatch.setenv("TSMV_PERSIST", "1")
    A = synth.attach_values(synth.rmat(13, 16, seed=4), seed=4)
    C = oracle.csc_of(A)
    Ms = [tsmv.TiledMatrix.from_csr(A.to(DEV), build_bfs=0) for _ in range(2)]
    for s, M in enumerate(Ms):
        xi, xv = synth.sample_x(A.n, 300, seed=30 + s)
        yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
        check_spmspv(C, yi, yv, xi, xv)
    for M in Ms:
        M.close()


@pytest.mark.parametrize("semiring", ["plus_times", "or_and", "min_second"])
def test_hot_rows_opt_in(tsmv, monkeypatch, semiring):
    """TSMV_HOT=1 (opt-in since r2 session 5): the heaviest tile rows privatised in
    shared memory per CTA and flushed once per (CTA, row); integer-exact against
    the oracle on R-MAT (power-law rows) over densities, every semiring."""
    monkeypatch.setenv("TSMV_HOT", "1")
    A = synth.attach_values(synth.rmat(14, 16, seed=12), seed=3, integer=True)
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), build_bfs=0)
    sr = {"plus_times": oracle.PLUS_TIMES, "or_and": oracle.OR_AND, "min_second": oracle.MIN_SECOND}[semiring]
    for d in (0.001, 0.01, 0.1, 1.0):
        xi, xv = synth.sample_x(A.n, max(1, synth.density_k(A.n, d)), seed=5, integer=True)
        yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV), semiring=semiring)
        check_spmspv(C, yi, yv, xi, xv, semiring=sr, exact=True)
    M.close()
