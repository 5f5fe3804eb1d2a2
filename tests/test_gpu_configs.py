"""BASELINE.json configs at their full sizes, through the C ABI, in the launch
configuration bench.py uses: parity against closed forms and the oracle.

  C1  2D 5-point 64x64, fp64, x 1 %, BFS from 0         (test_gpu_spmspv / test_gpu_bfs)
  C2  R-MAT s20 ef16 sweep 0.01..10 %, fp64 + fp32        (test_gpu_spmspv::test_c2_*)
  C3  TileBFS on R-MAT s22 (push/pull switching)          (here: every source level-exact)
  C4  3D 7-point 256^3 and banded (2^20, b=64): TileBFS levels == closed forms (every vertex),
      SpMSpV at 1 % == oracle (every entry)
  C5  R-MAT s26 on one GPU at full size: test_gpu_bench_configs.py::test_c5_s26; the
      partitioned path: test_gpu_dist_sim.py (simulated ranks), test_dist_gloo.py (CPU, gloo)."""
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


def test_c4_3d_stencil_256(tsmv):
    k = 256
    A = synth.stencil3d(k, device=DEV)
    M = tsmv.TiledMatrix.from_csr(A)                      # fp64 context with BFS tiles
    lv, st = M.bfs(0)
    v = torch.arange(k ** 3, device=DEV, dtype=torch.int64)
    closed = (v // (k * k) + (v // k) % k + v % k).to(torch.int32)
    assert torch.equal(lv, closed)
    assert st["nlevels"] == 3 * (k - 1) + 1
    # SpMSpV at 1 % on the same context, full compare with the oracle
    Ah = A.to("cpu")
    C = oracle.csc_of(Ah)
    xi, xv = synth.sample_x(A.n, synth.density_k(A.n, 0.01), seed=4)
    yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
    check_spmspv(C, yi, yv, xi, xv)
    M.close()


def test_c4_banded(tsmv):
    n, b = 1 << 20, 64
    A = synth.banded(n, b, device=DEV)
    M = tsmv.TiledMatrix.from_csr(A)
    lv, st = M.bfs(0)
    v = torch.arange(n, device=DEV, dtype=torch.int64)
    assert torch.equal(lv, ((v + b - 1) // b).to(torch.int32))
    assert st["nlevels"] == (n - 1 + b - 1) // b + 1
    Ah = A.to("cpu")
    C = oracle.csc_of(Ah)
    xi, xv = synth.sample_x(n, synth.density_k(n, 0.01), seed=6)
    yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
    check_spmspv(C, yi, yv, xi, xv)
    M.close()


def test_c3_rmat_s22_sources(tsmv):
    A = synth.rmat(22, 16, seed=1, symmetrize=True, device=DEV)
    M = tsmv.TiledMatrix.from_csr(A, dtype="pattern")
    Ah = A.to("cpu")
    C = oracle.csc_of(Ah)
    for s in [0] + synth.sample_sources(Ah, 3, seed=1):
        lv, st = M.bfs(s)
        ref = oracle.bfs_queue(C, s)
        assert np.array_equal(lv.cpu().numpy(), ref)
        assert "pull_csc" in st["dirs"]                   # direction switching exercised
    M.close()


def test_t_rmat_s22_fp32_and_semirings(tsmv):
    """Config T (roofline target) in fp32 and the Boolean / min semirings, full compare."""
    base = synth.rmat(22, 16, seed=1, device=DEV)
    A = synth.attach_values(base, seed=1, dtype="f32").to("cpu")
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype="f32", build_bfs=0)
    xi, xv = synth.sample_x(A.n, synth.density_k(A.n, 0.01), seed=2, dtype="f32")
    yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
    check_spmspv(C, yi, yv, xi, xv, dtype="f32", Cabs=abs_csc(C))
    yi, _ = M.spmspv(xi.to(DEV), None, semiring="or_and")
    check_spmspv(C, yi, None, xi, None, semiring=oracle.OR_AND)
    yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV), semiring="min_second")
    check_spmspv(C, yi, yv, xi, xv, semiring=oracle.MIN_SECOND, dtype="f32")
    M.close()


def test_c3_rmat_s22_parents_and_multisource(tsmv):
    """C3 at full size with the library default threshold (thr = 2): min-id BFS
    parents (MIN_SECOND, NEXT-2) against the oracle's Alg 3 over MIN_SECOND, and
    the 64-source TileBFS (NEXT-3) against the queue BFS on sampled source
    columns.  The bench's own contexts (thr = 8, all sources, all 64 columns) are
    checked in test_gpu_bench_configs.py."""
    A = synth.rmat(22, 16, seed=1, symmetrize=True, device=DEV)
    M = tsmv.TiledMatrix.from_csr(A, dtype="pattern")
    Ah = A.to("cpu")
    C = oracle.csc_of(Ah)
    lv, _ = M.bfs(0)
    par = M.bfs_parents(lv).cpu().numpy()
    rl, rp = oracle.bfs_parents(C, 0)
    assert np.array_equal(lv.cpu().numpy(), rl)
    assert np.array_equal(par, rp)
    src = [0] + synth.sample_sources(Ah, 63, seed=2)
    mlv, st = M.msbfs(src)
    got = mlv.cpu().numpy()
    for i in (0, 17, 63):
        assert np.array_equal(got[:, i], oracle.bfs_queue(C, src[i])), f"source column {i}"
    assert st["pairs_reached"] == int((got >= 0).sum())
    M.close()
