"""Full-size oracle parity for exactly the configurations bench.py times
(VERDICT r1 "next 1"): the same generators, seeds, contexts (tile size,
very-sparse threshold, dtype) and sources, read from bench.py's own defaults.

  C3  TileBFS on R-MAT s22 symmetrised, pattern, thr = bench --bfs-thr: every
      timed source's levels, the min-id parents, all 64 multi-source columns
  T   SpMSpV at R-MAT s22 1 % (the bench's timed step is also checked inside
      bench.py, "parity")
  relabelled s22: SpMSpV 1 % and TileBFS (bench configs["rmat_s22_permuted"])
  C5  R-MAT s26 on one GPU: SpMSpV 1 % (every y entry) and TileBFS from vertex 0
      (every level) against the oracle on the host (~1-2 min, 196 GB host RAM)
  queue overflow of the fused list levels (TSMV_BFS_QCAP) on high-diameter graphs."""
import os

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


@pytest.fixture(autouse=True)
def _memory_report():
    torch.cuda.empty_cache()
    print("\n[mem] free GiB at test start", round(torch.cuda.mem_get_info()[0] / 2**30, 1),
          "torch allocated", round(torch.cuda.memory_allocated() / 2**30, 2))
    yield


@pytest.fixture(scope="module")
def cfg():
    import bench
    return bench.parse([])


def test_c3_bench_bfs_context_all_sources(tsmv, cfg):
    import bench
    A = synth.rmat(cfg.bfs_scale, 16, seed=1, symmetrize=True, device=DEV)
    M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", tile_dim=cfg.tile_dim, sparse_tile_max_nnz=cfg.bfs_thr)
    Ah = A.to("cpu")
    C = oracle.csc_of(Ah)
    srcs = bench.bfs_sources(A, cfg.bfs_sources)
    assert len(srcs) == cfg.bfs_sources == 16
    lv = torch.empty(A.n, dtype=torch.int32, device=DEV)
    for s in srcs:
        _, st = M.bfs(s, levels=lv)
        ref = oracle.bfs_queue(C, s)
        assert np.array_equal(lv.cpu().numpy(), ref), f"source {s}"
        assert st["reached"] == int((ref >= 0).sum())
    # min-id parents of the last traversal (bench: parents of the last source)
    par = M.bfs_parents(lv).cpu().numpy()
    rl, rp = oracle.bfs_parents(C, srcs[-1])
    assert np.array_equal(lv.cpu().numpy(), rl)
    assert np.array_equal(par, rp)
    # all 64 columns of the bench's multi-source traversal
    src = [0] + synth.sample_sources(A, 63, seed=2)
    mlv, st = M.msbfs(src)
    got = mlv.cpu().numpy()
    for i in range(64):
        assert np.array_equal(got[:, i], oracle.bfs_queue(C, src[i])), f"source column {i}"
    assert st["pairs_reached"] == int((got >= 0).sum())
    M.close()


def test_t_bench_context(tsmv, cfg):
    import bench
    A = bench.make_matrix(cfg.scale, cfg.dtype, DEV)
    M = tsmv.TiledMatrix.from_csr(A, dtype=cfg.dtype, tile_dim=cfg.tile_dim, sparse_tile_max_nnz=cfg.thr,
                                  build_bfs=0)
    C = oracle.csc_of(A.to("cpu"))
    Cabs = abs_csc(C)
    k = synth.density_k(A.n, cfg.density)
    for xi, xv in bench.x_samples(A.n, k, 3, cfg.dtype, DEV):
        yi, yv = M.spmspv(xi, xv)
        check_spmspv(C, yi, yv, xi, xv, Cabs=Cabs)
    M.close()


def test_relabelled_s22_bench_configs(tsmv, cfg):
    A = synth.attach_values(synth.rmat(22, 16, seed=1, device=DEV, permute=True), seed=1)
    M = tsmv.TiledMatrix.from_csr(A, build_bfs=0)
    C = oracle.csc_of(A.to("cpu"))
    k = synth.density_k(A.n, 0.01)
    xi, xv = synth.sample_x(A.n, k, seed=3, device=DEV)
    yi, yv = M.spmspv(xi, xv)
    check_spmspv(C, yi, yv, xi, xv)
    M.close()
    del A, C
    A = synth.rmat(22, 16, seed=1, symmetrize=True, device=DEV, permute=True)
    M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", sparse_tile_max_nnz=cfg.bfs_thr)
    C = oracle.csc_of(A.to("cpu"))
    for s in [synth.sample_sources(A, 1, seed=1)[0], 0]:
        lv, _ = M.bfs(s)
        assert np.array_equal(lv.cpu().numpy(), oracle.bfs_queue(C, s))
    M.close()


@pytest.mark.slow
def test_c5_s26(tsmv, cfg):
    """C5 at full size on one GPU, every output against the oracle on the host."""
    A = synth.attach_values(synth.rmat(26, 16, seed=1, device=DEV), seed=1)
    M = tsmv.TiledMatrix.from_csr(A, build_bfs=0)
    k = synth.density_k(A.n, 0.01)
    xi, xv = synth.sample_x(A.n, k, seed=1, device=DEV)
    yi, yv = M.spmspv(xi, xv)
    yi, yv = yi.cpu(), yv.cpu()
    M.close()
    Ah = A.to("cpu")
    del A
    torch.cuda.empty_cache()
    C = oracle.csc_of(Ah)
    del Ah
    check_spmspv(C, yi, yv, xi, xv)
    del C
    A = synth.rmat(26, 16, seed=1, symmetrize=True, device=DEV)
    torch.cuda.empty_cache()
    print("free GiB before the symmetric build", torch.cuda.mem_get_info()[0] / 2**30,
          "torch allocated GiB", torch.cuda.memory_allocated() / 2**30)
    M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", tile_dim=cfg.tile_dim, sparse_tile_max_nnz=cfg.bfs_thr)
    lv, st = M.bfs(0)
    lv = lv.cpu().numpy()
    M.close()
    Ah = A.to("cpu")
    del A
    torch.cuda.empty_cache()
    C = oracle.csc_of(Ah)
    del Ah
    ref = oracle.bfs_queue(C, 0)
    assert np.array_equal(lv, ref)
    assert st["reached"] == int((ref >= 0).sum())


@pytest.mark.parametrize("qcap", ["1", "16"])
def test_list_level_queue_overflow(tsmv, qcap):
    """The fused kernel's per-CTA discovery queue spills to the global list when
    full; a small usable capacity (TSMV_BFS_QCAP) forces that path on every level."""
    os.environ["TSMV_BFS_QCAP"] = qcap
    try:
        k = 48
        A = synth.stencil3d(k, device=DEV)
        M = tsmv.TiledMatrix.from_csr(A, dtype="pattern")
        lv, _ = M.bfs(0)
        v = torch.arange(k ** 3, device=DEV)
        assert torch.equal(lv, (v // (k * k) + (v // k) % k + v % k).to(torch.int32))
        M.close()
        n, b = 1 << 16, 32
        A = synth.banded(n, b, device=DEV)
        M = tsmv.TiledMatrix.from_csr(A, dtype="pattern")
        lv, _ = M.bfs(0)
        v = torch.arange(n, device=DEV)
        assert torch.equal(lv, ((v + b - 1) // b).to(torch.int32))
        M.close()
        A = synth.rmat(16, 16, seed=1, symmetrize=True)
        C = oracle.csc_of(A)
        M = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype="pattern", sparse_tile_max_nnz=8)
        for s in [0] + synth.sample_sources(A, 2, seed=4):
            lv, _ = M.bfs(s)
            assert np.array_equal(lv.cpu().numpy(), oracle.bfs_queue(C, s))
        M.close()
    finally:
        os.environ.pop("TSMV_BFS_QCAP")
