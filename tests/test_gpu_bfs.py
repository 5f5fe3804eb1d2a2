"""GPU parity of tsmv_bfs (TileBFS: Push-CSC / Push-CSR / Pull-CSC, Sec 3.4)
against the oracle's queue BFS: bit-exact int32 levels, for every forced
direction and the automatic rule, over tile sizes, thresholds, directed and
undirected graphs, and the BASELINE BFS configs."""
import json
import os

import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)
GOLD = os.path.join(os.path.dirname(__file__), "golden")
DIRS = [0, 1, 2, 3]   # auto, push_csc, push_csr, pull_csc


@pytest.fixture(scope="module")
def tsmv():
    from paper_conf_icpp_jisl0t022_b200 import tsmv as t
    return t


def _levels(tsmv, A, sources, dirs=DIRS, **opts):
    C = oracle.csc_of(A)
    Ad = A.to(DEV)
    for d in dirs:
        M = tsmv.TiledMatrix.from_csr(Ad, dtype="pattern", force_dir=d, **opts)
        for s in sources:
            lv, st = M.bfs(s)
            ref = oracle.bfs_queue(C, s)
            got = lv.cpu().numpy()
            assert np.array_equal(got, ref), f"dir={d} src={s}: {np.sum(got != ref)} levels differ"
            assert st["reached"] == int((ref >= 0).sum())
            assert st["nlevels"] == int(ref.max()) + 1
        M.close()


def test_c1_grid_closed_form(tsmv):
    A = synth.stencil2d(64, 64)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV))      # fp64 context also carries the BFS tiles
    lv, st = M.bfs(0)
    v = np.arange(4096)
    assert np.array_equal(lv.cpu().numpy(), v // 64 + v % 64)
    assert st["nlevels"] == 127
    _levels(tsmv, A, [0, 2080, 4095])


@pytest.mark.parametrize("nt", [16, 32, 64])
@pytest.mark.parametrize("thr", [0, 2, 8])
def test_rmat_sym_tiles(tsmv, nt, thr):
    A = synth.rmat(12, 16, seed=3, symmetrize=True)
    _levels(tsmv, A, synth.sample_sources(A, 2, seed=1) + [0], tile_dim=nt, sparse_tile_max_nnz=thr)


@pytest.mark.parametrize("nt", [16, 64])
def test_rmat_directed_pull_uses_in_edges(tsmv, nt):
    A = synth.rmat(12, 8, seed=6)        # directed: A != A^T
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype="pattern")
    assert M.info()["symmetric"] == 0
    _levels(tsmv, A, synth.sample_sources(A, 3, seed=4), tile_dim=nt)


def test_3d_and_band(tsmv):
    A = synth.stencil3d(16)
    _levels(tsmv, A, [0, 2000])
    B = synth.banded(4096, 8)
    M = tsmv.TiledMatrix.from_csr(B.to(DEV))
    lv, st = M.bfs(0)
    v = np.arange(4096)
    assert np.array_equal(lv.cpu().numpy(), (v + 7) // 8)
    _levels(tsmv, B, [100], dirs=[0, 1, 3])


def test_toys_and_ragged(tsmv):
    _levels(tsmv, synth.from_edges(5, [(0, 1), (1, 2), (2, 3), (3, 4)]), [0, 2])
    _levels(tsmv, synth.from_edges(6, [(0, 1), (2, 3)]), [0, 5])          # isolated source
    _levels(tsmv, synth.from_edges(3, [(1, 0), (2, 1)], symmetric=False), [0, 2])
    _levels(tsmv, synth.uniform(1000, 1000, 2, seed=3), [0, 999])        # n not a multiple of 32
    _levels(tsmv, synth.rmat(9, 4, seed=2, symmetrize=True), [0], tile_dim=64)
    _levels(tsmv, synth.from_edges(1, []) if False else synth.csr_from_keys(torch.tensor([0]), 1, 1), [0])


def test_fig5_graph_and_bitmasks(tsmv):
    g = json.load(open(os.path.join(GOLD, "fig5_bfs_trace.json")))
    A = synth.from_edges(g["n"], g["undirected_edges"])
    _levels(tsmv, A, [0])
    # bitmask tiles of the GPU builder == oracle's Sec 3.2.3 tiles (nt = 16 here)
    B = synth.rmat(8, 8, seed=1, symmetrize=True)
    for thr in (0, 2):
        M = tsmv.TiledMatrix.from_csr(B.to(DEV), dtype="pattern", sparse_tile_max_nnz=thr)
        for orient in (0, 1):
            got = M.export_bitmask_tiles(orient)
            ref = oracle.bitmask_tiles(B.m, B.n, B.row_ptr, B.col_idx, 16, orient, max_tiles=1 << 14)
            assert got == ref


def test_repeated_traversals_clean_state(tsmv):
    A = synth.rmat(13, 16, seed=8, symmetrize=True)
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype="pattern")
    for s in synth.sample_sources(A, 5, seed=9):
        lv, _ = M.bfs(s)
        assert np.array_equal(lv.cpu().numpy(), oracle.bfs_queue(C, s))
    host = torch.empty(A.n, dtype=torch.int32)
    lv, _ = M.bfs(0, levels=host)
    assert np.array_equal(host.numpy(), oracle.bfs_queue(C, 0))


def test_c3_rmat_s20_sym_directions(tsmv):
    A = synth.rmat(20, 16, seed=1, symmetrize=True, device=DEV).to("cpu")
    _levels(tsmv, A, [0] + synth.sample_sources(A, 1, seed=1))


@pytest.mark.slow
def test_c3_rmat_s22_sym(tsmv):
    A = synth.rmat(22, 16, seed=1, symmetrize=True, device=DEV).to("cpu")
    _levels(tsmv, A, [0], dirs=[0])


@pytest.mark.parametrize("nt", [16, 32, 64])
@pytest.mark.parametrize("sym", [True, False])
def test_bfs_parents_min_second(tsmv, nt, sym):
    """tsmv_bfs_parents == oracle_bfs_parents (Alg 3 over MIN_SECOND), bit-exact."""
    A = synth.rmat(12, 16, seed=3, symmetrize=sym)
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype="pattern", tile_dim=nt)
    for s in [0] + synth.sample_sources(A, 2, seed=4):
        lv, _ = M.bfs(s)
        par = M.bfs_parents(lv)
        rl, rp = oracle.bfs_parents(C, s)
        assert np.array_equal(lv.cpu().numpy(), rl)
        got = par.cpu().numpy()
        assert np.array_equal(got, rp), f"src={s}: {np.sum(got != rp)} parents differ"
    M.close()


def test_bfs_parents_grid_and_3d(tsmv):
    for A in (synth.stencil2d(64, 64), synth.stencil3d(24), synth.banded(3000, 7)):
        A = A.with_values(None)
        M = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype="pattern")
        lv, _ = M.bfs(0)
        got = M.bfs_parents(lv).cpu().numpy()
        _, rp = oracle.bfs_parents(oracle.csc_of(A), 0)
        assert np.array_equal(got, rp)
        M.close()


def test_permuted_rmat(tsmv):
    """Graph500-style relabelled R-MAT (hubs spread over the id space): levels,
    parents and multi-source levels still equal the oracle."""
    A = synth.rmat(12, 16, seed=6, symmetrize=True, permute=True)
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype="pattern")
    src = synth.sample_sources(A, 3, seed=1)
    for s in src:
        lv, _ = M.bfs(s)
        assert np.array_equal(lv.cpu().numpy(), oracle.bfs_queue(C, s))
        _, rp = oracle.bfs_parents(C, s)
        assert np.array_equal(M.bfs_parents(lv).cpu().numpy(), rp)
    mlv, _ = M.msbfs(src)
    for i, s in enumerate(src):
        assert np.array_equal(mlv[:, i].cpu().numpy(), oracle.bfs_queue(C, s))
    M.close()


@pytest.mark.parametrize("env", [None, "TSMV_BFS_HOSTLOOP"])
def test_path_longer_than_stats_arrays(tsmv, env):
    """A traversal with more levels than TSMV_MAX_LEVELS (the size of the stats
    arrays) runs to completion: path graph (band b = 1) of 70,000 vertices,
    level(v) = v (the fused loop used to stop at 65,536 levels)."""
    n = 70_000
    A = synth.banded(n, 1)
    if env:
        os.environ[env] = "1"
    try:
        M = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype="pattern")
        lv, st = M.bfs(0)
    finally:
        if env:
            os.environ.pop(env)
    assert np.array_equal(lv.cpu().numpy(), np.arange(n, dtype=np.int32))
    assert st["nlevels"] == n and st["reached"] == n
    assert len(st["dirs"]) == tsmv.MAX_LEVELS
    M.close()


def test_level_times(tsmv):
    """Per-level device times (Fig 10 analysis): one entry per level,
    non-negative, summing to about the traversal time."""
    A = synth.rmat(16, 16, seed=1, symmetrize=True, device=DEV)
    M = tsmv.TiledMatrix.from_csr(A, dtype="pattern")
    for s in [0] + synth.sample_sources(A.to("cpu"), 2, seed=3):
        _, st = M.bfs(s)
        t = st["level_ms"]
        assert len(t) == st["nlevels"] and all(x >= 0 for x in t)
        assert 0.5 * st["ms"] <= sum(t) <= 1.05 * st["ms"] + 0.01, (sum(t), st["ms"])
    M.close()


@pytest.mark.parametrize("host_min", [None, "1"])
@pytest.mark.parametrize("sym", [True, False])
def test_bulk_push_levels(tsmv, monkeypatch, sym, host_min):
    """Heavy Push-CSC levels (push items > n / 8) run in bulk mode (reductions into
    the next frontier, then one pass new = Fn & ~V): forced push on R-MAT makes
    every middle level heavy; levels equal the oracle's with and without it."""
    if host_min:  # (session 5) every bulk level handed to the host's k_push / k_bulk_fix
        monkeypatch.setenv("TSMV_BFS_BULK_HOST_MIN", host_min)
    A = synth.rmat(14, 16, seed=21, symmetrize=sym)
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype="pattern", force_dir=tsmv.DIR_PUSH_CSC, sparse_tile_max_nnz=8)
    for s in [0] + synth.sample_sources(A, 3, seed=6):
        ref = oracle.bfs_queue(C, s)
        lv, st = M.bfs(s)
        assert np.array_equal(lv.cpu().numpy(), ref)
        assert st["reached"] == int((ref >= 0).sum())
        monkeypatch.setenv("TSMV_BFS_NO_BULK", "1")
        lv2, _ = M.bfs(s)
        monkeypatch.delenv("TSMV_BFS_NO_BULK")
        assert np.array_equal(lv2.cpu().numpy(), ref)
    M.close()


@pytest.mark.parametrize("env", [{}, {"TSMV_PULL_ILP": "0"}, {"TSMV_PULL_ILP": "2"}, {"TSMV_PULL_ILP": "8"},
                                 {"TSMV_BFS_NO_RELIST": "1"}, {"TSMV_BFS_FULL_FSTATS": "1", "TSMV_BFS_HOST_DECIDE": "1"},
                                 {"TSMV_BFS_HOST_DECIDE": "1"}, {"TSMV_PULL_W": "32"}, {"TSMV_PULL_W": "16"},
                                 {"TSMV_PULL_W": "4"}])
def test_pull_side_claims_relist_stats(tsmv, monkeypatch, env):
    """R-MAT s18 (symmetrised, thr 8, as the bench's TileBFS): its explosive level
    is a dense pull level on the host kernels (side part: warp-aggregated claims,
    K vertices per thread) with the persistent kernel resumed right behind it (or,
    TSMV_BFS_HOST_DECIDE, the host deciding from the lite / full statistics pass),
    and the small push levels after the scan levels are converted back to list /
    solo levels.  Levels equal the oracle's for every variant, including the r2
    kernels."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    A = synth.rmat(18, 16, seed=1, symmetrize=True)
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype="pattern", sparse_tile_max_nnz=8)
    for s in [0] + synth.sample_sources(A, 3, seed=2):
        ref = oracle.bfs_queue(C, s)
        lv, st = M.bfs(s)
        assert np.array_equal(lv.cpu().numpy(), ref)
        assert "pull_csc" in st["dirs"]
        assert st["reached"] == int((ref >= 0).sum())
    M.close()


@pytest.mark.parametrize("nt", [16, 32, 64])
@pytest.mark.parametrize("relist", [True, False])
def test_relist_all_tile_sizes(tsmv, monkeypatch, nt, relist):
    """Scan levels converted back to list / solo levels (session 5) at every tile
    size (the frontier words are cleared per segment: 16-bit halves, 32-bit words,
    64-bit pairs), on and off, directed and symmetric R-MAT: levels equal the
    oracle's."""
    if not relist:
        monkeypatch.setenv("TSMV_BFS_NO_RELIST", "1")
    for sym in (True, False):
        A = synth.rmat(15, 16, seed=11, symmetrize=sym)
        C = oracle.csc_of(A)
        M = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype="pattern", tile_dim=nt, sparse_tile_max_nnz=8)
        for s in [0] + synth.sample_sources(A, 3, seed=9):
            ref = oracle.bfs_queue(C, s)
            lv, _ = M.bfs(s)
            assert np.array_equal(lv.cpu().numpy(), ref), (nt, relist, sym, s)
        M.close()
