"""GPU parity of tsmv_msbfs (multi-source TileBFS): for every
source s, column s of the vertex-major level matrix must equal the oracle's queue
BFS from s, bit for bit (levels are unique); stats are checked against the
oracle's reached counts and the R16 edge count."""
import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


@pytest.fixture(scope="module")
def tsmv():
    from paper_conf_icpp_jisl0t022_b200 import tsmv as t
    return t


def _check(tsmv, A, sources, **opts):
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype="pattern", **opts)
    lv, st = M.msbfs(sources)
    got = lv.cpu().numpy()
    assert got.shape == (A.n, len(sources))
    outdeg = np.diff(C.col_ptr)
    pairs = edges = 0
    maxl = 0
    for s_i, s in enumerate(sources):
        ref = oracle.bfs_queue(C, s)
        assert np.array_equal(got[:, s_i], ref), f"source {s}: {np.sum(got[:, s_i] != ref)} levels differ"
        pairs += int((ref >= 0).sum())
        edges += int(outdeg[ref >= 0].sum())
        maxl = max(maxl, int(ref.max()) + 1)
    assert st["pairs_reached"] == pairs
    assert st["edges_traversed"] == edges
    assert st["nlevels"] == maxl
    M.close()


@pytest.mark.parametrize("nsrc", [1, 7, 64])
def test_msbfs_rmat_sym(tsmv, nsrc):
    A = synth.rmat(12, 16, seed=3, symmetrize=True)
    src = ([0] + synth.sample_sources(A, nsrc - 1, seed=7))[:nsrc]
    _check(tsmv, A, src)


def test_msbfs_rmat_directed_uses_in_edges(tsmv):
    A = synth.rmat(12, 16, seed=4)
    _check(tsmv, A, [0] + synth.sample_sources(A, 40, seed=2))


@pytest.mark.parametrize("thr", [0, 8])
def test_msbfs_side_threshold_and_repeats(tsmv, thr):
    A = synth.rmat(11, 16, seed=5, symmetrize=True)
    src = synth.sample_sources(A, 20, seed=3)
    _check(tsmv, A, src + src[:3] + [0], sparse_tile_max_nnz=thr)   # repeated sources allowed


def test_msbfs_stencils_and_band(tsmv):
    _check(tsmv, synth.stencil2d(64, 64).with_values(None), [0, 4095, 2080, 63])
    _check(tsmv, synth.stencil3d(20).with_values(None), list(range(0, 8000, 125)))
    _check(tsmv, synth.banded(3001, 7).with_values(None), [0, 3000, 1500])


def test_msbfs_rejects(tsmv):
    A = synth.stencil2d(16, 16).with_values(None)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype="pattern")
    with pytest.raises(tsmv.TsmvError):
        M.msbfs(list(range(65)))
    with pytest.raises(tsmv.TsmvError):
        M.msbfs([A.n])
    M.close()
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype="pattern", tile_dim=32)
    with pytest.raises(tsmv.TsmvError):
        M.msbfs([0])
    M.close()
