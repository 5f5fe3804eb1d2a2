"""2D-partitioned TileBFS (DESIGN.md §8 "2D") on simulated
ranks of one GPU: every rank's block in its own libtsmv context, the exchanges by
concatenation (what the collectives return).  Levels bit-exact against the
oracle's queue BFS; the three 2D kernels against their plain definitions."""
import ctypes

import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_icpp_jisl0t022_b200 import dist2d as D2

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


@pytest.fixture(scope="module")
def tsmv():
    from paper_conf_icpp_jisl0t022_b200 import tsmv as t
    return t


def _engines(A, Pr, Pc, balance="rows", **opts):
    g = D2.Grid2D(A.n, Pr, Pc, row_ptr=A.row_ptr, balance=balance)
    Ad = A.to(DEV)
    E = [D2.Dist2DBFS(D2.block_2d(Ad, g, *g.coords(r)), g, r, **opts) for r in range(g.P)]
    D2.sim_degrees(Ad, E)
    return g, E


def _level_stats(A, lv):
    """(|F|, m_f, m_u) per level from the oracle's levels (Alg 3's statistics)."""
    outdeg = np.bincount(A.col_idx.numpy(), minlength=A.n)
    indeg = np.diff(A.row_ptr.numpy())
    out = []
    for L in range(int(lv.max()) + 1):
        fr = lv == L
        unv = (lv < 0) | (lv > L)
        out.append((int(fr.sum()), int(outdeg[fr].sum()), int(indeg[unv].sum())))
    return out


@pytest.mark.parametrize("Pr,Pc", [(1, 1), (1, 2), (2, 1), (2, 2), (2, 3), (3, 2)])
@pytest.mark.parametrize("sym", [True, False])
@pytest.mark.parametrize("mode", ["dopt", "push"])
def test_bfs2d_levels(Pr, Pc, sym, mode):
    A = synth.rmat(12, 16, seed=9, symmetrize=sym)
    C = oracle.csc_of(A)
    g, E = _engines(A, Pr, Pc, balance="nnz" if sym else "rows", mode=mode)
    for s in [0] + synth.sample_sources(A, 2, seed=4):
        trace = []
        nl = D2.sim_bfs2d(E, s, trace=trace)
        ref = oracle.bfs_queue(C, s)
        got = D2.gather_levels(E).cpu().numpy()
        assert np.array_equal(got, ref), f"{Pr}x{Pc} src {s}: {np.sum(got != ref)} levels differ"
        assert nl == int(ref.max()) + 1
        # summed statistics shares = Alg 3's |F| of every level after the source's
        assert [t["f"] for t in trace] == [x[0] for x in _level_stats(A, ref)[1:]] + [0]
    for e in E:
        e.close()


@pytest.mark.parametrize("force", [1, 2, 3])
def test_bfs2d_forced_directions(force):
    """Every direction kernel on the blocks alone (force_dir), directed R-MAT."""
    A = synth.rmat(12, 16, seed=2)
    C = oracle.csc_of(A)
    g, E = _engines(A, 2, 3, force_dir=force)
    for s in [0] + synth.sample_sources(A, 2, seed=8):
        D2.sim_bfs2d(E, s)
        assert np.array_equal(D2.gather_levels(E).cpu().numpy(), oracle.bfs_queue(C, s))
    for e in E:
        e.close()


def test_bfs2d_stencil_closed_form():
    """2D 5-point grid: level(64 i + j) = i + j from vertex 0 (closed form)."""
    A = synth.stencil2d(64, 64)
    g, E = _engines(A, 2, 2)
    D2.sim_bfs2d(E, 0)
    got = D2.gather_levels(E).cpu().numpy()
    v = np.arange(64 * 64)
    assert np.array_equal(got, v // 64 + v % 64)
    for e in E:
        e.close()


def test_bfs2d_kernels(tsmv):
    """scatter / merge / list against their plain definitions (ragged sizes)."""
    M = tsmv.TiledMatrix.from_csr(synth.stencil2d(8, 8).to(DEV), dtype="pattern", build_bfs=0)
    rng = np.random.default_rng(5)
    st = torch.cuda.current_stream().cuda_stream
    # list: bitmap -> ascending ids
    for nbits in (1, 31, 32, 33, 4095, 4096 * 8 + 17, 300000):
        nw = (nbits + 31) // 32
        bits = rng.random(nw * 32) < 0.07
        bits[nbits:] = False
        w = torch.from_numpy(np.packbits(bits, bitorder="little").view("<u4").view(np.int32).copy()).to(DEV)
        out = torch.empty(nbits, dtype=torch.int32, device=DEV)
        k = ctypes.c_int64(-1)
        tsmv.check(tsmv.tsmv_bfs2d_list(M.ctx, w.data_ptr(), nbits, out.data_ptr(), ctypes.byref(k), st))
        assert np.array_equal(out[:k.value].cpu().numpy(), np.nonzero(bits)[0])
    # scatter: ids -> bitmap (y_nnz on the device, clipped at y_cap)
    ids = np.sort(rng.choice(64, 20, replace=False)).astype(np.int32)
    yi = torch.from_numpy(ids).to(DEV)
    yn = torch.tensor([20], dtype=torch.int64, device=DEV)
    words = torch.full((2,), -1, dtype=torch.int32, device=DEV)
    tsmv.check(tsmv.tsmv_bfs2d_scatter(M.ctx, yi.data_ptr(), yn.data_ptr(), 20, words.data_ptr(), 2, st))
    got = np.unpackbits(words.cpu().numpy().view(np.uint8), bitorder="little").astype(bool)
    ref = np.zeros(64, bool)
    ref[ids] = True
    assert np.array_equal(got, ref)
    # merge: OR of nseg partial bitmaps, minus visited, levels, count
    nverts, nseg, stride = 100, 3, 5
    segs = rng.integers(0, 2**32, size=nseg * stride, dtype=np.uint64).astype(np.uint32)
    vis = rng.integers(0, 2**32, size=stride, dtype=np.uint64).astype(np.uint32)
    lev = np.full(stride * 32, -1, np.int32)
    d_segs = torch.from_numpy(segs.view(np.int32).copy()).to(DEV)
    d_vis = torch.from_numpy(vis.view(np.int32).copy()).to(DEV)
    d_lev = torch.from_numpy(lev.copy()).to(DEV)
    d_front = torch.zeros(stride, dtype=torch.int32, device=DEV)
    d_cnt = torch.zeros(3, dtype=torch.int64, device=DEV)
    od = rng.integers(0, 1000, size=nverts).astype(np.int32)
    idg = rng.integers(0, 1000, size=nverts).astype(np.int32)
    d_od, d_id = torch.from_numpy(od).to(DEV), torch.from_numpy(idg).to(DEV)
    tsmv.check(tsmv.tsmv_bfs2d_merge(M.ctx, d_segs.data_ptr(), nseg, stride, nverts, d_vis.data_ptr(),
                                     d_lev.data_ptr(), 7, d_front.data_ptr(), d_od.data_ptr(), d_id.data_ptr(),
                                     d_cnt.data_ptr(), st))

    def unpack(a):
        return np.unpackbits(a.view(np.uint8), bitorder="little").astype(bool)
    orb = np.zeros(stride * 32, bool)
    for p in range(nseg):
        orb |= unpack(segs[p * stride:(p + 1) * stride])
    orb[nverts:] = False
    new = orb & ~unpack(vis)
    assert np.array_equal(unpack(d_front.cpu().numpy().view(np.uint32)), new)
    assert np.array_equal(unpack(d_vis.cpu().numpy().view(np.uint32)), unpack(vis) | new)
    ref_lev = lev.copy()
    ref_lev[new] = 7
    assert np.array_equal(d_lev.cpu().numpy(), ref_lev)
    nv = new[:nverts]
    assert d_cnt.cpu().tolist() == [int(nv.sum()), int(od[nv].sum()), int(idg[nv].sum())]
    M.close()
