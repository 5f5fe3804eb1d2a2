"""Simulated ranks on one GPU: P libtsmv contexts built from the row blocks of
`dist.partition_rows`, with the exchange done by concatenation (what the NCCL
all-gather returns).  Exercises the distributed C-ABI calls
(tsmv_bfs_dist_begin/expand/merge, row_splits contexts) against the oracle."""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_icpp_jisl0t022_b200 import dist as D

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


def _ranks(A, P, dtype="pattern", **opts):
    splits = D.partition_rows(A.row_ptr, P)
    engines = []
    for r in range(P):
        Al = D.local_rows(A, splits, r).to(DEV)
        if dtype == "pattern":
            Al = Al.with_values(None)
        engines.append(D.DistTiledMatrix(Al, splits, r, P, dtype=dtype, **opts))
    # no process group: the caller hands every rank the global out-degrees
    deg = sum(D.DistTiledMatrix.column_counts(D.local_rows(A, splits, r)).to(torch.int64) for r in range(P))
    for e in engines:
        e.set_degrees(deg.to(torch.int32))
    return splits, engines


def _level_stats(A, lv):
    """(|F|, m_f, m_u) of every level from the oracle's levels: F = vertices of the
    level, m_f = their out-degrees (column counts), m_u = in-degrees (row lengths)
    of the vertices still unvisited after it (Alg 3's direction statistics)."""
    outdeg = np.bincount(A.col_idx.numpy(), minlength=A.n)
    indeg = np.diff(A.row_ptr.numpy())
    out = []
    for L in range(int(lv.max()) + 1):
        fr = lv == L
        unv = (lv < 0) | (lv > L)
        out.append((int(fr.sum()), int(outdeg[fr].sum()), int(indeg[unv].sum())))
    return out


def _sim_bfs(engines, source, dev_stats=False, expect=None):
    st = [e.begin(source) for e in engines]
    level = 0
    fprev = 0
    while sum(s[0] for s in st) > 0:
        # every rank returns its shares over its own rows; the sums are the global numbers
        f = sum(s[0] for s in st)
        mf = sum(s[1] for s in st)
        mu = sum(s[2] for s in st)
        if expect is not None:
            assert (f, mf, mu) == expect[level], level
        level += 1
        d = engines[0].choose(engines[0].n, f, mf, mu, fprev)
        fprev = f
        nnz = sum(e.M.nnz for e in engines)
        owned = [e.expand(d, wide=mu * 4 < nnz).clone() for e in engines]   # late-pull hint as bfs_loop
        stride = engines[0].stride
        gathered = torch.zeros(len(engines) * stride, dtype=torch.int32, device=DEV)
        for p, o in enumerate(owned):
            gathered[p * stride:p * stride + o.numel()] = o
        if dev_stats:   # merge with device statistics (tsmv_bfs_dist_merge, device out_stats)
            st = [tuple(int(x) for x in e.merge_dev(gathered, stride).clone().cpu()) for e in engines]
        else:
            st = [e.merge(gathered, stride) for e in engines]
    return np.concatenate([e.levels[:e.m_local].cpu().numpy() for e in engines])


@pytest.mark.parametrize("P", [2, 3, 4])
@pytest.mark.parametrize("sym", [True, False])
def test_sim_ranks_bfs(P, sym):
    A = synth.rmat(13, 16, seed=7, symmetrize=sym)
    C = oracle.csc_of(A)
    _, engines = _ranks(A, P)
    for s in [0] + synth.sample_sources(A, 2, seed=2):
        ref = oracle.bfs_queue(C, s)
        assert np.array_equal(_sim_bfs(engines, s, expect=_level_stats(A, ref)), ref)


@pytest.mark.parametrize("force", [1, 2, 3])
def test_sim_ranks_forced_directions(force):
    A = synth.stencil2d(64, 64)
    C = oracle.csc_of(A)
    _, engines = _ranks(A, 3, force_dir=force)
    assert np.array_equal(_sim_bfs(engines, 0), oracle.bfs_queue(C, 0))


@pytest.mark.parametrize("P", [2, 4])
def test_sim_ranks_spmspv(P):
    A = synth.attach_values(synth.rmat(13, 16, seed=3), seed=2, integer=True)
    C = oracle.csc_of(A)
    splits, engines = _ranks(A, P, dtype="f64")
    xi, xv = synth.sample_x(A.n, 500, seed=5, integer=True)
    ys_i, ys_v = [], []
    for e in engines:
        yi, yv = e.M.spmspv(xi.to(DEV), xv.to(DEV))     # the all-gathered x
        ys_i.append(yi.cpu().numpy())
        ys_v.append(yv.cpu().numpy())
    ri, rv = oracle.spmspv(C, xi.numpy(), xv.numpy())
    assert np.array_equal(np.concatenate(ys_i), ri)      # global row ids, ascending across ranks
    assert np.array_equal(np.concatenate(ys_v), rv)


@pytest.mark.parametrize("P", [2, 3])
def test_sim_ranks_bfs_device_stats(P):
    """The device-statistics merge gives the same levels (and |F| on every rank)."""
    A = synth.rmat(12, 16, seed=11, symmetrize=True)
    C = oracle.csc_of(A)
    _, engines = _ranks(A, P)
    for s in [0] + synth.sample_sources(A, 2, seed=5):
        got = _sim_bfs(engines, s, dev_stats=True)
        assert np.array_equal(got, oracle.bfs_queue(C, s))


@pytest.mark.parametrize("P", [2, 3])
def test_sim_ranks_dist_spmspv_owned_x(P, monkeypatch):
    """DistTiledMatrix.spmspv / spmspv_async with per-owner x slices (one rank owns
    no entry): the size and entry all-gathers are replaced by concatenation, so
    the owner filter, the exchange glue and the local multiply are all checked."""
    A = synth.attach_values(synth.rmat(12, 16, seed=4), seed=3)
    C = oracle.csc_of(A)
    splits, engines = _ranks(A, P, dtype="f64")
    xi, xv = synth.sample_x(A.n, 300, seed=8)
    lo_empty, hi_empty = splits[1], splits[2]          # rank 1 owns no x entry
    keep = (xi < lo_empty) | (xi >= hi_empty)
    xi, xv = xi[keep], xv[keep]
    owned = [((xi >= splits[r]) & (xi < splits[r + 1])) for r in range(P)]
    parts_i = [xi[o].to(DEV) for o in owned]
    parts_v = [xv[o].to(DEV) for o in owned]
    sizes = [int(p.numel()) for p in parts_i]
    assert sizes[1] == 0
    monkeypatch.setattr(D, "allgather_sizes", lambda count, device, group=None: sizes)

    def varlen(t, group=None, sizes=None):
        src = parts_i if t.dtype == torch.int32 else parts_v
        return torch.cat([p.to(t.dtype) for p in src])
    monkeypatch.setattr(D, "allgather_varlen", varlen)
    ri, rv = oracle.spmspv(C, xi.numpy(), xv.numpy())
    gi, gv, ai, av = [], [], [], []
    for r, e in enumerate(engines):
        yi, yv = e.spmspv(parts_i[r].to(torch.int32), parts_v[r])
        gi.append(yi.cpu().numpy())
        gv.append(yv.cpu().numpy())
        y_i = torch.empty(e.m_local, dtype=torch.int32, device=DEV)
        y_v = torch.empty(e.m_local, dtype=torch.float64, device=DEV)
        y_n = torch.zeros(1, dtype=torch.int64, device=DEV)
        e.spmspv_async(parts_i[r].to(torch.int32), parts_v[r], y_i, y_v, y_n)
        k = int(y_n.item())
        ai.append(y_i[:k].cpu().numpy())
        av.append(y_v[:k].cpu().numpy())
    for I, V in ((gi, gv), (ai, av)):
        assert np.array_equal(np.concatenate(I), ri)
        assert np.allclose(np.concatenate(V), rv, rtol=1e-12, atol=0)


def test_sim_ranks_bulk_push(monkeypatch):
    """Heavy Push-CSC levels of the per-level kernels in bulk mode (k_push ORs into
    the next frontier, k_bulk_fix takes new = Fn & ~V over the owned words):
    forced push on simulated ranks, with and without it."""
    A = synth.rmat(13, 16, seed=17, symmetrize=True)
    C = oracle.csc_of(A)
    _, engines = _ranks(A, 3, force_dir=1)
    for s in [0] + synth.sample_sources(A, 2, seed=9):
        ref = oracle.bfs_queue(C, s)
        assert np.array_equal(_sim_bfs(engines, s, expect=_level_stats(A, ref)), ref)
        monkeypatch.setenv("TSMV_BFS_NO_BULK", "1")
        assert np.array_equal(_sim_bfs(engines, s), ref)
        monkeypatch.delenv("TSMV_BFS_NO_BULK")
