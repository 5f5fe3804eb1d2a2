"""Pins for the oracle's BFS (queue BFS and Algorithm 3): closed forms
on stencils and bands, scipy shortest paths, Graph500 validation rules, toy
graphs and the Figure 5 trace (tests/golden/fig5_bfs_trace.json)."""
import json
import os

import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse.csgraph import shortest_path

import oracle
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _levels_both(A, s):
    C = oracle.csc_of(A)
    a = oracle.bfs_queue(C, s)
    b = oracle.bfs_alg3(C, s)
    assert np.array_equal(a, b)
    return a


def test_2d_closed_form():
    A = synth.stencil2d(64, 64)
    lv = _levels_both(A, 0)
    v = np.arange(4096)
    assert np.array_equal(lv, v // 64 + v % 64)
    assert lv.max() == 126


@pytest.mark.parametrize("k", [4, 8, 16])
def test_3d_closed_form(k):
    A = synth.stencil3d(k)
    lv = _levels_both(A, 0)
    v = np.arange(k ** 3)
    assert np.array_equal(lv, v // (k * k) + (v // k) % k + v % k)


@pytest.mark.parametrize("n,b", [(4096, 8), (1000, 7), (65, 64)])
def test_band_closed_form(n, b):
    A = synth.banded(n, b)
    lv = _levels_both(A, 0)
    v = np.arange(n)
    assert np.array_equal(lv, (v + b - 1) // b)


def _scipy_levels(A, s):
    S = sp.csr_matrix((np.ones(A.nnz), A.col_idx.numpy(), A.row_ptr.numpy()), shape=(A.m, A.n))
    # edge j -> i iff A[i, j] stored (y = A x); csgraph uses G[u, v] as u -> v
    d = shortest_path(S.T.tocsr(), unweighted=True, directed=True, indices=s)
    return np.where(np.isinf(d), -1, d).astype(np.int64)


@pytest.mark.parametrize("sym", [True, False])
def test_scipy_shortest_path(sym):
    A = synth.rmat(11, 8, seed=2, symmetrize=sym)
    for s in synth.sample_sources(A, 3, seed=1):
        assert np.array_equal(_levels_both(A, s), _scipy_levels(A, s))


def test_graph500_rules_directed():
    A = synth.rmat(12, 16, seed=5)
    s = synth.sample_sources(A, 1, seed=2)[0]
    lv = _levels_both(A, s).astype(np.int64)
    rows = A.rows().numpy()
    cols = A.col_idx.numpy().astype(np.int64)
    # edge cols -> rows
    src_reached = lv[cols] >= 0
    assert np.all(lv[rows][src_reached] >= 0)
    assert np.all(lv[rows][src_reached] <= lv[cols][src_reached] + 1)
    # every reached vertex at level L > 0 has an in-neighbour at level L-1
    good = np.zeros(A.n, bool)
    ok = (lv[cols] >= 0) & (lv[rows] == lv[cols] + 1)
    good[rows[ok]] = True
    need = lv > 0
    assert np.all(good[need])
    assert lv[s] == 0 and np.sum(lv == 0) == 1


def test_toys():
    path = synth.from_edges(5, [(0, 1), (1, 2), (2, 3), (3, 4)])
    assert _levels_both(path, 0).tolist() == [0, 1, 2, 3, 4]
    assert _levels_both(path, 2).tolist() == [2, 1, 0, 1, 2]
    star = synth.from_edges(6, [(0, i) for i in range(1, 6)])
    assert _levels_both(star, 3).tolist() == [1, 2, 2, 0, 2, 2]
    disc = synth.from_edges(6, [(0, 1), (2, 3)])
    assert _levels_both(disc, 0).tolist() == [0, 1, -1, -1, -1, -1]
    iso = synth.from_edges(3, [(1, 2)])
    assert _levels_both(iso, 0).tolist() == [0, -1, -1]
    # directed: A[1,0] stored = edge 0 -> 1 only
    d = synth.from_edges(3, [(1, 0), (2, 1)], symmetric=False)
    assert _levels_both(d, 0).tolist() == [0, 1, 2]
    assert _levels_both(d, 2).tolist() == [-1, -1, 0]


def test_fig5_levels():
    g = json.load(open(os.path.join(GOLD, "fig5_bfs_trace.json")))
    A = synth.from_edges(g["n"], g["undirected_edges"])
    lv = _levels_both(A, 0)
    for L, verts in enumerate(g["levels_sets"]):
        assert sorted(np.nonzero(lv == L)[0].tolist()) == verts


# ---------------------------------------------------------------- min-id parents (NEXT-2)
# oracle_bfs_parents follows Alg 3 over MIN_SECOND.
# Pins: closed forms (path, 2D grid), a hand-worked diamond, and -- on R-MAT,
# directed and symmetric -- the Graph500 parent rules plus minimality, checked
# from the CSR rows with numpy (no oracle code involved).

def _csr(n, edges):
    """A[v][u] = 1 for every edge u -> v (column u holds u's out-neighbours)."""
    r = np.array([v for u, v in edges], np.int64)
    c = np.array([u for u, v in edges], np.int64)
    M = sp.csr_matrix((np.ones(len(edges)), (r, c)), shape=(n, n))
    M.sum_duplicates()
    M.sort_indices()
    return synth.CSR(n, n, _t(M.indptr, "int64"), _t(M.indices, "int32"), None, "toy")


def _t(a, dt):
    import torch
    return torch.from_numpy(np.ascontiguousarray(a).astype(dt))


def test_parents_path_closed_form():
    n = 50
    A = _csr(n, [(i, i + 1) for i in range(n - 1)])
    lv, par = oracle.bfs_parents(oracle.csc_of(A), 0)
    assert np.array_equal(lv, np.arange(n))
    assert np.array_equal(par, np.r_[0, np.arange(n - 1)])


def test_parents_diamond_hand_worked():
    # 0 -> 2, 0 -> 1, 2 -> 3, 1 -> 3, 3 -> 4, 1 -> 4 ; 5 isolated
    A = _csr(6, [(0, 2), (0, 1), (2, 3), (1, 3), (3, 4), (1, 4)])
    lv, par = oracle.bfs_parents(oracle.csc_of(A), 0)
    assert lv.tolist() == [0, 1, 1, 2, 2, -1]
    # vertex 3: in-neighbours 1 and 2 on layer 1 -> 1; vertex 4: 1 (layer 1) beats 3 (layer 2)
    assert par.tolist() == [0, 0, 0, 1, 1, -1]


def test_parents_grid_closed_form():
    A = synth.stencil2d(64, 64)
    lv, par = oracle.bfs_parents(oracle.csc_of(A), 0)
    v = np.arange(4096)
    assert np.array_equal(lv, v // 64 + v % 64)
    want = np.where(v >= 64, v - 64, v - 1)
    want[0] = 0
    assert np.array_equal(par, want)


@pytest.mark.parametrize("sym", [True, False])
def test_parents_graph500_rules_and_minimal(sym):
    A = synth.rmat(10, 16, seed=5, symmetrize=sym)
    C = oracle.csc_of(A)
    for s in [0] + synth.sample_sources(A, 3, seed=2):
        lv, par = oracle.bfs_parents(C, s)
        assert np.array_equal(lv, oracle.bfs_queue(C, s))
        rp, ci = A.row_ptr.numpy(), A.col_idx.numpy()
        assert par[s] == s and np.all(par[lv < 0] == -1)
        for v in np.nonzero(lv > 0)[0]:
            ins = ci[rp[v]:rp[v + 1]]                      # u with A[v][u]: edges u -> v
            ok = ins[lv[ins] == lv[v] - 1]
            assert ok.size > 0 and par[v] == ok.min(), f"v={v}"
