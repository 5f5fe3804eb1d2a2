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
