"""Pins for the oracle's tiled structures: Figure 3 tiled vector,
tile census vs brute force and Table 2 monotonicity, and the
Figure 5 bitmask words (tests/golden/fig5_bfs_trace.json)."""
import json
import os

import numpy as np
import pytest

import oracle
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def test_fig3_tiled_vector():
    g = json.load(open(os.path.join(GOLD, "fig3_tiled_vector.json")))
    x_ptr, x_tile = oracle.tile_vector(g["n"], g["nt"], np.array(g["x_idx"], np.int32),
                                       np.array(g["x_val"]))
    assert x_ptr.tolist() == g["x_ptr"]
    assert x_tile.size == g["x_tile_len"]
    nt = g["nt"]
    for i, v in zip(g["x_idx"], g["x_val"]):   # access formula (Alg 4 line 6)
        assert x_tile[x_ptr[i // nt] * nt + i % nt] == v
    # zeros inside non-empty tiles are stored as dense zeros
    assert np.count_nonzero(x_tile) == len(g["x_idx"])


def _census_bruteforce(A, nt, thr):
    rows = A.rows().numpy()
    cols = A.col_idx.numpy().astype(np.int64)
    tk = (rows // nt) * ((A.n + nt - 1) // nt) + cols // nt
    _, cnt = np.unique(tk, return_counts=True)
    return cnt.size, int((cnt > thr).sum()), int(cnt[cnt <= thr].sum())


@pytest.mark.parametrize("maker", [lambda: synth.rmat(10, 16, seed=1),
                                   lambda: synth.stencil2d(64, 64),
                                   lambda: synth.uniform(1000, 777, 5, seed=2),
                                   lambda: synth.banded(1000, 9)])
def test_tile_census(maker):
    A = maker()
    counts = {}
    for nt in (16, 32, 64):
        for thr in (0, 2, 8):
            got = oracle.tile_census(A.m, A.n, A.row_ptr, A.col_idx, nt, thr)
            assert got == _census_bruteforce(A, nt, thr)
            assert got[1] + 0 <= got[0]
        counts[nt] = got[0]
    # Table 2 monotonicity
    assert counts[16] >= counts[32] >= counts[64] >= counts[16] / 16


def test_stencil_tile_counts_closed_form():
    # 2D 64x64 5-point: tile row I (16 rows) touches tiles J in {I-4, I-1, I, I+1, I+4} clipped
    A = synth.stencil2d(64, 64)
    n_tiles, _, _ = oracle.tile_census(A.m, A.n, A.row_ptr, A.col_idx, 16, 0)
    expect = 0
    for I in range(256):
        rows = range(16 * I, 16 * I + 16)
        Js = set()
        for r in rows:
            i, j = divmod(r, 64)
            for (di, dj) in [(-1, 0), (0, -1), (0, 0), (0, 1), (1, 0)]:
                if 0 <= i + di < 64 and 0 <= j + dj < 64:
                    Js.add(((i + di) * 64 + j + dj) // 16)
        expect += len(Js)
    assert n_tiles == expect == 1144


def test_fig5_bitmask_words():
    g = json.load(open(os.path.join(GOLD, "fig5_bfs_trace.json")))
    A = synth.from_edges(g["n"], g["undirected_edges"])
    nt = g["nt"]
    A1 = oracle.bitmask_tiles(A.m, A.n, A.row_ptr, A.col_idx, nt, 0)
    A2 = oracle.bitmask_tiles(A.m, A.n, A.row_ptr, A.col_idx, nt, 1)
    assert len(A1) == len(A2) == g["non_empty_tiles"]
    # undirected: A1 and A2 hold the same arrays
    d1 = {(I, J): w for I, J, w in A1}
    d2 = {(J, I): w for I, J, w in A2}
    assert d1 == d2
    # Push-CSC, x1 = {0}: OR of column-0 words of tile column 0, per tile row
    y1 = [0] * (g["n"] // nt)
    for I, J, w in A1:
        if J == 0:
            y1[I] |= w[0]
    assert y1 == g["y1_push_csc"]
    m1 = g["x1"]
    x2 = [y & ~m & ((1 << nt) - 1) for y, m in zip(y1, m1)]
    assert x2 == g["x2"]
    assert [d2[(0, 0)][0], d2[(1, 0)][0]] == g["A2_row0_tiles_00_01"]
    col3 = [0] * (g["n"] // nt)
    for I, J, w in A1:
        if J == 0:
            col3[I] = w[3]
    assert col3 == g["A1_column3_words_by_tile_row"]
    assert g["x3_first_item"] == 1  # {0,0,0,1} = vertex 3 unvisited after level 2
