"""Pins for the oracle's SpMSpV (Algorithm 2) against things other
than itself: dense brute force, scipy SpMV with x densified, unit vectors,
cancellation (structural y), integer exactness, Algorithm 1 (row-wise)."""
import numpy as np
import pytest
import scipy.sparse as sp
import torch

import oracle
import synth


def _scipy(A):
    vals = A.values.numpy() if A.values is not None else np.ones(A.nnz)
    return sp.csr_matrix((vals, A.col_idx.numpy(), A.row_ptr.numpy()), shape=(A.m, A.n))


def test_hash_matches_python_reference():
    c = torch.tensor([0, 1, 2, 12345, 2**40 + 7], dtype=torch.int64)
    h = synth.hash_u64(1, synth.S_RMAT, c)
    for ci, hi in zip(c.tolist(), h.tolist()):
        assert (hi & ((1 << 64) - 1)) == synth.hash_u64_ref(1, synth.S_RMAT, ci)


@pytest.mark.parametrize("m,n,seed", [(1, 1, 0), (7, 13, 1), (64, 40, 2), (200, 256, 3)])
def test_dense_bruteforce_integer(m, n, seed):
    rng = np.random.default_rng(seed)
    D = rng.integers(-9, 10, size=(m, n)) * (rng.random((m, n)) < 0.15)
    A = synth.from_dense_pattern(torch.from_numpy(D))
    k = max(1, n // 5)
    xi = np.sort(rng.choice(n, size=k, replace=False)).astype(np.int32)
    xv = rng.integers(1, 50, size=k).astype(np.float64) * rng.choice([-1, 1], size=k)
    yi, yv = oracle.spmspv(oracle.csc_of(A), xi, xv)
    xd = np.zeros(n)
    xd[xi] = xv
    ref = D.astype(np.float64) @ xd                      # dense brute force
    struct = (D[:, xi] != 0).any(axis=1)                 # structural pattern
    assert np.array_equal(yi, np.nonzero(struct)[0])
    assert np.array_equal(yv, ref[struct])               # integer -> exact


def test_scipy_spmv_densified_x_float():
    A = synth.attach_values(synth.rmat(10, 8, seed=3), seed=3)
    xi, xv = synth.sample_x(A.n, 60, seed=5)
    yi, yv = oracle.spmspv(oracle.csc_of(A), xi, xv)
    S = _scipy(A)
    xd = np.zeros(A.n)
    xd[xi.numpy()] = xv.numpy()
    ref = S @ xd
    pat = (S.astype(bool).astype(np.int64) @ (xd != 0).astype(np.int64)) > 0
    assert np.array_equal(yi, np.nonzero(pat)[0])
    absref = abs(S) @ abs(xd)
    assert np.all(np.abs(yv - ref[yi]) <= 1e-12 * absref[yi])


def test_unit_vector_gives_column():
    A = synth.attach_values(synth.uniform(300, 200, 6, seed=4), seed=9)
    S = _scipy(A).tocsc()
    for j in [0, 17, 199]:
        yi, yv = oracle.spmspv(oracle.csc_of(A), np.array([j], np.int32), np.array([1.0]))
        col = S[:, j]
        assert np.array_equal(yi, col.indices)
        assert np.array_equal(yv, col.data)


def test_laplacian_cancellation_is_structural():
    A = synth.stencil2d(8, 8)
    xi = np.arange(64, dtype=np.int32)
    yi, yv = oracle.spmspv(oracle.csc_of(A), xi, np.ones(64))
    assert np.array_equal(yi, np.arange(64))             # every row present
    inner = [i * 8 + j for i in range(1, 7) for j in range(1, 7)]
    assert np.all(yv[inner] == 0.0)                       # exact zeros kept
    assert yv[0] == 2.0                                   # corner: 4 - 2


def test_rectangular_not_transposed():
    D = np.zeros((3, 5))
    D[2, 4] = 7.0
    D[0, 1] = 3.0
    A = synth.from_dense_pattern(torch.from_numpy(D))
    yi, yv = oracle.spmspv(oracle.csc_of(A), np.array([4], np.int32), np.array([2.0]))
    assert yi.tolist() == [2] and yv.tolist() == [14.0]


def test_alg1_rowwise_equals_alg2():
    """Algorithm 1 (row-wise, matrix-driven) written here as a plain
    loop must give the same y as the oracle's Algorithm 2."""
    A = synth.attach_values(synth.rmat(8, 8, seed=7), seed=1, integer=True)
    xi, xv = synth.sample_x(A.n, 40, seed=2, integer=True)
    xd = {int(i): float(v) for i, v in zip(xi, xv)}
    rp, ci, va = A.row_ptr.numpy(), A.col_idx.numpy(), A.values.numpy()
    ref_i, ref_v = [], []
    for i in range(A.m):
        yi_, hit = 0.0, False
        for p in range(rp[i], rp[i + 1]):
            if int(ci[p]) in xd:                          # "if x_j != 0"
                yi_ += va[p] * xd[int(ci[p])]
                hit = True
        if hit:
            ref_i.append(i)
            ref_v.append(yi_)
    yi, yv = oracle.spmspv(oracle.csc_of(A), xi, xv)
    assert yi.tolist() == ref_i and yv.tolist() == ref_v


def test_or_and_is_boolean_product():
    A = synth.rmat(9, 8, seed=11)
    xi, _ = synth.sample_x(A.n, 30, seed=3)
    yi, yv = oracle.spmspv(oracle.csc_of(A), xi, None, oracle.OR_AND)
    S = _scipy(A).astype(bool)
    xd = np.zeros(A.n, bool)
    xd[xi.numpy()] = True
    pat = (S.astype(np.int64) @ xd.astype(np.int64)) > 0
    assert np.array_equal(yi, np.nonzero(pat)[0])
    assert np.all(yv == 1.0)


def test_min_second_bruteforce():
    rng = np.random.default_rng(4)
    D = (rng.random((50, 60)) < 0.1).astype(np.float64) * rng.integers(1, 9, (50, 60))
    A = synth.from_dense_pattern(torch.from_numpy(D))
    xi = np.sort(rng.choice(60, 25, replace=False)).astype(np.int32)
    xv = rng.normal(size=25)
    yi, yv = oracle.spmspv(oracle.csc_of(A), xi, xv, oracle.MIN_SECOND)
    ref_i, ref_v = [], []
    for i in range(50):
        cand = [xv[e] for e, j in enumerate(xi) if D[i, j] != 0]
        if cand:
            ref_i.append(i)
            ref_v.append(min(cand))
    assert yi.tolist() == ref_i and yv.tolist() == ref_v


def test_min_second_parent_ids():
    """MIN_SECOND with x_j = j gives the minimum-id in-neighbour (BFS parent)."""
    A = synth.from_edges(6, [(0, 1), (0, 2), (1, 3), (2, 3), (3, 4)])
    xi = np.array([1, 2], np.int32)
    yi, yv = oracle.spmspv(oracle.csc_of(A), xi, xi.astype(np.float64), oracle.MIN_SECOND)
    assert yi.tolist() == [0, 3] and yv.tolist() == [1.0, 1.0]


def test_empty_and_invalid():
    A = synth.stencil2d(4, 4)
    C = oracle.csc_of(A)
    yi, yv = oracle.spmspv(C, np.zeros(0, np.int32), np.zeros(0))
    assert yi.size == 0
    with pytest.raises(ValueError):
        oracle.spmspv(C, np.array([3, 3], np.int32), np.ones(2))
    with pytest.raises(ValueError):
        oracle.spmspv(C, np.array([16], np.int32), np.ones(1))
    # unsorted input is accepted (oracle sorts); output ascending
    yi2, yv2 = oracle.spmspv(C, np.array([9, 2], np.int32), np.array([1.0, 2.0]))
    yi3, yv3 = oracle.spmspv(C, np.array([2, 9], np.int32), np.array([2.0, 1.0]))
    assert np.array_equal(yi2, yi3) and np.array_equal(yv2, yv3)
