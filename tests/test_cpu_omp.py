"""The OpenMP CPU speed baseline (cpu_omp/, timed by bench.py beside the oracle)
computes what the oracle computes: same y index set, values within the fp64
parity bar (its summation order differs), bit-exact BFS levels."""
import numpy as np
import pytest

import cpu_omp
import oracle
import synth


@pytest.mark.parametrize("threads", [1, 3, 0])
def test_spmspv_matches_oracle(threads):
    A = synth.attach_values(synth.rmat(13, 16, seed=2), seed=2)
    C = oracle.csc_of(A)
    Co = cpu_omp.csc_of(A)
    Ca = oracle.CSC(C.m, C.n, C.col_ptr, C.row_idx, np.abs(C.val))
    for d in (0.0005, 0.01, 0.2):
        xi, xv = synth.sample_x(A.n, synth.density_k(A.n, d), seed=5)
        ri, rv = oracle.spmspv(C, xi.numpy(), xv.numpy())
        gi, gv = cpu_omp.spmspv(Co, xi.numpy(), xv.numpy(), nthreads=threads)
        assert np.array_equal(gi, ri)
        _, mag = oracle.spmspv(Ca, xi.numpy(), np.abs(xv.numpy()))
        assert np.all(np.abs(gv - rv) <= 1e-12 * mag)


def test_spmspv_cancellation_and_empty():
    A = synth.stencil2d(16, 16)
    Co, C = cpu_omp.csc_of(A), oracle.csc_of(A)
    xi = np.arange(256, dtype=np.int32)
    xv = np.ones(256)
    gi, gv = cpu_omp.spmspv(Co, xi, xv)
    ri, rv = oracle.spmspv(C, xi, xv)
    assert np.array_equal(gi, ri) and np.allclose(gv, rv, atol=1e-12)
    gi, _ = cpu_omp.spmspv(Co, np.zeros(0, np.int32), np.zeros(0))
    assert gi.size == 0


@pytest.mark.parametrize("gen", ["rmat_sym", "rmat_dir", "grid"])
def test_bfs_matches_oracle(gen):
    A = {"rmat_sym": lambda: synth.rmat(13, 16, seed=1, symmetrize=True),
         "rmat_dir": lambda: synth.rmat(12, 16, seed=4),
         "grid": lambda: synth.stencil2d(40, 30)}[gen]()
    C, Co = oracle.csc_of(A), cpu_omp.csc_of(A)
    for s in [0] + synth.sample_sources(A, 3, seed=2):
        assert np.array_equal(cpu_omp.bfs(Co, s), oracle.bfs_queue(C, s))
