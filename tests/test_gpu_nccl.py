"""The distributed path with the context's OWN communicator,
on one GPU: a one-rank NCCL communicator made from tsmv_nccl_unique_id, so
tsmv_bfs / tsmv_spmspv run their collective level loop / x exchange inside
libtsmv.so (in-place frontier broadcasts, count all-gather + x broadcasts,
global-degree statistics) and must give the oracle's results.  Several ranks
need several GPUs; their kernels are covered rank by rank in test_gpu_dist_sim.py."""
import numpy as np
import pytest
import torch

import oracle
import synth
from parity import check_spmspv

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


@pytest.fixture(scope="module")
def tsmv():
    from paper_conf_icpp_jisl0t022_b200 import tsmv as t
    return t


def _comm_ctx(tsmv, A, **kw):
    return tsmv.TiledMatrix.from_csr(A, rank=0, nranks=1, nccl_unique_id=tsmv.nccl_unique_id(), **kw)


@pytest.mark.parametrize("sym", [True, False])
def test_one_rank_comm_bfs(tsmv, sym):
    A = synth.rmat(14, 16, seed=5, symmetrize=sym)
    C = oracle.csc_of(A)
    Mc = _comm_ctx(tsmv, A.to(DEV), dtype="pattern")
    Ms = tsmv.TiledMatrix.from_csr(A.to(DEV), dtype="pattern")
    for s in [0] + synth.sample_sources(A, 3, seed=6):
        lc, sc = Mc.bfs(s)
        ls, ss = Ms.bfs(s)
        ref = oracle.bfs_queue(C, s)
        assert np.array_equal(lc.cpu().numpy(), ref)
        assert (sc["nlevels"], sc["reached"], sc["edges_traversed"]) == \
            (ss["nlevels"], ss["reached"], ss["edges_traversed"])
        assert len(sc["level_ms"]) == sc["nlevels"]
    Mc.close()
    Ms.close()


def test_one_rank_comm_forced_directions(tsmv):
    A = synth.stencil2d(48, 40)
    C = oracle.csc_of(A)
    for d in (1, 2, 3):
        M = _comm_ctx(tsmv, A.to(DEV), dtype="pattern", force_dir=d)
        lv, _ = M.bfs(7)
        assert np.array_equal(lv.cpu().numpy(), oracle.bfs_queue(C, 7))
        M.close()


@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_one_rank_comm_spmspv(tsmv, dtype):
    A = synth.attach_values(synth.rmat(13, 16, seed=2), seed=4, dtype=dtype)
    C = oracle.csc_of(A)
    M = _comm_ctx(tsmv, A.to(DEV), dtype=dtype, build_bfs=0)
    for d in (0.001, 0.05):
        xi, xv = synth.sample_x(A.n, synth.density_k(A.n, d), seed=9, dtype=dtype)
        yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
        check_spmspv(C, yi, yv, xi, xv, dtype=dtype)
        yi, yv = M.spmspv(xi, xv)                          # host x: staged for NCCL
        check_spmspv(C, yi, yv, xi, xv, dtype=dtype)
    yi, yv = M.spmspv(torch.zeros(0, dtype=torch.int32, device=DEV), torch.zeros(0, device=DEV))
    assert yi.numel() == 0
    M.close()


def test_dist_matrix_bootstrap_one_rank(tsmv):
    from paper_conf_icpp_jisl0t022_b200 import dist as D
    A = synth.rmat(12, 16, seed=3, symmetrize=True)
    C = oracle.csc_of(A)
    splits = D.partition_rows(A.row_ptr, 1)
    Dm = D.DistMatrix(D.local_rows(A, splits, 0).to(DEV), splits, 0, 1, tsmv.nccl_unique_id(), dtype="pattern")
    lv, st = Dm.bfs(0)
    assert np.array_equal(lv.cpu().numpy(), oracle.bfs_queue(C, 0))
    Dm.close()


def test_unsorted_x_any_order(tsmv):
    """Reading R21 (round 2): x may come in any order of unique indices; duplicates
    and out-of-range indices are rejected and leave the context usable."""
    A = synth.attach_values(synth.rmat(13, 16, seed=6), seed=1)
    C = oracle.csc_of(A)
    M = tsmv.TiledMatrix.from_csr(A.to(DEV), build_bfs=0)
    xi, xv = synth.sample_x(A.n, 800, seed=3)
    perm = torch.randperm(xi.numel(), generator=torch.Generator().manual_seed(1))
    for sr in ("plus_times", "min_second", "or_and"):
        yi, yv = M.spmspv(xi[perm].to(DEV), xv[perm].to(DEV), semiring=sr)
        check_spmspv(C, yi, yv, xi, xv, semiring={"plus_times": 0, "or_and": 1, "min_second": 2}[sr])
    dup = torch.cat([xi[:5], xi[:1]])
    with pytest.raises(tsmv.TsmvError) as e:
        M.spmspv(dup.to(DEV), torch.ones(6, dtype=torch.float64, device=DEV))
    assert e.value.status == tsmv.EINVAL
    yi, yv = M.spmspv(xi.to(DEV), xv.to(DEV))
    check_spmspv(C, yi, yv, xi, xv)
    M.close()
