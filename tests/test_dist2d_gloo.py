"""Host logic of the 2D-partitioned TileBFS (DESIGN.md §8
"2D"): the grid, the padded blocks, and the level loop `dist2d.bfs2d_loop` over
torch.distributed sub-groups (gloo, world size 4, CPU).  The per-rank compute is a
small numpy engine with the Dist2DBFS contract (the CUDA engine is covered by
test_gpu_dist2d.py on simulated ranks); levels are checked against the oracle."""
import os
import socket
import tempfile

import numpy as np
import pytest
import scipy.sparse as sp
import torch
import torch.distributed as tdist
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_icpp_jisl0t022_b200 import dist2d as D2

WORLD = 4


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_grid_shape():
    assert [D2.grid_shape(p) for p in (1, 2, 3, 4, 6, 8, 9, 16)] == \
        [(1, 1), (1, 2), (1, 3), (2, 2), (2, 3), (2, 4), (3, 3), (4, 4)]


@pytest.mark.parametrize("bal", ["rows", "nnz"])
def test_grid_pieces(bal):
    A = synth.rmat(12, 16, seed=2, symmetrize=True)
    g = D2.Grid2D(A.n, 2, 3, row_ptr=A.row_ptr, balance=bal)
    assert g.pieces[0] == 0 and g.pieces[-1] == A.n and len(g.pieces) == 7
    assert all(g.pieces[q] <= g.pieces[q + 1] for q in range(6))
    assert all(x % 64 == 0 for x in g.pieces[:-1])
    assert g.S % 64 == 0 and g.S >= max(g.pieces[q + 1] - g.pieces[q] for q in range(6))
    if bal == "nnz":
        rp = A.row_ptr.numpy()
        rows = [int(rp[g.pieces[3 * i + 3]] - rp[g.pieces[3 * i]]) for i in range(2)]
        assert max(rows) / (A.nnz / 2) < 1.1      # row blocks R_i nnz-balanced


def test_block_2d_reassembles_A():
    """The P blocks with their padded ids map back onto exactly the entries of A."""
    A = synth.rmat(11, 8, seed=3)
    rp, ci = A.row_ptr.numpy(), A.col_idx.numpy()
    ref = {(r, int(c)) for r in range(A.m) for c in ci[rp[r]:rp[r + 1]]}
    for Pr, Pc, bal in ((2, 2, "rows"), (2, 3, "nnz"), (1, 4, "rows"), (3, 1, "nnz")):
        g = D2.Grid2D(A.n, Pr, Pc, row_ptr=A.row_ptr, balance=bal)
        got = []
        for r in range(g.P):
            i, j = g.coords(r)
            B = D2.block_2d(A, g, i, j)
            assert B.m == Pc * g.S and B.n == Pr * g.S
            brp, bci = B.row_ptr.numpy(), B.col_idx.numpy()
            for lr in range(B.m):
                cols = bci[brp[lr]:brp[lr + 1]]
                assert np.all(np.diff(cols) > 0)
                sp_, off = divmod(lr, g.S)
                q = i * Pc + sp_
                for lc in cols:
                    pi, coff = divmod(int(lc), g.S)
                    qc = pi * Pc + j
                    assert off < g.pieces[q + 1] - g.pieces[q] and coff < g.pieces[qc + 1] - g.pieces[qc]
                    got.append((g.pieces[q] + off, g.pieces[qc] + coff))
        assert len(got) == len(ref) and set(got) == ref


def _pack(bits: np.ndarray) -> torch.Tensor:
    return torch.from_numpy(np.packbits(bits, bitorder="little").view("<u4").view(np.int32).copy())


def _unpack(words: torch.Tensor, count: int) -> np.ndarray:
    return np.unpackbits(words.numpy().view(np.uint8), bitorder="little")[:count].astype(bool)


class NumpyEngine2D:
    """Per-rank stand-in for Dist2DBFS: same begin / expand / merge contract."""

    needs_rows = True

    def __init__(self, A, grid, rank, comm):
        self.g, self.rank = grid, rank
        self.i, self.j = grid.coords(rank)
        B = D2.block_2d(A, grid, self.i, self.j)
        self.B = sp.csr_matrix((np.ones(B.nnz), B.col_idx.numpy(), B.row_ptr.numpy()), shape=(B.m, B.n))
        self.own0, p1 = grid.piece(rank)
        self.nown = p1 - self.own0
        od, idg, self.nnz_total = comm.degrees(B)     # the degree reductions under test
        self.outdeg, self.indeg = od.numpy(), idg.numpy()
        self.seen = []

    def choose(self, f, mf, mu, fprev=0):
        self.seen.append((f, mf, mu))
        return 1

    def begin(self, s):
        S = self.g.S
        self.visited = np.zeros(S, bool)
        self.vis_rows = np.zeros(self.g.Pc * S, bool)
        self.levels = np.full(self.nown, -1, np.int32)
        self.seen = []
        front = np.zeros(S, bool)
        st = [0, 0, 0]
        if self.own0 <= s < self.own0 + self.nown:
            o = s - self.own0
            front[o] = self.visited[o] = True
            self.levels[o] = 0
            st = [1, int(self.outdeg[o]), int(self.indeg[o])]
        self.stats = torch.tensor(st, dtype=torch.int64)
        return _pack(front)

    def expand(self, x_words, d, row_new, level):
        # row_new: R_i's new vertices, replicated over the processor row (masks y)
        self.vis_rows |= _unpack(row_new, self.g.Pc * self.g.S)
        x = _unpack(x_words, self.g.Pr * self.g.S)
        return _pack(((self.B @ x.astype(np.float64)) > 0) & ~self.vis_rows)

    def merge(self, recv, level):
        S = self.g.S
        allb = _unpack(recv, self.g.Pc * S).reshape(self.g.Pc, S)
        acc = allb.any(axis=0)
        acc[self.nown:] = False
        new = acc & ~self.visited
        self.visited |= new
        own = new[:self.nown]
        self.levels[own] = level
        st = [int(own.sum()), int(self.outdeg[own].sum()), int(self.indeg[own].sum())]
        return _pack(new), torch.tensor(st, dtype=torch.int64)


def _worker(rank, world, port, tmp, Pr, Pc, sym):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    tdist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A = synth.rmat(11, 8, seed=5, symmetrize=sym)
        g = D2.Grid2D(A.n, Pr, Pc, row_ptr=A.row_ptr, balance="nnz" if sym else "rows")
        comm = D2.TorchComm2D(g, rank)
        eng = NumpyEngine2D(A, g, rank, comm)
        srcs = [0] + synth.sample_sources(A, 2, seed=3)
        for s in srcs:
            nl = D2.bfs2d_loop(eng, s, comm)
            np.save(os.path.join(tmp, f"lv{rank}_{s}.npy"), eng.levels)
            np.save(os.path.join(tmp, f"nl{rank}_{s}.npy"), np.array([nl]))
            np.save(os.path.join(tmp, f"seen{rank}_{s}.npy"), np.array(eng.seen, dtype=np.int64))
        np.save(os.path.join(tmp, "srcs.npy"), np.array(srcs))
        tdist.barrier()
    finally:
        tdist.destroy_process_group()


@pytest.mark.parametrize("Pr,Pc,sym", [(2, 2, True), (2, 2, False), (1, 4, True), (4, 1, False)])
def test_bfs2d_loop_gloo(Pr, Pc, sym):
    tmp = tempfile.mkdtemp()
    mp.spawn(_worker, args=(WORLD, _free_port(), tmp, Pr, Pc, sym), nprocs=WORLD, join=True)
    A = synth.rmat(11, 8, seed=5, symmetrize=sym)
    C = oracle.csc_of(A)
    for s in np.load(os.path.join(tmp, "srcs.npy")):
        got = np.concatenate([np.load(os.path.join(tmp, f"lv{r}_{s}.npy")) for r in range(WORLD)])
        ref = oracle.bfs_queue(C, int(s))
        assert np.array_equal(got, ref)
        assert all(int(np.load(os.path.join(tmp, f"nl{r}_{s}.npy"))[0]) == int(ref.max()) + 1 for r in range(WORLD))
        # every rank decided on the same summed statistics, equal to Alg 3's per level
        outdeg = np.bincount(A.col_idx.numpy(), minlength=A.n)
        indeg = np.diff(A.row_ptr.numpy())
        want = [(int((ref == L).sum()), int(outdeg[ref == L].sum()), int(indeg[(ref < 0) | (ref > L)].sum()))
                for L in range(int(ref.max()) + 1)]
        for r in range(WORLD):
            assert [tuple(x) for x in np.load(os.path.join(tmp, f"seen{r}_{s}.npy"))] == want
