"""Multi-process (world size 2, gloo, CPU) tests of the row-block partitioned path
(DESIGN.md §8): partition, the two exchanges (x all-gather, frontier all-gather)
and the distributed TileBFS level loop `dist.bfs_loop`.  The per-rank compute is
a small numpy engine here (the CUDA engine is covered by test_gpu_dist_sim.py);
what is under test is the host logic and the bitmap-word conventions."""
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
from paper_conf_icpp_jisl0t022_b200 import dist as D

WORLD = 2


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_partition_rows_properties():
    A = synth.rmat(14, 16, seed=1)
    nnz = A.nnz
    for P in (1, 2, 3, 4, 8):
        s = D.partition_rows(A.row_ptr, P)
        assert len(s) == P + 1 and s[0] == 0 and s[-1] == A.m
        assert all(s[i] <= s[i + 1] for i in range(P))
        assert all(x % 64 == 0 for x in s[:-1])
        rp = A.row_ptr.numpy()
        loads = [int(rp[s[i + 1]] - rp[s[i]]) for i in range(P)]
        assert sum(loads) == nnz
        if P > 1:
            # unpermuted R-MAT: equal row blocks would give max/mean ~1.5-3.4 (S§8(e))
            assert max(loads) / (nnz / P) < 1.25
    # equal-row split on a uniform matrix stays equal
    U = synth.uniform(4096, 4096, 8, seed=3)
    s = D.partition_rows(U.row_ptr, 4)
    assert all(abs(s[i] - 1024 * i) <= 64 for i in range(5))


def _pack_words(bits: np.ndarray) -> torch.Tensor:
    """bool[n_owned] -> int32 words, bit v%32 of word v//32 (LSB-first) as in libtsmv."""
    nw = (bits.size + 31) // 32
    pad = np.zeros(nw * 32, dtype=bool)
    pad[:bits.size] = bits
    b8 = np.packbits(pad, bitorder="little")
    return torch.from_numpy(b8.view("<u4").astype(np.int64).astype(np.uint32).view(np.int32).copy())


def _unpack_words(words: torch.Tensor, count: int) -> np.ndarray:
    u8 = words.numpy().view(np.uint32).astype("<u4").view(np.uint8)
    return np.unpackbits(u8, bitorder="little")[:count].astype(bool)


class NumpyEngine:
    """Per-rank stand-in for DistTiledMatrix: same interface, numpy compute."""

    def __init__(self, A, splits, rank):
        self.n = A.n
        self.splits = splits
        self.rank = rank
        self.r0, self.r1 = splits[rank], splits[rank + 1]
        Al = D.local_rows(A, splits, rank)
        self.B = sp.csr_matrix((np.ones(Al.nnz), Al.col_idx.numpy(), Al.row_ptr.numpy()), shape=(Al.m, A.n))
        # global out-degrees (column counts of all blocks), as tsmv_bfs_dist_set_degrees
        self.outdeg = np.bincount(A.col_idx.numpy(), minlength=A.n).astype(np.int64)
        self.indeg = np.diff(Al.row_ptr.numpy()).astype(np.int64)
        self.stride = max((splits[p + 1] - splits[p] + 31) // 32 for p in range(len(splits) - 1))
        self.device = torch.device("cpu")
        self.levels = None
        from paper_conf_icpp_jisl0t022_b200 import tsmv
        self.tsmv = tsmv

    def choose(self, n, f, mf, mu, fprev=0):
        return self.tsmv.choose_dir(n, f, mf, mu, None, fprev)

    def _stats(self):
        # this rank's shares over its own rows (the libtsmv r2 semantics); bfs_loop sums them
        own_f = self.F[self.r0:self.r1]
        own_unvisited = ~self.V[self.r0:self.r1]
        return (int(own_f.sum()), int(self.outdeg[self.r0:self.r1][own_f].sum()),
                int(self.indeg[own_unvisited].sum()))

    def begin(self, s):
        self.V = np.zeros(self.n, bool)
        self.F = np.zeros(self.n, bool)
        self.V[s] = self.F[s] = True
        self.levels = np.full(self.r1 - self.r0, -1, np.int32)
        if self.r0 <= s < self.r1:
            self.levels[s - self.r0] = 0
        self.L = 0
        return self._stats()

    def expand(self, d, wide=False):  # wide: late-pull hint (no effect on results)
        y = (self.B @ self.F.astype(np.float64)) > 0
        new = y & ~self.V[self.r0:self.r1]
        return _pack_words(new)

    def merge(self, gathered, stride):
        new = np.zeros(self.n, bool)
        for p in range(len(self.splits) - 1):
            cnt = self.splits[p + 1] - self.splits[p]
            seg = gathered[p * stride:p * stride + (cnt + 31) // 32]
            new[self.splits[p]:self.splits[p + 1]] = _unpack_words(seg, cnt)
        self.V |= new
        self.F = new
        self.L += 1
        own = new[self.r0:self.r1]
        self.levels[own] = self.L
        return self._stats()


def _worker(rank, world, port, tmp, which):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    tdist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        if which == "exchange":
            t = torch.arange(3 + 4 * rank, dtype=torch.int32) + 100 * rank
            out = D.allgather_varlen(t)
            np.save(os.path.join(tmp, f"ag{rank}.npy"), out.numpy())
            w = torch.full((2 + rank,), 7 + rank, dtype=torch.int32)
            g = D.exchange_frontier(w, stride=4)
            np.save(os.path.join(tmp, f"ex{rank}.npy"), g.numpy())
        elif which.startswith("bfs"):
            sym = which == "bfs_sym"
            A = synth.rmat(11, 8, seed=5, symmetrize=sym)
            splits = D.partition_rows(A.row_ptr, world)
            eng = NumpyEngine(A, splits, rank)
            srcs = synth.sample_sources(A, 2, seed=3)
            for s in srcs:
                D.bfs_loop(eng, s)
                np.save(os.path.join(tmp, f"lv{rank}_{s}.npy"), eng.levels)
            np.save(os.path.join(tmp, "srcs.npy"), np.array(srcs))
            np.save(os.path.join(tmp, "splits.npy"), np.array(splits))
        elif which == "bootstrap":
            # DistMatrix bootstrap: one NCCL unique id made on rank 0, shared over the group
            uid = D.bootstrap_unique_id()
            np.save(os.path.join(tmp, f"uid{rank}.npy"), np.frombuffer(uid, dtype=np.uint8))
            uid2 = D.bootstrap_unique_id()
            np.save(os.path.join(tmp, f"uidb{rank}.npy"), np.frombuffer(uid2, dtype=np.uint8))
        elif which == "spmspv":
            A = synth.attach_values(synth.rmat(10, 8, seed=2), seed=1, integer=True)
            splits = D.partition_rows(A.row_ptr, world)
            xi, xv = synth.sample_x(A.n, 120, seed=4, integer=True)
            own = (xi >= splits[rank]) & (xi < splits[rank + 1])
            gi = D.allgather_varlen(xi[own])
            gv = D.allgather_varlen(xv[own])
            assert torch.equal(gi, xi) and torch.equal(gv, xv)
            Al = D.local_rows(A, splits, rank)
            yi, yv = oracle.spmspv(oracle.csc_of(Al), gi.numpy(), gv.numpy())   # local engine stand-in
            np.save(os.path.join(tmp, f"yi{rank}.npy"), yi + splits[rank])
            np.save(os.path.join(tmp, f"yv{rank}.npy"), yv)
        tdist.barrier()
    finally:
        tdist.destroy_process_group()


def _run(which):
    tmp = tempfile.mkdtemp()
    mp.spawn(_worker, args=(WORLD, _free_port(), tmp, which), nprocs=WORLD, join=True)
    return tmp


def test_exchanges_gloo():
    tmp = _run("exchange")
    ref = np.concatenate([np.arange(3) + 0, np.arange(7) + 100]).astype(np.int32)
    for r in range(WORLD):
        assert np.array_equal(np.load(os.path.join(tmp, f"ag{r}.npy")), ref)
        ex = np.load(os.path.join(tmp, f"ex{r}.npy"))
        assert ex.tolist() == [7, 7, 0, 0, 8, 8, 8, 0]


@pytest.mark.parametrize("which", ["bfs_sym", "bfs_dir"])
def test_distributed_bfs_loop_gloo(which):
    tmp = _run(which)
    A = synth.rmat(11, 8, seed=5, symmetrize=which == "bfs_sym")
    C = oracle.csc_of(A)
    for s in np.load(os.path.join(tmp, "srcs.npy")):
        got = np.concatenate([np.load(os.path.join(tmp, f"lv{r}_{s}.npy")) for r in range(WORLD)])
        assert np.array_equal(got, oracle.bfs_queue(C, int(s)))


def test_bootstrap_unique_id_gloo():
    """dist.bootstrap_unique_id: every rank gets rank 0's 128 bytes; a second call
    (a second communicator) gets a new id."""
    tmp = _run("bootstrap")
    ids = [np.load(os.path.join(tmp, f"uid{r}.npy")) for r in range(WORLD)]
    idsb = [np.load(os.path.join(tmp, f"uidb{r}.npy")) for r in range(WORLD)]
    assert ids[0].size == 128 and ids[0].any()
    assert all(np.array_equal(ids[0], x) for x in ids) and all(np.array_equal(idsb[0], x) for x in idsb)
    assert not np.array_equal(ids[0], idsb[0])


def test_distributed_spmspv_gloo():
    tmp = _run("spmspv")
    A = synth.attach_values(synth.rmat(10, 8, seed=2), seed=1, integer=True)
    xi, xv = synth.sample_x(A.n, 120, seed=4, integer=True)
    ri, rv = oracle.spmspv(oracle.csc_of(A), xi.numpy(), xv.numpy())
    gi = np.concatenate([np.load(os.path.join(tmp, f"yi{r}.npy")) for r in range(WORLD)])
    gv = np.concatenate([np.load(os.path.join(tmp, f"yv{r}.npy")) for r in range(WORLD)])
    assert np.array_equal(gi, ri) and np.array_equal(gv, rv)


def test_partition_rows_unaligned_m():
    """m not a multiple of 64: interior splits stay multiples of 64 and
    never pass the last aligned row, also when the nonzeros sit in the last rows."""
    import synth as S
    for m, P in ((120, 8), (120, 2), (1000, 3), (65, 2)):
        counts = torch.zeros(m, dtype=torch.int64)
        counts[-8:] = 50                                  # tail-heavy
        rp = torch.zeros(m + 1, dtype=torch.int64)
        rp[1:] = torch.cumsum(counts, 0)
        s = D.partition_rows(rp, P)
        assert s[0] == 0 and s[-1] == m and len(s) == P + 1
        assert all(x % 64 == 0 for x in s[1:-1]), s
        assert all(s[i] <= s[i + 1] for i in range(P)), s
    U = S.uniform(1000, 1000, 4, seed=1)
    s = D.partition_rows(U.row_ptr, 4)
    assert all(x % 64 == 0 for x in s[1:-1]) and s[-1] == 1000
