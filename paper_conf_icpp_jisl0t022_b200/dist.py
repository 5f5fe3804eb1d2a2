"""Row-block multi-GPU TileSpMSpV / TileBFS.

The paper is single-GPU; the partitioned path is this build's addition
(BASELINE.json north_star item 4).  One process per GPU.  Rank p owns global
rows [splits[p], splits[p+1]) of A (contiguous, nnz-balanced, cut at multiples
of 64 rows so tile rows and bitmap words never straddle ranks) in its own
libtsmv context; columns stay global.

The product path is `DistMatrix`: this module only BOOTSTRAPS it (the row
partition, and one ncclUniqueId from rank 0 shared over torch.distributed);
the context then owns its NCCL communicator and `tsmv_bfs` / `tsmv_spmspv`
are collective calls whose level loop and exchanges run inside libtsmv.so
(comm.cu: in-place broadcasts of the owned frontier words per level; count
all-gather + broadcasts of the owned x entries).

`DistTiledMatrix` + `bfs_loop` keep the caller-driven form (the
tsmv_bfs_dist_* primitives, exchange by torch.distributed or by concatenation):
it runs where a communicator cannot (several simulated ranks on one GPU, the
gloo CPU tests) and checks the partitioned kernels rank by rank.
"""
from __future__ import annotations

import ctypes
import os
from typing import List, Optional, Sequence

import torch
import torch.distributed as dist

ALIGN = 64
# late pull levels (unvisited in-edges mu * WIDE_MULT < nnz) take the wide form; the
# library's host loops use the same rule (csrc/bfs.cu bfs_wide_mult, TSMV_BFS_WIDE_MULT)
WIDE_MULT = int(os.environ.get("TSMV_BFS_WIDE_MULT", "64"))
# row blocks of a TileBFS context balance nnz + BFS_ROW_WEIGHT x rows: R-MAT's
# nnz-balanced blocks put the many low-degree tail vertices on the last ranks, whose
# dense pull level then dominates (s26 projection at P = 8: 1097 GTEPS with weight
# 0, 1294 / 1328 / 1364 / 1352 / 1336 with 16 / 64 / 128 / 256 / 512; r2 session 5)
BFS_ROW_WEIGHT = float(os.environ.get("TSMV_BFS_ROW_WEIGHT", "128"))


def partition_rows(row_ptr: torch.Tensor, nranks: int, align: int = ALIGN,
                   row_weight: Optional[float] = None) -> List[int]:
    """nnz-balanced contiguous row blocks: split p is the multiple of `align` nearest
    to the row where the running nnz reaches p/nranks of the total.  With
    row_weight w (default: env TSMV_PART_ROW_WEIGHT, else 0) the balanced quantity
    is nnz + w x rows (a dense pull level's work grows with the block's unvisited
    vertices, not only its nonzeros).
    Returns nranks+1 global row boundaries (first 0, last m)."""
    rp = row_ptr.detach().to("cpu", torch.int64)
    m = rp.numel() - 1
    if row_weight is None:
        row_weight = float(os.environ.get("TSMV_PART_ROW_WEIGHT", "0"))
    if row_weight:
        rp = rp + torch.round(torch.arange(m + 1, dtype=torch.float64) * row_weight).to(torch.int64)
    nnz = int(rp[-1])
    splits = [0]
    for p in range(1, nranks):
        target = (nnz * p + nranks - 1) // nranks
        r = int(torch.searchsorted(rp, torch.tensor(target, dtype=torch.int64), right=False))
        # nearest multiple of `align`, never past the last aligned row (an interior
        # split must stay a multiple of `align` even when m is not)
        r = min((m // align) * align, ((r + align // 2) // align) * align)
        splits.append(max(r, splits[-1]))
    splits.append(m)
    return splits


class RowBlock:
    """A CSR row block: m local rows, n global columns (row_ptr int64, col_idx int32)."""

    def __init__(self, m, n, row_ptr, col_idx, values=None, name="block"):
        self.m, self.n, self.row_ptr, self.col_idx, self.values, self.name = m, n, row_ptr, col_idx, values, name

    @property
    def nnz(self):
        return int(self.col_idx.numel())

    def to(self, device):
        v = None if self.values is None else self.values.to(device)
        return RowBlock(self.m, self.n, self.row_ptr.to(device), self.col_idx.to(device), v, self.name)

    def with_values(self, values):
        return RowBlock(self.m, self.n, self.row_ptr, self.col_idx, values, self.name)


def local_rows(A, splits: Sequence[int], rank: int) -> RowBlock:
    """The CSR block of A holding rows [splits[rank], splits[rank+1]) (global columns)."""
    r0, r1 = int(splits[rank]), int(splits[rank + 1])
    rp = A.row_ptr[r0:r1 + 1]
    base = int(rp[0])
    cols = A.col_idx[base:int(rp[-1])]
    vals = None if A.values is None else A.values[base:int(rp[-1])]
    return RowBlock(r1 - r0, A.n, rp - base, cols, vals, f"{getattr(A, 'name', 'A')}[{r0}:{r1}]")


def bootstrap_unique_id(group=None) -> bytes:
    """One ncclUniqueId made by rank 0 and shared with every rank of `group` over
    torch.distributed (object broadcast: works on gloo and NCCL groups).  An id
    creates ONE communicator: bootstrap a new one for every DistMatrix."""
    from . import tsmv
    obj = [tsmv.nccl_unique_id() if dist.get_rank(group) == 0 else None]
    dist.broadcast_object_list(obj, src=dist.get_global_rank(group, 0) if group is not None else 0, group=group)
    return obj[0]


class DistMatrix:
    """This rank's row block in a libtsmv context that owns its NCCL communicator:
    bfs() and spmspv() are collective calls running entirely in the library."""

    def __init__(self, A_local, splits: Sequence[int], rank: int, nranks: int, unique_id: bytes,
                 dtype: Optional[str] = None, device: int = 0, **opts):
        from . import tsmv
        self.splits = [int(s) for s in splits]
        self.rank, self.nranks = rank, nranks
        self.m_local, self.n = A_local.m, A_local.n
        self.device = torch.device("cuda", device)
        kw = dict(rank=rank, nranks=nranks, nccl_unique_id=unique_id)
        opts.setdefault("build_bfs", 1)
        if nranks > 1:
            kw["row_splits"] = self.splits
        self.M = tsmv.TiledMatrix(A_local.m, A_local.n, A_local.row_ptr, A_local.col_idx, A_local.values,
                                  dtype=dtype, device=device, **kw, **opts)

    def bfs(self, source: int, levels: Optional[torch.Tensor] = None):
        """Collective: levels of this rank's rows, global statistics."""
        return self.M.bfs(source, levels=levels)

    def spmspv(self, x_idx_owned: torch.Tensor, x_val_owned: Optional[torch.Tensor], semiring="plus_times",
               y_idx: Optional[torch.Tensor] = None, y_val: Optional[torch.Tensor] = None):
        """Collective: x entries owned by this rank (indices in its row range) in,
        y of this rank's rows out."""
        return self.M.spmspv(x_idx_owned, x_val_owned, semiring=semiring, y_idx=y_idx, y_val=y_val)

    def close(self):
        self.M.close()


def allgather_sizes(count: int, device, group=None) -> List[int]:
    """Per-rank element counts (one all-gather, one host read)."""
    world = dist.get_world_size(group)
    n = torch.tensor([count], dtype=torch.int64, device=device)
    out = torch.empty(world, dtype=torch.int64, device=device)
    dist.all_gather_into_tensor(out, n, group=group)
    return out.tolist()


def allgather_varlen(t: torch.Tensor, group=None, sizes: Optional[List[int]] = None) -> torch.Tensor:
    """Concatenation, in rank order, of a 1-D tensor of per-rank length (`sizes`,
    if the caller already exchanged them)."""
    world = dist.get_world_size(group)
    if sizes is None:
        sizes = allgather_sizes(t.numel(), t.device, group)
    mx = max(sizes) if sizes else 0
    pad = torch.zeros(max(mx, 1), dtype=t.dtype, device=t.device)
    pad[:t.numel()] = t
    out = torch.empty(world * max(mx, 1), dtype=t.dtype, device=t.device)
    dist.all_gather_into_tensor(out, pad, group=group)
    return torch.cat([out[p * max(mx, 1):p * max(mx, 1) + sizes[p]] for p in range(world)])


def exchange_frontier(owned_words: torch.Tensor, stride: int, group=None) -> torch.Tensor:
    """All-gather of the owned frontier-bitmap segments, each padded to `stride`
    uint32 words (int32 storage), rank-major: out[p*stride + w]."""
    world = dist.get_world_size(group)
    buf = torch.zeros(stride, dtype=owned_words.dtype, device=owned_words.device)
    buf[:owned_words.numel()] = owned_words
    out = torch.empty(world * stride, dtype=owned_words.dtype, device=owned_words.device)
    dist.all_gather_into_tensor(out, buf, group=group)
    return out


def bfs_loop(engine, source: int, group=None) -> int:
    """Level-synchronous distributed TileBFS driver (Alg 3, one
    exchange per level).  `engine` provides begin(source) -> this rank's shares
    (|F|, m_f, m_u) of its own rows, expand(dir) -> owned words, merge(gathered,
    stride) -> shares, stride (padded words), n, choose(n, |F|, m_f, m_u).  The three
    shares are summed over the ranks (one all-reduce per level), so every rank
    decides the direction on the same global numbers.  Returns the number of levels."""
    dev = engine.device
    red = torch.tensor(list(engine.begin(source)), dtype=torch.int64, device=dev)
    dist.all_reduce(red, group=group)
    f, gmf, gmu = (int(x) for x in red.tolist())
    levels = 0
    fprev = 0   # |F| of the previous level (direction rule R9')
    while f > 0:
        d = engine.choose(engine.n, f, gmf, gmu, fprev)
        fprev = f
        # late pull levels (few unvisited edges) take the wide row-tile test
        wide = getattr(engine, "nnz_total", 0) > 0 and gmu * WIDE_MULT < engine.nnz_total
        owned = engine.expand(d, wide=wide)
        gathered = exchange_frontier(owned, engine.stride, group)
        if hasattr(engine, "merge_dev"):
            # statistics stay on the device: one all-reduce, one read per level
            red = engine.merge_dev(gathered, engine.stride).clone()
        else:
            red = torch.tensor(list(engine.merge(gathered, engine.stride)), dtype=torch.int64, device=dev)
        dist.all_reduce(red, group=group)
        f, gmf, gmu = (int(x) for x in red.tolist())
        levels += 1
    return levels


class DistTiledMatrix:
    """This rank's row block of A in a libtsmv context, plus the exchange steps."""

    def __init__(self, A_local, splits: Sequence[int], rank: int, nranks: int, group=None,
                 dtype: Optional[str] = None, device: int = 0, **opts):
        from . import tsmv
        self.tsmv = tsmv
        self.splits = [int(s) for s in splits]
        self.rank, self.nranks, self.group = rank, nranks, group
        self.n = A_local.n
        self.m_local = A_local.m
        self.device = torch.device("cuda", device)
        self.M = tsmv.TiledMatrix(A_local.m, A_local.n, A_local.row_ptr, A_local.col_idx, A_local.values,
                                  dtype=dtype, device=device, rank=rank, nranks=nranks,
                                  row_splits=self.splits, build_bfs=1, **opts)
        self.stride = max((self.splits[p + 1] - self.splits[p] + 31) // 32 for p in range(nranks))
        self.owned = torch.zeros(max(1, (self.m_local + 31) // 32), dtype=torch.int32, device=self.device)
        self.levels = torch.empty(max(1, self.m_local), dtype=torch.int32, device=self.device)
        self._stats = (torch.zeros(3, dtype=torch.int64))
        self._stats_dev = torch.zeros(3, dtype=torch.int64, device=self.device)
        # global nnz (one all-reduce at construction): the late-pull hint of bfs_loop;
        # 0 (no hint) when there is no process group (simulated ranks)
        self.nnz_total = 0
        if dist.is_available() and dist.is_initialized():
            on = self.device if dist.get_backend(group) == "nccl" else "cpu"
            tot = torch.tensor([int(A_local.nnz)], dtype=torch.int64, device=on)
            dist.all_reduce(tot, group=group)
            self.nnz_total = int(tot)
            # global out-degrees: the column counts of all row blocks (m_f of Alg 3's
            # direction rule counts every block's edges of a frontier vertex)
            deg = self.column_counts(A_local).to(on)
            dist.all_reduce(deg, group=group)
            self.set_degrees(deg)

    @staticmethod
    def column_counts(A_local) -> torch.Tensor:
        """int32[n] column counts of this row block (host-side marshalling for
        set_degrees; summed over the ranks they are the global out-degrees)."""
        ci = A_local.col_idx.to(torch.int64)
        return torch.bincount(ci, minlength=A_local.n).to(torch.int32)

    def set_degrees(self, outdeg_global: torch.Tensor):
        """Global out-degrees (int32[n]) for the direction statistics; set by the
        constructor when a process group exists, by the caller for simulated ranks."""
        d = outdeg_global.to(device=self.device, dtype=torch.int32).contiguous()
        self.tsmv.check(self.tsmv.tsmv_bfs_dist_set_degrees(self.M.ctx, d.data_ptr()),
                        "tsmv_bfs_dist_set_degrees")

    # ---- SpMSpV: x entries are distributed by owner (x_idx in this rank's row range)
    def spmspv(self, x_idx_owned: torch.Tensor, x_val_owned: Optional[torch.Tensor], semiring="plus_times"):
        sizes = allgather_sizes(x_idx_owned.numel(), x_idx_owned.device, self.group)
        xi = allgather_varlen(x_idx_owned.to(torch.int32), self.group, sizes)
        xv = None if x_val_owned is None else allgather_varlen(x_val_owned, self.group, sizes)
        if xi.numel() == 0:
            return xi, xv
        return self.M.spmspv(xi, xv, semiring=semiring)

    def spmspv_async(self, x_idx_owned: torch.Tensor, x_val_owned: Optional[torch.Tensor], y_idx: torch.Tensor,
                     y_val: Optional[torch.Tensor], y_nnz: torch.Tensor, semiring="plus_times"):
        """spmspv() without the final synchronisation: y for the owned rows and its
        size (int64[1] on the device) are written on the current stream."""
        sizes = allgather_sizes(x_idx_owned.numel(), x_idx_owned.device, self.group)
        xi = allgather_varlen(x_idx_owned.to(torch.int32), self.group, sizes)
        xv = None if x_val_owned is None else allgather_varlen(x_val_owned, self.group, sizes)
        if xi.numel() == 0:
            y_nnz.zero_()
            return
        self.M.spmspv_async(xi, xv, y_idx, y_val, y_nnz, semiring=semiring)

    # ---- BFS engine interface
    def choose(self, n, f, mf, mu, fprev=0):
        return self.tsmv.choose_dir(n, f, mf, mu, self.M.opts, fprev)

    def begin(self, source):
        import ctypes
        st = (ctypes.c_int64 * 3)()
        self.tsmv.check(self.tsmv.tsmv_bfs_dist_begin(self.M.ctx, int(source), self.levels.data_ptr(), st,
                                                      torch.cuda.current_stream().cuda_stream),
                        "tsmv_bfs_dist_begin")
        return st[0], st[1], st[2]

    def expand(self, d, wide=False):
        d = int(d) | (self.tsmv.DIST_WIDE if wide else 0)
        self.tsmv.check(self.tsmv.tsmv_bfs_dist_expand(self.M.ctx, d, self.owned.data_ptr(),
                                                       torch.cuda.current_stream().cuda_stream),
                        "tsmv_bfs_dist_expand")
        return self.owned

    def merge(self, gathered, stride):
        import ctypes
        st = (ctypes.c_int64 * 3)()
        self.tsmv.check(self.tsmv.tsmv_bfs_dist_merge(self.M.ctx, gathered.data_ptr(), int(stride), st,
                                                      torch.cuda.current_stream().cuda_stream),
                        "tsmv_bfs_dist_merge")
        return st[0], st[1], st[2]

    def merge_dev(self, gathered, stride):
        """merge() with the statistics left on the device (int64[3], no sync)."""
        self.tsmv.check(self.tsmv.tsmv_bfs_dist_merge(self.M.ctx, gathered.data_ptr(), int(stride),
                                                      ctypes.cast(self._stats_dev.data_ptr(),
                                                                  ctypes.POINTER(ctypes.c_int64)),
                                                      torch.cuda.current_stream().cuda_stream),
                        "tsmv_bfs_dist_merge")
        return self._stats_dev

    def bfs(self, source: int):
        nl = bfs_loop(self, source, self.group)
        return self.levels[:self.m_local], nl
