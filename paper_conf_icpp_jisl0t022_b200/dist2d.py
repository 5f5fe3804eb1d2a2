"""2D (processor row x processor column) partitioned TileBFS (SURVEY §8(f)
NEXT-4, "beyond one GPU's memory"; DESIGN.md §8 "2D").

P = Pr x Pc ranks, rank r = i * Pc + j.  The vertices are cut into P contiguous
pieces (multiples of 64); piece q = i * Pc + j is R_ij, the vertices rank (i, j)
owns (visited bits, levels).  Row block R_i = pieces i*Pc .. i*Pc+Pc-1 (contiguous);
column block C_j = pieces j, Pc + j, 2 Pc + j, ... (one per processor row).  Rank
(i, j) holds A_ij = A[R_i, C_j] in an ordinary libtsmv context whose local ids are
PADDED: every piece gets a slot of S bits (S = the largest piece, rounded up to
64), local row = (sub-piece) * S + offset, local column = (processor row of the
piece) * S + offset.  With that layout every exchange is an equal-size collective.
A level (Alg 3) on rank (i, j):

    x_j   = all-gather over processor column j of the owners' frontier words
            (Pr slots of S / 32 words = C_j's bitmap in local column ids);
    rows  = all-gather over processor row i of the same words (R_i's new vertices,
            ORed into the row-replicated visited bitmap; direction-optimising mode);
    dir   = Alg 3's rule (reading R9) on the summed statistics of the last merge;
    y     = tsmv_bfs2d_expand: the row-block path's Push-CSC / Push-CSR / Pull-CSC
            kernels on A_ij -> partial bitmap over R_i, Pc slots ("dopt"), or the
            OR-AND SpMSpV of A_ij + tsmv_bfs2d_scatter ("push");
    recv  = all-to-all over processor row i (slot j' goes to rank (i, j'));
    front = tsmv_bfs2d_merge(recv): OR of the Pc partials, minus visited, levels,
            statistics shares {|F|, m_f, m_u decrement} of the owned new vertices;
    stats = all-reduce of the three shares (direction + termination).

Per-rank state is O(|R_i| + |C_j|) bits plus its own levels and degrees, against
the row-block design's replicated O(n) bitmaps and degree arrays,
and the bytes a rank moves per level are S / 8 x (Pr + 2 Pc) instead of n / 8.

Every step of a level runs in libtsmv kernels; this module only slices the input
blocks and calls the collectives.  `bfs2d_loop` takes any `comm` with the
exchanges (TorchComm2D), `sim_bfs2d` runs P simulated ranks on one GPU.
"""
from __future__ import annotations

import ctypes
import math
from typing import List, Optional, Sequence

import torch
import torch.distributed as dist

from .dist import ALIGN, RowBlock, partition_rows


def grid_shape(P: int) -> tuple:
    """Near-square Pr x Pc with Pr <= Pc (Pr = the largest divisor <= sqrt P)."""
    pr = max(d for d in range(1, int(math.isqrt(P)) + 1) if P % d == 0)
    return pr, P // pr


def _round_up(x: int, a: int = ALIGN) -> int:
    return (x + a - 1) // a * a


class Grid2D:
    """The vertex pieces of a Pr x Pc grid and the padded local id spaces."""

    def __init__(self, n: int, Pr: int, Pc: int, row_ptr: Optional[torch.Tensor] = None, balance: str = "rows"):
        self.n, self.Pr, self.Pc, self.P = int(n), int(Pr), int(Pc), int(Pr) * int(Pc)
        P = self.P
        if balance == "rows" or row_ptr is None:
            # equal pieces (the Graph500 setting: a permuted graph balances the blocks)
            pieces = [min(self.n, _round_up((self.n * q) // P)) if q < P else self.n for q in range(P + 1)]
            pieces[0] = 0
        elif balance == "nnz":
            # nnz-balanced row blocks R_i, each cut into Pc nnz-balanced sub-pieces
            rb = partition_rows(row_ptr, self.Pr)
            rp = row_ptr.detach().to("cpu", torch.int64)
            pieces = []
            for i in range(self.Pr):
                r0, r1 = rb[i], rb[i + 1]
                sub = partition_rows(rp[r0:r1 + 1] - rp[r0], self.Pc)
                pieces += [r0 + s for s in sub[:-1]]
            pieces.append(self.n)
        else:
            raise ValueError(f"balance must be 'rows' or 'nnz', not {balance!r}")
        for q in range(P):
            pieces[q + 1] = max(pieces[q + 1], pieces[q])
        self.pieces = pieces
        self.S = max(_round_up(max(1, pieces[q + 1] - pieces[q])) for q in range(P))
        self.sw = self.S // 32              # words per slot

    def rank_of(self, i: int, j: int) -> int:
        return i * self.Pc + j

    def coords(self, r: int) -> tuple:
        return divmod(r, self.Pc)

    def piece(self, q: int) -> tuple:
        return self.pieces[q], self.pieces[q + 1]

    def owner(self, v: int) -> int:
        for q in range(self.P):
            if self.pieces[q] <= v < self.pieces[q + 1]:
                return q
        raise ValueError(f"vertex {v} out of range")


def block_2d(A, grid: Grid2D, i: int, j: int, chunk: int = 1 << 26) -> RowBlock:
    """A_ij = A[R_i, C_j] with padded local ids (module docstring): m = Pc x S rows,
    n = Pr x S columns; entries keep their order (ascending local columns per row).
    Rows are sliced in chunks of about `chunk` entries to bound the temporaries."""
    Pc, S = grid.Pc, grid.S
    dev = A.row_ptr.device
    pieces = torch.tensor(grid.pieces, dtype=torch.int64, device=dev)
    r0, r1 = grid.pieces[i * Pc], grid.pieces[(i + 1) * Pc]
    rp_all = A.row_ptr.to(torch.int64)
    cnt = torch.zeros(Pc * S, dtype=torch.int64, device=dev)
    cols_out, vals_out = [], []
    ra = r0
    while ra < r1:
        # rows [ra, rb) hold about `chunk` entries (at least one row)
        target = int(rp_all[ra]) + chunk
        rb = int(torch.searchsorted(rp_all[ra:r1 + 1], torch.tensor(target, device=dev), right=True)) + ra - 1
        rb = min(r1, max(rb, ra + 1))
        rp = rp_all[ra:rb + 1]
        base, end = int(rp[0]), int(rp[-1])
        cols = A.col_idx[base:end].to(torch.int64)
        qc = torch.searchsorted(pieces, cols, right=True) - 1
        keep = (qc % Pc) == j
        lcol = ((qc // Pc) * S + (cols - pieces[qc]))[keep]
        del cols
        rows = torch.repeat_interleave(torch.arange(ra, rb, device=dev, dtype=torch.int64), rp[1:] - rp[:-1])[keep]
        qr = torch.searchsorted(pieces, rows, right=True) - 1
        cnt += torch.bincount((qr - i * Pc) * S + (rows - pieces[qr]), minlength=Pc * S)
        del rows, qr, qc
        cols_out.append(lcol.to(torch.int32))
        if A.values is not None:
            vals_out.append(A.values[base:end][keep])
        del keep, lcol
        ra = rb
    row_ptr = torch.zeros(Pc * S + 1, dtype=torch.int64, device=dev)
    row_ptr[1:] = torch.cumsum(cnt, 0)
    col_idx = torch.cat(cols_out) if cols_out else torch.zeros(0, dtype=torch.int32, device=dev)
    vals = torch.cat(vals_out) if vals_out else None
    return RowBlock(Pc * S, grid.Pr * S, row_ptr, col_idx, vals, f"A[{i},{j}]")


class Dist2DBFS:
    """Rank (i, j)'s block and BFS state; begin / expand / merge are the per-rank
    steps of a level (all compute in libtsmv), `bfs2d_loop` drives them.

    mode "dopt" (default): direction-optimising levels, tsmv_bfs2d_expand runs the
    row-block path's Push-CSC / Push-CSR / Pull-CSC kernels on the block (context
    built with build_bfs = 2), with R_i's visited bitmap replicated over the
    processor row (the all-gather of the owners' new words, `needs_rows`).
    mode "push": every level is the OR-AND SpMSpV of the block (Alg 3 + Alg 5
    only), no row replication."""

    def __init__(self, A_block: RowBlock, grid: Grid2D, rank: int, device: int = 0, mode: str = "dopt", **opts):
        from . import tsmv
        if mode not in ("dopt", "push"):
            raise ValueError(f"mode must be 'dopt' or 'push', not {mode!r}")
        self.tsmv = tsmv
        self.grid = grid
        self.rank = rank
        self.mode = mode
        self.needs_rows = mode == "dopt"
        self.i, self.j = grid.coords(rank)
        self.device = torch.device("cuda", device)
        d = self.device
        opts["build_bfs"] = 2 if mode == "dopt" else 0
        self.M = tsmv.TiledMatrix(A_block.m, A_block.n, A_block.row_ptr.to(d), A_block.col_idx.to(d), None,
                                  dtype="pattern", device=device, **opts)
        S, sw = grid.S, grid.sw
        p0, p1 = grid.piece(rank)
        self.own0, self.nown = p0, p1 - p0
        self.visited = torch.zeros(sw, dtype=torch.int32, device=d)
        self.levels = torch.full((S,), -1, dtype=torch.int32, device=d)
        self.front = torch.zeros(sw, dtype=torch.int32, device=d)
        self.ywords = torch.zeros(grid.Pc * sw, dtype=torch.int32, device=d)
        self.stats = torch.zeros(3, dtype=torch.int64, device=d)
        self.outdeg = self.indeg = None
        self.nnz_total = 0
        if mode == "push":
            self.x_idx = torch.empty(grid.Pr * S, dtype=torch.int32, device=d)
            self.y_idx = torch.empty(grid.Pc * S, dtype=torch.int32, device=d)
            self.y_nnz = torch.zeros(1, dtype=torch.int64, device=d)
            self._k = ctypes.c_int64(0)
        else:
            self.vis_rows = torch.zeros(grid.Pc * sw, dtype=torch.int32, device=d)
            self.levels_rows = torch.empty(grid.Pc * S, dtype=torch.int32, device=d)

    def set_degrees(self, outdeg_own: torch.Tensor, indeg_own: torch.Tensor, nnz_total: int):
        """GLOBAL out-degrees (column counts of A) and in-degrees (row counts) of this
        rank's vertices, and nnz(A): the direction statistics of Alg 3."""
        self.outdeg = outdeg_own.to(self.device, torch.int32).contiguous()
        self.indeg = indeg_own.to(self.device, torch.int32).contiguous()
        self.nnz_total = int(nnz_total)

    def _st(self):
        return torch.cuda.current_stream(self.device).cuda_stream

    def choose(self, f, mf, mu, fprev=0):
        return self.tsmv.choose_dir(self.grid.n, f, mf, mu, self.M.opts, fprev)

    def begin(self, source: int) -> torch.Tensor:
        """Reset the state; the owner of `source` marks it (level 0) in its frontier
        words and puts its statistics shares in `stats`."""
        self.visited.zero_()
        self.levels.fill_(-1)
        self.front.zero_()
        self.stats.zero_()
        if self.needs_rows:
            self.vis_rows.zero_()
        if self.own0 <= source < self.own0 + self.nown:
            o = source - self.own0
            bit = torch.tensor([1 << (o & 31)], dtype=torch.int64).to(torch.int32).to(self.device)
            self.front[o >> 5] = bit
            self.visited[o >> 5] = bit
            self.levels[o] = 0
            self.stats[0] = 1
            if self.outdeg is not None:
                self.stats[1] = self.outdeg[o].to(torch.int64)
                self.stats[2] = self.indeg[o].to(torch.int64)
        return self.front

    def expand(self, x_words: torch.Tensor, d: int = 1, row_new: Optional[torch.Tensor] = None,
               level: int = 0) -> torch.Tensor:
        """x_words = C_j's frontier bitmap (Pr slots, the processor-column
        all-gather); returns the partial bitmap over R_i (Pc slots = the all-to-all
        send buffer).  dopt: direction d (| DIST_WIDE), row_new = R_i's vertices of
        this level (processor-row all-gather).  push: list + OR-AND SpMSpV + scatter."""
        t = self.tsmv
        if self.mode == "dopt":
            t.check(t.tsmv_bfs2d_expand(self.M.ctx, int(d), x_words.data_ptr(),
                                        None if row_new is None else row_new.data_ptr(), self.vis_rows.data_ptr(),
                                        self.ywords.data_ptr(), self.levels_rows.data_ptr(), int(level),
                                        self._st()), "tsmv_bfs2d_expand")
            return self.ywords
        t.check(t.tsmv_bfs2d_list(self.M.ctx, x_words.data_ptr(), self.grid.Pr * self.grid.S,
                                  self.x_idx.data_ptr(), ctypes.byref(self._k), self._st()), "tsmv_bfs2d_list")
        k = self._k.value
        if k == 0:
            self.y_nnz.zero_()
        else:
            self.M.spmspv_async(self.x_idx[:k], None, self.y_idx, None, self.y_nnz, semiring="or_and")
        t.check(t.tsmv_bfs2d_scatter(self.M.ctx, self.y_idx.data_ptr(), self.y_nnz.data_ptr(), self.y_idx.numel(),
                                     self.ywords.data_ptr(), self.ywords.numel(), self._st()), "tsmv_bfs2d_scatter")
        return self.ywords

    def merge(self, recv: torch.Tensor, level: int) -> tuple:
        """recv = the Pc partial bitmaps of R_ij (the processor-row all-to-all).
        Returns (frontier words, statistics shares int64[3] on the device)."""
        t = self.tsmv
        t.check(t.tsmv_bfs2d_merge(self.M.ctx, recv.data_ptr(), self.grid.Pc, self.grid.sw, self.nown,
                                   self.visited.data_ptr(), self.levels.data_ptr(), int(level),
                                   self.front.data_ptr(), None if self.outdeg is None else self.outdeg.data_ptr(),
                                   None if self.indeg is None else self.indeg.data_ptr(), self.stats.data_ptr(),
                                   self._st()), "tsmv_bfs2d_merge")
        return self.front, self.stats

    def owned_levels(self) -> torch.Tensor:
        return self.levels[:self.nown]

    def close(self):
        self.M.close()


def block_counts(B: RowBlock, grid: Grid2D) -> tuple:
    """(column counts int64[Pr x S], row counts int64[Pc x S]) of a padded block."""
    cc = torch.bincount(B.col_idx.to(torch.int64), minlength=grid.Pr * grid.S)
    rc = B.row_ptr[1:] - B.row_ptr[:-1]
    return cc, rc.to(torch.int64)


class TorchComm2D:
    """The exchanges of a 2D level over torch.distributed sub-groups (NCCL on GPUs,
    gloo on CPU).  Every rank must construct it (new_group is collective)."""

    def __init__(self, grid: Grid2D, rank: int):
        self.grid = grid
        Pr, Pc = grid.Pr, grid.Pc
        self.row_groups = [dist.new_group([i * Pc + j for j in range(Pc)]) for i in range(Pr)]
        self.col_groups = [dist.new_group([i * Pc + j for i in range(Pr)]) for j in range(Pc)]
        self.i, self.j = grid.coords(rank)
        self.row, self.col = self.row_groups[self.i], self.col_groups[self.j]

    def col_allgather(self, words: torch.Tensor) -> torch.Tensor:
        parts = [torch.empty_like(words) for _ in range(self.grid.Pr)]
        dist.all_gather(parts, words.contiguous(), group=self.col)
        return torch.cat(parts)

    def row_allgather(self, words: torch.Tensor) -> torch.Tensor:
        parts = [torch.empty_like(words) for _ in range(self.grid.Pc)]
        dist.all_gather(parts, words.contiguous(), group=self.row)
        return torch.cat(parts)

    def row_alltoall(self, words: torch.Tensor) -> torch.Tensor:
        out = torch.empty_like(words)
        dist.all_to_all_single(out, words.contiguous(), group=self.row)
        return out

    def allreduce(self, stats: torch.Tensor) -> List[int]:
        t = stats.clone()
        dist.all_reduce(t)
        return [int(x) for x in t.tolist()]

    def degrees(self, B: RowBlock) -> tuple:
        """This rank's GLOBAL (out-degree, in-degree) slices and nnz(A): the block's
        column counts summed over the processor column, its row counts over the
        processor row, the block nnz over all ranks."""
        g, S = self.grid, self.grid.S
        cc, rc = block_counts(B, g)
        dist.all_reduce(cc, group=self.col)
        dist.all_reduce(rc, group=self.row)
        tot = torch.tensor([B.nnz], dtype=torch.int64, device=cc.device)
        dist.all_reduce(tot)
        p0, p1 = g.piece(g.rank_of(self.i, self.j))
        n_own = p1 - p0
        return cc[self.i * S:self.i * S + n_own], rc[self.j * S:self.j * S + n_own], int(tot)


def bfs2d_loop(engine, source: int, comm) -> int:
    """Level-synchronous 2D BFS (Alg 3): gather x_j in the processor column (and,
    direction-optimising, R_i's new vertices in the processor row), decide the
    direction from the summed statistics (R9), expand, all-to-all the partial
    bitmaps in the processor row, merge; stop when the summed |F| is 0.  Returns
    the number of levels."""
    front = engine.begin(source)
    f, mf, dmu = comm.allreduce(engine.stats)
    mu = engine.nnz_total - dmu
    level = 0
    fprev = 0
    while True:
        x = comm.col_allgather(front)
        rn = comm.row_allgather(front) if engine.needs_rows else None
        d = engine.choose(f, mf, mu, fprev)
        fprev = f
        if engine.nnz_total > 0 and mu * 4 < engine.nnz_total:
            d |= DIST_WIDE
        y = engine.expand(x, d, rn, level)
        recv = comm.row_alltoall(y)
        front, stats = engine.merge(recv, level + 1)
        f, mf, dmu = comm.allreduce(stats)
        mu -= dmu
        if f == 0:
            return level + 1
        level += 1


DIST_WIDE = 0x100   # tsmv.DIST_WIDE (late pull levels); a constant here so CPU engines need no libtsmv


def sim_degrees(A, engines: Sequence[Dist2DBFS]):
    """Global degrees of every simulated rank's vertices from the whole A."""
    dev = engines[0].device
    outdeg = torch.bincount(A.col_idx.to(dev, torch.int64), minlength=A.n).to(torch.int32)
    indeg = (A.row_ptr[1:] - A.row_ptr[:-1]).to(dev, torch.int32)
    for e in engines:
        e.set_degrees(outdeg[e.own0:e.own0 + e.nown], indeg[e.own0:e.own0 + e.nown], A.nnz)


def sim_bfs2d(engines: Sequence[Dist2DBFS], source: int, trace: Optional[list] = None) -> int:
    """`bfs2d_loop` for P simulated ranks on one GPU (exchanges by concatenation /
    slicing, what the collectives return).  trace: per level (dir, max expand ms,
    max merge ms) when given.  Returns the number of levels."""
    g = engines[0].grid
    Pr, Pc, sw = g.Pr, g.Pc, g.sw
    fronts = [e.begin(source) for e in engines]
    f, mf, dmu = (int(x) for x in sum(e.stats for e in engines).tolist())
    nnz_total = engines[0].nnz_total
    mu = nnz_total - dmu
    level = 0
    fprev = 0
    while True:
        xs = [torch.cat([fronts[g.rank_of(i, j)] for i in range(Pr)]) for j in range(Pc)]
        rows = [torch.cat([fronts[g.rank_of(i, j)] for j in range(Pc)]) for i in range(Pr)] \
            if engines[0].needs_rows else [None] * Pr
        d = engines[0].choose(f, mf, mu, fprev)
        fprev = f
        if nnz_total > 0 and mu * 4 < nnz_total:
            d |= DIST_WIDE
        te, tm, ys = [], [], []
        for e in engines:
            if trace is not None:
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
            ys.append(e.expand(xs[e.j], d, rows[e.i], level).clone())
            if trace is not None:
                b.record()
                torch.cuda.synchronize()
                te.append(a.elapsed_time(b))
        tot = torch.zeros(3, dtype=torch.int64, device=engines[0].device)
        for e in engines:
            recv = torch.cat([ys[g.rank_of(e.i, jj)][e.j * sw:(e.j + 1) * sw] for jj in range(Pc)])
            if trace is not None:
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
            fr, st = e.merge(recv, level + 1)
            if trace is not None:
                b.record()
                torch.cuda.synchronize()
                tm.append(a.elapsed_time(b))
            fronts[e.rank] = fr.clone()
            tot += st
        f, mf, dmu = (int(x) for x in tot.tolist())
        mu -= dmu
        if trace is not None:
            trace.append({"dir": d & 3, "expand_max": max(te), "merge_max": max(tm), "f": f})
        if f == 0:
            return level + 1
        level += 1


def gather_levels(engines: Sequence[Dist2DBFS]) -> torch.Tensor:
    """Global levels from simulated ranks (pieces are in vertex order)."""
    return torch.cat([e.owned_levels() for e in sorted(engines, key=lambda e: e.rank)])
