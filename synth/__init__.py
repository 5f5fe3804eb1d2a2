"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

This module holds NO arithmetic of the method (no tiling, no SpMSpV, no BFS).
It only produces the inputs: CSR matrices shaped like the paper's workloads
(SuiteSparse-like power-law, stencil, banded, uniform; §4.1
P:1682-1690) and sparse vectors "generated randomly with random seeds 1"
(P:1762-1764).  DESIGN.md §"Input recipe" states the recipe.

Randomness is a counter-based hash (SplitMix64 of (seed, stream, counter)),
evaluated with wrapping int64 torch arithmetic, so the same call yields the
same matrix on CPU and on CUDA.  `hash_u64_ref` is a pure-Python copy used by
the tests to check the vectorised one.
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import Optional

import torch

_M64 = (1 << 64) - 1
_GOLDEN = 0x9E3779B97F4A7C15
_C1 = 0xBF58476D1CE4E5B9
_C2 = 0x94D049BB133111EB

# streams (independent hash families)
S_RMAT = 1
S_XIDX = 3
S_XVAL = 4
S_AVAL = 5
S_UNIF = 6
S_SRC = 7
S_PERM = 8   # .. 10: vertex permutation rounds


def _s64(c: int) -> int:
    c &= _M64
    return c - (1 << 64) if c >= (1 << 63) else c


def _splitmix_py(z: int) -> int:
    z = (z + _GOLDEN) & _M64
    z = ((z ^ (z >> 30)) * _C1) & _M64
    z = ((z ^ (z >> 27)) * _C2) & _M64
    return z ^ (z >> 31)


def _key(seed: int, stream: int) -> int:
    return _splitmix_py(((seed & 0xFFFFFFFF) << 20) ^ stream)


def hash_u64_ref(seed: int, stream: int, counter: int) -> int:
    """Pure-Python reference of `hash_u64` (returns an unsigned 64-bit int)."""
    return _splitmix_py((counter * _GOLDEN + _key(seed, stream)) & _M64)


def _lsr(z: torch.Tensor, s: int) -> torch.Tensor:
    # logical right shift on int64 tensors
    return (z >> s) & ((1 << (64 - s)) - 1)


def hash_u64(seed: int, stream: int, counter: torch.Tensor) -> torch.Tensor:
    """SplitMix64((counter*golden + key(seed,stream))) as int64 bit patterns."""
    z = counter.to(torch.int64) * _s64(_GOLDEN) + _s64(_key(seed, stream))
    z = z + _s64(_GOLDEN)
    z = (z ^ _lsr(z, 30)) * _s64(_C1)
    z = (z ^ _lsr(z, 27)) * _s64(_C2)
    return z ^ _lsr(z, 31)


def unit24(h: torch.Tensor) -> torch.Tensor:
    """Top 24 bits as an integer in [0, 2^24)."""
    return _lsr(h, 40)


def unit53(h: torch.Tensor) -> torch.Tensor:
    """Top 53 bits as a float64 in [0, 1)."""
    return _lsr(h, 11).to(torch.float64) * (1.0 / (1 << 53))


@dataclass
class CSR:
    """A CSR matrix: row_ptr int64[m+1], col_idx int32[nnz] (sorted, unique per
    row), values float64/float32[nnz] or None (pattern)."""
    m: int
    n: int
    row_ptr: torch.Tensor
    col_idx: torch.Tensor
    values: Optional[torch.Tensor]
    name: str = ""

    @property
    def nnz(self) -> int:
        return int(self.col_idx.numel())

    def to(self, device) -> "CSR":
        return CSR(self.m, self.n, self.row_ptr.to(device), self.col_idx.to(device),
                   None if self.values is None else self.values.to(device), self.name)

    def with_values(self, values: Optional[torch.Tensor]) -> "CSR":
        return CSR(self.m, self.n, self.row_ptr, self.col_idx, values, self.name)

    def rows(self) -> torch.Tensor:
        """Row id of every stored entry (int64)."""
        counts = self.row_ptr[1:] - self.row_ptr[:-1]
        return torch.repeat_interleave(
            torch.arange(self.m, device=self.row_ptr.device, dtype=torch.int64), counts)


_UNIQUE_MAX = 1 << 30   # torch.unique (CUB) refuses >= 2^31 elements


def _unique_sorted(keys: torch.Tensor, lo: int, hi: int) -> torch.Tensor:
    """Sorted distinct values of `keys` (all in [lo, hi)); large inputs are split
    by value range (R-MAT scale 26 symmetrised has ~2^31 keys)."""
    if keys.numel() <= _UNIQUE_MAX or hi - lo < 2:
        return torch.unique(keys, sorted=True)
    mid = (lo + hi) // 2
    sel = keys < mid
    left = keys[sel]
    right = keys[~sel]
    del sel, keys
    a = _unique_sorted(left, lo, mid)
    del left
    b = _unique_sorted(right, mid, hi)
    del right
    return torch.cat([a, b])


def csr_from_keys(keys: torch.Tensor, m: int, n: int, name: str = "") -> CSR:
    """keys = row*n + col, any order, duplicates allowed -> pattern CSR
    (duplicates coalesced, columns ascending)."""
    keys = _unique_sorted(keys.to(torch.int64), 0, m * n)
    rows = torch.div(keys, n, rounding_mode="floor")
    cols = (keys - rows * n).to(torch.int32)
    del keys
    counts = torch.bincount(rows, minlength=m)
    row_ptr = torch.zeros(m + 1, dtype=torch.int64, device=cols.device)
    row_ptr[1:] = torch.cumsum(counts, 0)
    return CSR(m, n, row_ptr, cols, None, name)


def attach_values(A: CSR, seed: int = 1, dtype: str = "f64", integer: bool = False) -> CSR:
    """Values v(i,j) = 1 + u(i,j) (u from the hash of the flat index), or, with
    integer=True, nonzero integers in [-1024,-1] U [1,1024] (exact in fp32/fp64
    under any summation order of <= 2^20 terms)."""
    rows = A.rows()
    flat = rows * A.n + A.col_idx.to(torch.int64)
    h = hash_u64(seed, S_AVAL, flat)
    if integer:
        mag = (_lsr(h, 20) % 1024) + 1
        sign = torch.where((_lsr(h, 63) & 1) == 1, -1, 1)
        v = (mag * sign).to(torch.float64)
    else:
        v = 1.0 + unit53(h)
    if dtype == "f32":
        v = v.to(torch.float32)
    return A.with_values(v)


# --------------------------------------------------------------------------- matrices

def permute_bits(v: torch.Tensor, bits: int, seed: int = 1) -> torch.Tensor:
    """A seeded bijection of [0, 2^bits): three rounds of (x * odd) mod 2^bits and
    x ^= x >> ceil(bits/2) (each invertible on bits-bit integers)."""
    mask = (1 << bits) - 1
    x = v.to(torch.int64) & mask
    sh = max(1, (bits + 1) // 2)
    for rnd in range(3):
        odd = (_key(seed, S_PERM + rnd) | 1) & 0x7FFFFFFFFFFF
        x = (x * odd) & mask
        x = x ^ (x >> sh)
    return x


def rmat(scale: int, edgefactor: int = 16, a: float = 0.57, b: float = 0.19, c: float = 0.19,
         seed: int = 1, symmetrize: bool = False, device="cpu", chunk: int = 1 << 24,
         permute: bool = False) -> CSR:
    """R-MAT / Kronecker power-law graph (Graph500 parameters by default), no
    vertex permutation, duplicate edges coalesced.  Edge j->i is stored as A[i, j]
    ... here we simply store generated tuple (r, c) as A[r, c]; with
    symmetrize=True the union with the transpose is taken."""
    n = 1 << scale
    E = edgefactor * n
    ta = int(a * (1 << 24))
    tab = int((a + b) * (1 << 24))
    tabc = int((a + b + c) * (1 << 24))
    parts = []
    for e0 in range(0, E, chunk):
        e = torch.arange(e0, min(E, e0 + chunk), device=device, dtype=torch.int64)
        r = torch.zeros_like(e)
        cc = torch.zeros_like(e)
        for lvl in range(scale):
            u = unit24(hash_u64(seed, S_RMAT, e * scale + lvl))
            rb = u >= tab
            cb = ((u >= ta) & (u < tab)) | (u >= tabc)
            r |= rb.to(torch.int64) << lvl
            cc |= cb.to(torch.int64) << lvl
        if permute:  # Graph500-style vertex relabelling: hubs no longer sit at low ids
            r = permute_bits(r, scale, seed)
            cc = permute_bits(cc, scale, seed)
        parts.append(r * n + cc)
        if symmetrize:
            parts.append(cc * n + r)
    keys = torch.cat(parts)
    del parts
    return csr_from_keys(keys, n, n, f"rmat_s{scale}_ef{edgefactor}{'_sym' if symmetrize else ''}"
                         f"{'_perm' if permute else ''}")


def stencil2d(nx: int, ny: int, device="cpu") -> CSR:
    """2D 5-point Laplacian on an nx-by-ny grid, natural order v = i*ny + j;
    diagonal 4, neighbours -1."""
    n = nx * ny
    v = torch.arange(n, device=device, dtype=torch.int64)
    i, j = v // ny, v % ny
    cand = [(v - ny, i > 0, -1.0), (v - 1, j > 0, -1.0), (v, torch.ones_like(v, dtype=torch.bool), 4.0),
            (v + 1, j < ny - 1, -1.0), (v + ny, i < nx - 1, -1.0)]
    return _from_candidates(n, v, cand, f"stencil2d_{nx}x{ny}")


def stencil3d(k: int, device="cpu") -> CSR:
    """3D 7-point Laplacian on a k^3 grid, v = (i*k + j)*k + l; diagonal 6, neighbours -1."""
    n = k ** 3
    v = torch.arange(n, device=device, dtype=torch.int64)
    i, j, l = v // (k * k), (v // k) % k, v % k
    t = torch.ones_like(v, dtype=torch.bool)
    cand = [(v - k * k, i > 0, -1.0), (v - k, j > 0, -1.0), (v - 1, l > 0, -1.0), (v, t, 6.0),
            (v + 1, l < k - 1, -1.0), (v + k, j < k - 1, -1.0), (v + k * k, i < k - 1, -1.0)]
    return _from_candidates(n, v, cand, f"stencil3d_{k}")


def _from_candidates(n, v, cand, name) -> CSR:
    cols = torch.stack([c for c, _, _ in cand], 1)
    ok = torch.stack([m for _, m, _ in cand], 1)
    vals = torch.tensor([x for _, _, x in cand], dtype=torch.float64, device=v.device).expand_as(cols)
    counts = ok.sum(1)
    row_ptr = torch.zeros(n + 1, dtype=torch.int64, device=v.device)
    row_ptr[1:] = torch.cumsum(counts, 0)
    return CSR(n, n, row_ptr, cols[ok].to(torch.int32), vals[ok].contiguous(), name)


def banded(n: int, b: int, device="cpu", seed: int = 1) -> CSR:
    """Full band of half-bandwidth b: A[i,j] stored iff |i-j| <= b; values 1+u."""
    v = torch.arange(n, device=device, dtype=torch.int64)
    lo = torch.clamp(v - b, min=0)
    hi = torch.clamp(v + b, max=n - 1)
    counts = hi - lo + 1
    row_ptr = torch.zeros(n + 1, dtype=torch.int64, device=device)
    row_ptr[1:] = torch.cumsum(counts, 0)
    rows = torch.repeat_interleave(v, counts)
    cols = lo[rows] + (torch.arange(rows.numel(), device=device) - row_ptr[rows])
    A = CSR(n, n, row_ptr, cols.to(torch.int32), None, f"banded_{n}_b{b}")
    return attach_values(A, seed)


def uniform(m: int, n: int, per_row: int, seed: int = 1, device="cpu") -> CSR:
    """Erdos-Renyi-like: per_row uniform columns per row, duplicates coalesced."""
    e = torch.arange(m * per_row, device=device, dtype=torch.int64)
    cols = _lsr(hash_u64(seed, S_UNIF, e), 11) % n
    rows = e // per_row
    return csr_from_keys(rows * n + cols, m, n, f"uniform_{m}x{n}_{per_row}")


def from_dense_pattern(D: torch.Tensor, values: bool = True) -> CSR:
    """Tiny helper for hand-written test matrices (D: 2-D tensor, nonzero = stored)."""
    m, n = D.shape
    nzr, nzc = torch.nonzero(D, as_tuple=True)
    counts = torch.bincount(nzr, minlength=m)
    row_ptr = torch.zeros(m + 1, dtype=torch.int64)
    row_ptr[1:] = torch.cumsum(counts, 0)
    vals = D[nzr, nzc].to(torch.float64) if values else None
    return CSR(m, n, row_ptr, nzc.to(torch.int32), vals, "dense")


def from_edges(n: int, edges, symmetric: bool = True) -> CSR:
    """Pattern CSR from an explicit edge list [(i, j), ...] (A[i,j] stored)."""
    keys = []
    for i, j in edges:
        keys.append(i * n + j)
        if symmetric:
            keys.append(j * n + i)
    return csr_from_keys(torch.tensor(keys, dtype=torch.int64), n, n, "edges")


# --------------------------------------------------------------------------- vectors

def sample_x(n: int, k: int, seed: int = 1, device="cpu", dtype: str = "f64",
             integer: bool = False):
    """k distinct indices uniform without replacement (ascending), values 1+u
    (or nonzero integers in [-1024,1024] with integer=True).  Returns
    (idx int32[k], val float64/float32[k])."""
    k = int(k)
    if k == 0:
        idx = torch.zeros(0, dtype=torch.int64, device=device)
    elif k >= n:
        idx = torch.arange(n, device=device, dtype=torch.int64)
    else:
        keys = _lsr(hash_u64(seed, S_XIDX, torch.arange(n, device=device, dtype=torch.int64)), 1)
        idx = torch.topk(keys, k, largest=False, sorted=False).indices
        idx, _ = torch.sort(idx)
    h = hash_u64(seed, S_XVAL, idx)
    if integer:
        mag = (_lsr(h, 20) % 1024) + 1
        sign = torch.where((_lsr(h, 63) & 1) == 1, -1, 1)
        val = (mag * sign).to(torch.float64)
    else:
        val = 1.0 + unit53(h)
    if dtype == "f32":
        val = val.to(torch.float32)
    return idx.to(torch.int32), val


def sample_sources(A: CSR, count: int, seed: int = 1):
    """`count` distinct vertices with nonzero out-degree (column count), chosen by hash order."""
    deg = torch.bincount(A.col_idx.to(torch.int64), minlength=A.n)
    cand = torch.nonzero(deg > 0).flatten()
    keys = _lsr(hash_u64(seed, S_SRC, cand), 1)
    order = torch.argsort(keys)
    return cand[order[:count]].tolist()


def density_k(n: int, density: float) -> int:
    return int(round(density * n))
