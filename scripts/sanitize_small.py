"""Small calls of every kernel family for compute-sanitizer (memcheck / racecheck /
synccheck): flat SpMSpV (C1 shape, R-MAT s12 at 1 % and 10 %, three semirings),
fused + host-loop TileBFS (solo levels, banded), parents, multi-source BFS, the
row-driven kernel, the distributed primitives (2 simulated ranks) and the 2D
block steps (2 x 2 simulated grid).  Dev aid:
  compute-sanitizer --tool racecheck python scripts/sanitize_small.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

dev = torch.device("cuda", 0)
A = synth.stencil2d(64, 64, device=dev)
M = tsmv.TiledMatrix.from_csr(A)
xi, xv = synth.sample_x(A.n, 41, seed=1, device=dev)
M.spmspv(xi, xv)
lv, _ = M.bfs(0)
M.bfs_parents(lv)
M.close()
A = synth.attach_values(synth.rmat(12, 16, seed=1, device=dev), seed=1)
M = tsmv.TiledMatrix.from_csr(A)
for d in (0.01, 0.1):
    xi, xv = synth.sample_x(A.n, synth.density_k(A.n, d), seed=2, device=dev)
    for sr in ("plus_times", "or_and", "min_second"):
        M.spmspv(xi, xv, semiring=sr)
M.close()
A = synth.rmat(12, 16, seed=1, symmetrize=True, device=dev)
M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", sparse_tile_max_nnz=8)
lv, _ = M.bfs(0)
M.bfs_parents(lv)
M.msbfs([0, 5, 9, 100])
os.environ["TSMV_BFS_HOSTLOOP"] = "1"
M.bfs(3)
os.environ.pop("TSMV_BFS_HOSTLOOP")
M.close()
# solo levels (banded, high diameter) and the row-driven SpMSpV kernel
A = synth.banded(1 << 12, 8, device=dev)
M = tsmv.TiledMatrix.from_csr(A)
M.bfs(0)
xi, xv = synth.sample_x(A.n, synth.density_k(A.n, 0.2), seed=3, device=dev)
M.spmspv(xi, xv)
M.close()
# distributed primitives: 2 simulated ranks (frontier scan, owned statistics, merge)
from paper_conf_icpp_jisl0t022_b200 import dist as D  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import dist2d as D2  # noqa: E402
A = synth.rmat(11, 16, seed=2, symmetrize=True, device=dev)
splits = D.partition_rows(A.row_ptr, 2)
E = [D.DistTiledMatrix(D.local_rows(A, splits, r), splits, r, 2, dtype="pattern") for r in range(2)]
deg = torch.bincount(A.col_idx.long(), minlength=A.n).to(torch.int32)
for e in E:
    e.set_degrees(deg)
st = [e.begin(0) for e in E]
g = torch.zeros(2 * E[0].stride, dtype=torch.int32, device=dev)
fprev = 0
while sum(x[0] for x in st) > 0:
    f, mf, mu = (sum(x[i] for x in st) for i in range(3))
    d = E[0].choose(E[0].n, f, mf, mu, fprev)
    fprev = f
    for p, e in enumerate(E):
        o = e.expand(d)
        g[p * E[0].stride:p * E[0].stride + o.numel()] = o
    st = [e.merge(g, E[0].stride) for e in E]
for e in E:
    e.M.close()
# 2D blocks, both modes
for mode in ("dopt", "push"):
    grid = D2.Grid2D(A.n, 2, 2, row_ptr=A.row_ptr, balance="nnz")
    E2 = [D2.Dist2DBFS(D2.block_2d(A, grid, *grid.coords(r)), grid, r, mode=mode) for r in range(4)]
    D2.sim_degrees(A, E2)
    D2.sim_bfs2d(E2, 0)
    for e in E2:
        e.close()
torch.cuda.synchronize()
print("sanitize_small done")
