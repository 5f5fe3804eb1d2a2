"""Small calls of every kernel family for compute-sanitizer (memcheck / racecheck /
synccheck): flat SpMSpV (C1 shape, R-MAT s12 at 1 % and 10 %, three semirings),
fused + host-loop TileBFS, parents, multi-source BFS.  Dev aid:
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
torch.cuda.synchronize()
print("sanitize_small done")
