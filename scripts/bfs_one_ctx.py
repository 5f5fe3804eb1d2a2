"""One TileBFS traversal from vertex 0 on the bench's C3 context (R-MAT s22
symmetrised, pattern, thr from bench.py) after one warm-up, for ncu launch lists.  Dev aid."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

cfg = bench.parse([])
dev = torch.device("cuda", 0)
A = synth.rmat(cfg.bfs_scale, 16, seed=1, symmetrize=True, device=dev)
M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", sparse_tile_max_nnz=cfg.bfs_thr)
src = int(sys.argv[1]) if len(sys.argv) > 1 else 0
M.bfs(src)
torch.cuda.synchronize()
_, st = M.bfs(src)
print("ms", st["ms"], "dirs", st["dirs"], "level_ms", [round(x, 4) for x in st["level_ms"]])
