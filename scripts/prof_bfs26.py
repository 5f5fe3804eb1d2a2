"""One TileBFS traversal on R-MAT s26 (symmetrised, thr 8, as bench.py's bfs_s26)
from a given source, for ncu captures of its pull kernels.  Dev aid."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

dev = torch.device("cuda", 0)
src = int(sys.argv[1]) if len(sys.argv) > 1 else 23860436
A = synth.rmat(26, 16, seed=1, symmetrize=True, device=dev)
torch.cuda.empty_cache()
M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", sparse_tile_max_nnz=8)
del A
torch.cuda.empty_cache()
_, st = M.bfs(src)
torch.cuda.synchronize()
print("ms", st["ms"], st["dirs"], flush=True)
