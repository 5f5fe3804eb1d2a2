"""TileBFS on R-MAT s22 (symmetrised) as bench.py runs it (sparse_tile_max_nnz 8,
L2 flushed before the traversal), source 0, for an ncu launch list.  Dev aid."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

dev = torch.device("cuda", 0)
sc = int(sys.argv[1]) if len(sys.argv) > 1 else 22
A = synth.rmat(sc, 16, seed=1, symmetrize=True, device=dev)
M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", sparse_tile_max_nnz=8)
w = torch.empty(64 << 20, dtype=torch.float32, device=dev)
for _ in range(3):
    w.zero_()
    torch.cuda.synchronize()
    _, st = M.bfs(0)
torch.cuda.synchronize()
print("levels", st["nlevels"], "ms", st["ms"], "dirs", st.get("dirs"), flush=True)
