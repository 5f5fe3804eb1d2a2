"""One TileBFS traversal for ncu captures: band (2^k, b), 3d (k), c1, rmat (scale).  Dev aid."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

dev = torch.device("cuda", 0)
g = sys.argv[1] if len(sys.argv) > 1 else "band"
if g == "band":
    A = synth.banded(1 << int(sys.argv[2]) if len(sys.argv) > 2 else 1 << 20, 64, device=dev)
elif g == "3d":
    A = synth.stencil3d(int(sys.argv[2]) if len(sys.argv) > 2 else 256, device=dev)
elif g == "c1":
    A = synth.stencil2d(64, 64, device=dev)
else:
    A = synth.rmat(int(sys.argv[2]) if len(sys.argv) > 2 else 22, 16, seed=1, symmetrize=True, device=dev)
M = tsmv.TiledMatrix.from_csr(A, dtype="pattern")
for _ in range(2):
    _, st = M.bfs(0)
torch.cuda.synchronize()
print("levels", st["nlevels"], "ms", st["ms"])
