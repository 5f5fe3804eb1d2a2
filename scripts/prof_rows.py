"""Small calls of the row-driven SpMSpV kernel for ncu (3D stencil, 1 %).  Dev aid."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["TSMV_SPMSPV_KERNEL"] = sys.argv[2] if len(sys.argv) > 2 else "rows"
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

dev = torch.device("cuda", 0)
A = synth.stencil3d(int(sys.argv[1]) if len(sys.argv) > 1 else 256, device=dev)
M = tsmv.TiledMatrix.from_csr(A, build_bfs=0)
k = synth.density_k(A.n, 0.01)
for s in range(1, 6):
    xi, xv = synth.sample_x(A.n, k, seed=s, device=dev)
    M.spmspv(xi, xv)
torch.cuda.synchronize()
print("done")
