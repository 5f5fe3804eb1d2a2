"""Small SpMSpV calls for ncu captures: C1 (2D 64x64, 1 %) or R-MAT s<scale> at density d."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
from paper_conf_icpp_jisl0t022_b200 import tsmv
dev = torch.device("cuda", 0)
which = sys.argv[1] if len(sys.argv) > 1 else "c1"
if which == "c1":
    A = synth.stencil2d(64, 64, device=dev); d = 0.01
else:
    A = synth.attach_values(synth.rmat(int(which), 16, seed=1, device=dev), seed=1); d = float(sys.argv[2])
M = tsmv.TiledMatrix.from_csr(A, build_bfs=0)
k = max(1, synth.density_k(A.n, d))
for s in range(1, 8):
    xi, xv = synth.sample_x(A.n, k, seed=s, device=dev)
    M.spmspv(xi, xv)
torch.cuda.synchronize()
print("done")
