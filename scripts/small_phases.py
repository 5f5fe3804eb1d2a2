import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
from paper_conf_icpp_jisl0t022_b200 import tsmv
dev = torch.device("cuda", 0)
A = synth.stencil2d(64, 64, device=dev)
M = tsmv.TiledMatrix.from_csr(A)
xs = [synth.sample_x(A.n, 41, seed=s, device=dev) for s in range(1, 20)]
yi = torch.empty(A.m, dtype=torch.int32, device=dev); yv = torch.empty(A.m, dtype=torch.float64, device=dev); yn = torch.zeros(1, dtype=torch.int64, device=dev)
for xi, xv in xs[:3]: M.spmspv_async(xi, xv, yi, yv, yn)
torch.cuda.synchronize()
M.set_timing(True)
for xi, xv in xs[3:]:
    M.spmspv_async(xi, xv, yi, yv, yn); torch.cuda.synchronize()
kt, n = M.get_timing()
print("C1 phases us:", [round(x / n * 1e3, 1) for x in kt], M.info()["n_dense_tiles"])
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for xi, xv in xs[3:]: M.spmspv_async(xi, xv, yi, yv, yn)
e1.record(); torch.cuda.synchronize()
print("C1 back-to-back us/call:", e0.elapsed_time(e1) * 1e3 / len(xs[3:]))
