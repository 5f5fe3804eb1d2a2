"""Phase breakdown of y = A x on a named config (dev aid).  usage: t_cfg.py grid3d256|band20_64|rmat22 [density]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
from paper_conf_icpp_jisl0t022_b200 import tsmv
dev = torch.device("cuda", 0)
w = torch.empty(64 << 20, dtype=torch.float32, device=dev); r = torch.ones(64 << 20, dtype=torch.float32, device=dev)
name = sys.argv[1]; d = float(sys.argv[2]) if len(sys.argv) > 2 else 0.01
if name.startswith("grid3d"): A = synth.stencil3d(int(name[6:]), device=dev)
elif name.startswith("band"):
    n, b = name[4:].split("_"); A = synth.banded(1 << int(n), int(b), device=dev)
else: A = synth.attach_values(synth.rmat(int(name[4:]), 16, seed=1, device=dev), seed=1)
M = tsmv.TiledMatrix.from_csr(A, build_bfs=0)
k = max(1, synth.density_k(A.n, d))
xs = [synth.sample_x(A.n, k, seed=s, device=dev) for s in range(1, 10)]
yi = torch.empty(A.m, dtype=torch.int32, device=dev); yv = torch.empty(A.m, dtype=torch.float64, device=dev)
yn = torch.zeros(1, dtype=torch.int64, device=dev)
for xi, xv in xs[:3]: M.spmspv_async(xi, xv, yi, yv, yn)
torch.cuda.synchronize(); M.set_timing(True); ts = []
for xi, xv in xs[3:]:
    w.zero_(); _ = r.sum()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); M.spmspv_async(xi, xv, yi, yv, yn); e1.record(); torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1) * 1e3)
kt, n = M.get_timing(); st = M.last_call_stats()
print(name, d, "k", k, "median us", sorted(ts)[len(ts)//2], "phases(A,B,C,all)", [round(x / n * 1e3, 1) for x in kt], st)
