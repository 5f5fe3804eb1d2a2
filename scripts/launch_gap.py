"""Where do the us between the events and the flat kernel's own globaltimer span go?
Times one y = A x at T under: L2 flush before (bench rule) vs none; a tiny torch
kernel between flush and events; persistence window on/off.  Dev aid."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
from paper_conf_icpp_jisl0t022_b200 import tsmv
dev = torch.device("cuda", 0)
w = torch.empty(64 << 20, dtype=torch.float32, device=dev); r = torch.ones(64 << 20, dtype=torch.float32, device=dev)
small = torch.zeros(1024, device=dev)
A = synth.attach_values(synth.rmat(22, 16, seed=1, device=dev), seed=1)
M = tsmv.TiledMatrix.from_csr(A, build_bfs=0)
k = synth.density_k(A.n, 0.01)
xs = [synth.sample_x(A.n, k, seed=s, device=dev) for s in range(1, 24)]
yi = torch.empty(A.m, dtype=torch.int32, device=dev); yv = torch.empty(A.m, dtype=torch.float64, device=dev)
yn = torch.zeros(1, dtype=torch.int64, device=dev)
for xi, xv in xs[:3]: M.spmspv_async(xi, xv, yi, yv, yn)
torch.cuda.synchronize()

def run(label, pre, what="call"):
    ts = []
    M.set_timing(True)
    for xi, xv in xs[3:]:
        pre()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        if what == "call": M.spmspv_async(xi, xv, yi, yv, yn)
        else: small.add_(1.0)
        e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    kt, n = M.get_timing(); M.set_timing(False)
    ts.sort()
    inner = kt[3] / max(n, 1) * 1e3 if what == "call" else 0
    print(f"{label:40s} event median {ts[len(ts)//2]:7.1f} us  min {ts[0]:7.1f}  kernel-internal {inner:6.1f} us", flush=True)

def flush(): w.zero_(); _ = r.sum()
def flush_small(): flush(); small.add_(1.0)
def nothing(): pass
run("flush + call", flush)
run("no flush + call", nothing)
run("flush + tiny kernel + call", flush_small)
run("flush + tiny kernel only", flush, what="tiny")
run("no flush + tiny kernel only", nothing, what="tiny")
