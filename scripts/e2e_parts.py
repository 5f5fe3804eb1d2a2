"""Break down the end-to-end C-ABI call at T (pinned host x and y).  Dev aid."""
import ctypes, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
from paper_conf_icpp_jisl0t022_b200 import tsmv
dev = torch.device("cuda", 0)
A = synth.attach_values(synth.rmat(22, 16, seed=1, device=dev), seed=1)
M = tsmv.TiledMatrix.from_csr(A, build_bfs=0)
k = synth.density_k(A.n, 0.01)
xs = [synth.sample_x(A.n, k, seed=s) for s in range(1, 30)]
hx = [(a.pin_memory(), b.pin_memory()) for a, b in xs]
hyi, hyv = torch.empty(A.m, dtype=torch.int32).pin_memory(), torch.empty(A.m, dtype=torch.float64).pin_memory()
dyi, dyv = torch.empty(A.m, dtype=torch.int32, device=dev), torch.empty(A.m, dtype=torch.float64, device=dev)
dyn = torch.zeros(1, dtype=torch.int64, device=dev)
dx = [(a.to(dev), b.to(dev)) for a, b in xs]

def tm(f, n=20):
    for i in range(3): f(i)
    torch.cuda.synchronize()
    ts = []
    for i in range(n):
        t0 = time.perf_counter(); f(i); ts.append(time.perf_counter() - t0)
    ts.sort(); return 1e6 * ts[len(ts) // 2]

ynnz = ctypes.c_int64(0)
def full(i): M.spmspv(hx[i][0], hx[i][1], y_idx=hyi, y_val=hyv)
def raw(i):
    tsmv.tsmv_spmspv(M.ctx, 0, k, hx[i][0].data_ptr(), hx[i][1].data_ptr(), A.m, hyi.data_ptr(), hyv.data_ptr(),
                     ctypes.byref(ynnz), None)
def dev_only(i):
    M.spmspv_async(dx[i][0], dx[i][1], dyi, dyv, dyn); torch.cuda.synchronize()
def d2h(i):
    n = 243000
    hyi[:n].copy_(dyi[:n], non_blocking=True); hyv[:n].copy_(dyv[:n], non_blocking=True); torch.cuda.synchronize()
def dev_host_x(i):
    tsmv.tsmv_spmspv_async(M.ctx, 0, k, hx[i][0].data_ptr(), hx[i][1].data_ptr(), A.m, dyi.data_ptr(), dyv.data_ptr(),
                           dyn.data_ptr(), None); torch.cuda.synchronize()
for name, f in [("binding M.spmspv (pinned x, y)", full), ("raw ctypes tsmv_spmspv", raw),
                ("device x/y async + sync", dev_only), ("device y, pinned x (zero copy) + sync", dev_host_x),
                ("D2H 243K y entries (copy engine)", d2h)]:
    print(f"{name:42s} {tm(f):8.1f} us", flush=True)
