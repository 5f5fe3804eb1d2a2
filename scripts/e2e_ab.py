"""End-to-end tsmv_spmspv with pinned host x / y (the bench's e2e protocol) under
environment switches (e.g. TSMV_Y_COPY=1).  Dev aid.
usage: python scripts/e2e_ab.py [scale] [density] [ENV=V,...] ..."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

dev = torch.device("cuda", 0)
sc = int(sys.argv[1]) if len(sys.argv) > 1 else 22
dens = float(sys.argv[2]) if len(sys.argv) > 2 else 0.01
A = synth.attach_values(synth.rmat(sc, 16, seed=1, device=dev), seed=1)
M = tsmv.TiledMatrix.from_csr(A, build_bfs=0)
k = synth.density_k(A.n, dens)
hx = [tuple(t.cpu().pin_memory() for t in synth.sample_x(A.n, k, seed=s)) for s in range(1, 24)]
hy_i = torch.empty(M.m, dtype=torch.int32).pin_memory()
hy_v = torch.empty(M.m, dtype=torch.float64).pin_memory()
w = torch.empty(64 << 20, dtype=torch.float32, device=dev)
ref = None
for conf in sys.argv[3:] or [""]:
    env = dict(kv.split("=") for kv in conf.split(",") if kv)
    os.environ.update(env)
    for xi, xv in hx[:3]:
        M.spmspv(xi, xv, y_idx=hy_i, y_val=hy_v)
    ts = []
    for xi, xv in hx[3:]:
        w.zero_()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        yi, yv = M.spmspv(xi, xv, y_idx=hy_i, y_val=hy_v)
        ts.append((time.perf_counter() - t0) * 1e6)
    got = (yi.clone(), yv.clone())
    if ref is None:
        ref = got
    same = torch.equal(ref[0], got[0]) and torch.equal(ref[1], got[1])
    for kk in env:
        os.environ.pop(kk, None)
    ts.sort()
    print(f"s{sc} d={dens} {conf or 'default':16s} e2e median {ts[len(ts) // 2]:7.1f} us  min {ts[0]:7.1f}  "
          f"mean {sum(ts) / len(ts):7.1f}  y_nnz {yi.numel()}  same_as_first {same}", flush=True)
