"""SpMSpV device time at T per tile size / side-matrix threshold (the format knobs;
results are invariant).  L2 flushed before each call.  Dev aid.
usage: python scripts/ab_thr.py [scale] [density] nt:thr ..."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

dev = torch.device("cuda", 0)
sc = int(sys.argv[1]) if len(sys.argv) > 1 else 22
d = float(sys.argv[2]) if len(sys.argv) > 2 else 0.01
A = synth.attach_values(synth.rmat(sc, 16, seed=1, device=dev), seed=1)
k = synth.density_k(A.n, d)
xs = [synth.sample_x(A.n, k, seed=s, device=dev) for s in range(1, 19)]
w = torch.empty(64 << 20, dtype=torch.float32, device=dev)
yi = torch.empty(A.m, dtype=torch.int32, device=dev)
yv = torch.empty(A.m, dtype=torch.float64, device=dev)
yn = torch.zeros(1, dtype=torch.int64, device=dev)
for spec in sys.argv[3:] or ["16:2"]:
    nt, thr = (int(v) for v in spec.split(":"))
    M = tsmv.TiledMatrix.from_csr(A, tile_dim=nt, sparse_tile_max_nnz=thr, build_bfs=0)
    for xi, xv in xs[:3]:
        M.spmspv_async(xi, xv, yi, yv, yn)
    ts = []
    for xi, xv in xs[3:]:
        w.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        M.spmspv_async(xi, xv, yi, yv, yn)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    ts.sort()
    print(f"s{sc} d={d} nt {nt} thr {thr}: median {ts[len(ts) // 2]:.1f} us  min {ts[0]:.1f}", flush=True)
    M.close()
    torch.cuda.empty_cache()
