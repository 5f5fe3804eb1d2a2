"""Per-kernel timing sweep of tsmv_spmspv on R-MAT (development aid, not the bench).

usage: python scripts/sweep.py [scale] [thr,...] [density,...] [nt]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

scale = int(sys.argv[1]) if len(sys.argv) > 1 else 22
thrs = [int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "2").split(",")]
dens = [float(x) for x in (sys.argv[3] if len(sys.argv) > 3 else "0.01").split(",")]
nt = int(sys.argv[4]) if len(sys.argv) > 4 else 16
srs = (sys.argv[5] if len(sys.argv) > 5 else "plus_times").split(",")
dev = torch.device("cuda", 0)
A = synth.attach_values(synth.rmat(scale, 16, seed=1, device=dev), seed=1)
w = torch.empty(64 << 20, dtype=torch.float32, device=dev)
r = torch.ones(64 << 20, dtype=torch.float32, device=dev)
for thr in thrs:
    M = tsmv.TiledMatrix.from_csr(A, tile_dim=nt, sparse_tile_max_nnz=thr, build_bfs=0)
    for d, sr in [(d_, s_) for d_ in dens for s_ in srs]:
        k = synth.density_k(A.n, d)
        xs = [synth.sample_x(A.n, k, seed=s, device=dev) for s in range(1, 12)]
        yi = torch.empty(A.m, dtype=torch.int32, device=dev)
        yv = torch.empty(A.m, dtype=torch.float64, device=dev)
        yn = torch.zeros(1, dtype=torch.int64, device=dev)
        for xi, xv in xs[:3]:
            M.spmspv_async(xi, xv, yi, yv, yn, semiring=sr)
        torch.cuda.synchronize()
        M.set_timing(True)
        for xi, xv in xs[3:]:
            w.zero_()
            _ = r.sum()
            M.spmspv_async(xi, xv, yi, yv, yn, semiring=sr)
            torch.cuda.synchronize()
        kt, n = M.get_timing()
        st = M.last_call_stats()
        print(f"thr={thr} d={d} {sr[:4]} k={k}: xscan {kt[0]/n*1e3:7.1f}us expand {kt[1]/n*1e3:7.1f}us "
              f"compact {kt[2]/n*1e3:7.1f}us total {kt[3]/n*1e3:7.1f}us | tiles {st['tile_items']} "
              f"side {st['side_items']} hit {st['hit_tiles']} macs {st['tile_macs']} y {st['y_nnz']}", flush=True)
    M.close()
