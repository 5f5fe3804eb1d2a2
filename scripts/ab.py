"""A/B device timing of y = A x (SpMSpV) under environment switches read per call
by libtsmv (e.g. TSMV_NO_PREFETCH=1).  Dev aid.

usage: python scripts/ab.py [matrix] [density,...] [ENV=V,ENV2=V ...]
matrix: 22 (R-MAT scale), stencil3d:256, banded:20:64, stencil2d:64
Each configuration: median / min event time of 15 calls (L2 flushed before each),
per-phase globaltimer times of CTA 0 (A, B, C, whole)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

dev = torch.device("cuda", 0)
spec = sys.argv[1] if len(sys.argv) > 1 else "22"
dens = [float(d) for d in (sys.argv[2] if len(sys.argv) > 2 else "0.01").split(",")]
confs = sys.argv[3:] or [""]
w = torch.empty(64 << 20, dtype=torch.float32, device=dev)
r = torch.ones(64 << 20, dtype=torch.float32, device=dev)
if spec.startswith("stencil3d"):
    A = synth.stencil3d(int(spec.split(":")[1]), device=dev)
elif spec.startswith("banded"):
    _, lg, bw = spec.split(":")
    A = synth.banded(1 << int(lg), int(bw), device=dev)
elif spec.startswith("stencil2d"):
    g = int(spec.split(":")[1])
    A = synth.stencil2d(g, g, device=dev)
else:
    A = synth.attach_values(synth.rmat(int(spec), 16, seed=1, device=dev), seed=1)
scale = spec
M = tsmv.TiledMatrix.from_csr(A, build_bfs=0)
yi = torch.empty(A.m, dtype=torch.int32, device=dev)
yv = torch.empty(A.m, dtype=torch.float64, device=dev)
yn = torch.zeros(1, dtype=torch.int64, device=dev)
for d in dens:
    k = max(1, synth.density_k(A.n, d))
    xs = [synth.sample_x(A.n, k, seed=s, device=dev) for s in range(1, 19)]
    for conf in confs:
        env = dict(kv.split("=") for kv in conf.split(",") if kv)
        for kk, v in env.items():
            os.environ[kk] = v
        for xi, xv in xs[:3]:
            M.spmspv_async(xi, xv, yi, yv, yn)
        torch.cuda.synchronize()
        M.set_timing(True)
        ts = []
        for xi, xv in xs[3:]:
            w.zero_()
            _ = r.sum()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            M.spmspv_async(xi, xv, yi, yv, yn)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) * 1e3)
        kt, n = M.get_timing()
        M.set_timing(False)
        for kk in env:
            os.environ.pop(kk, None)
        ts.sort()
        print(f"s{scale} d={d:<7g} {conf or 'default':28s} median {ts[len(ts) // 2]:7.1f} us  min {ts[0]:7.1f}  "
              f"phases(A,B,C,all) {[round(x / n * 1e3, 1) for x in kt] if n else '-'}", flush=True)
