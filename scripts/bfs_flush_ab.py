"""TileBFS device time with the L2 flushed before every traversal (the bench
protocol), under environment switches read per call by libtsmv.  Dev aid.
usage: python scripts/bfs_flush_ab.py band20_64|grid3d256|grid2d64|rmat22 [ENV=V,...] ..."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

dev = torch.device("cuda", 0)
name = sys.argv[1]
if name.startswith("rmat"):
    A = synth.rmat(int(name[4:]), 16, seed=1, symmetrize=True, device=dev)
elif name.startswith("grid3d"):
    A = synth.stencil3d(int(name[6:]), device=dev)
elif name.startswith("grid2d"):
    g = int(name[6:])
    A = synth.stencil2d(g, g, device=dev)
else:
    n, b = name[4:].split("_")
    A = synth.banded(1 << int(n), int(b), device=dev)
M = tsmv.TiledMatrix.from_csr(A)
w = torch.empty(64 << 20, dtype=torch.float32, device=dev)
r = torch.ones(64 << 20, dtype=torch.float32, device=dev)
lv = torch.empty(A.n, dtype=torch.int32, device=dev)
for conf in sys.argv[2:] or [""]:
    env = dict(kv.split("=") for kv in conf.split(",") if kv)
    os.environ.update(env)
    M.bfs(0, levels=lv)
    ts = []
    for _ in range(3):
        w.zero_()
        _ = r.sum()
        torch.cuda.synchronize()
        _, st = M.bfs(0, levels=lv)
        ts.append(st["ms"])
    for k in env:
        os.environ.pop(k, None)
    print(f"{name} {conf or 'default':24s} ms {[round(t, 3) for t in ts]}", flush=True)
