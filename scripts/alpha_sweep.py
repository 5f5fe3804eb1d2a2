"""TileBFS harmonic-mean GTEPS on R-MAT sym over the bench's sources for several
pull_alpha values (direction rule R9), L2 flushed before every traversal.  Dev aid.
usage: python scripts/alpha_sweep.py scale nsources alpha,alpha,... [push_csr_density,...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

dev = torch.device("cuda", 0)
sc, ns = int(sys.argv[1]), int(sys.argv[2])
alphas = [float(a) for a in sys.argv[3].split(",")]
denss = [float(a) for a in sys.argv[4].split(",")] if len(sys.argv) > 4 else [0.05]
A = synth.rmat(sc, 16, seed=1, symmetrize=True, device=dev)
srcs = [0] + synth.sample_sources(A, ns - 1, seed=1)
torch.cuda.empty_cache()
w = torch.empty(64 << 20, dtype=torch.float32, device=dev)
lv = torch.empty(A.n, dtype=torch.int32, device=dev)
M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", sparse_tile_max_nnz=8)
for al, de in [(a, d) for a in alphas for d in denss]:
    M.set_direction_rule(pull_alpha=al, push_csr_density=de)
    M.bfs(srcs[0], levels=lv)
    g, ms = [], []
    for s in srcs:
        w.zero_()
        torch.cuda.synchronize()
        _, st = M.bfs(s, levels=lv)
        g.append(st["edges_traversed"] / (st["ms"] * 1e-3) / 1e9)
        ms.append(round(st["ms"], 2))
    hm = len(g) / sum(1 / x for x in g)
    print(f"s{sc} alpha {al:6g} dens {de:5g}: hmean {hm:7.1f} GTEPS  ms {ms}", flush=True)
