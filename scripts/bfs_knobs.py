"""TileBFS direction-rule knobs on B200 (R9: Pull-CSC if m_f > m_u / alpha, else
Push-CSR if |F|/n >= push_csr_density, else Push-CSC): traversal time per
(density threshold, alpha) on the BASELINE BFS graphs; per-level time summary.
usage: python scripts/bfs_knobs.py [graphs] [dens:alpha,...]"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

dev = torch.device("cuda", 0)
which = (sys.argv[1] if len(sys.argv) > 1 else "c1,3d,band,rmat").split(",")
knobs = [(float(a), float(b)) for a, b in (kv.split(":") for kv in (sys.argv[2] if len(sys.argv) > 2 else "0.01:14,0.05:14,0.2:14,2:14,0.01:4,0.01:40,2:40,2:1e9").split(","))]
w = torch.empty(64 << 20, dtype=torch.float32, device=dev)
for g in which:
    if g == "c1":
        A, srcs, thr = synth.stencil2d(64, 64, device=dev), [0], 2
    elif g == "3d":
        A, srcs, thr = synth.stencil3d(256, device=dev), [0], 2
    elif g == "band":
        A, srcs, thr = synth.banded(1 << 20, 64, device=dev), [0], 2
    else:
        A = synth.rmat(22, 16, seed=1, symmetrize=True, device=dev)
        srcs, thr = [0] + synth.sample_sources(A, 3, seed=1), 8
    for dens, alpha in knobs:
        M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", sparse_tile_max_nnz=thr, push_csr_density=dens,
                                      pull_alpha=alpha)
        M.bfs(srcs[0])
        ts, dirs, lv = [], "", []
        for s in srcs:
            w.zero_()
            torch.cuda.synchronize()
            _, st = M.bfs(s)
            ts.append(st["ms"])
            if not dirs:
                dirs = "".join({"push_csc": "C", "push_csr": "R", "pull_csc": "P"}.get(d, "?") for d in st["dirs"])
                lv = st["level_ms"]
        M.close()
        d = dirs if len(dirs) <= 24 else f"{dirs[:12]}..{dirs[-8:]} ({len(dirs)} levels, C {dirs.count('C')} R {dirs.count('R')} P {dirs.count('P')})"
        print(f"{g:5s} dens {dens:<5g} alpha {alpha:<6g}: ms {statistics.mean(ts):8.3f}  level ms median {statistics.median(lv) * 1e3:7.2f} us  max {max(lv):.4f}  dirs {d}", flush=True)
