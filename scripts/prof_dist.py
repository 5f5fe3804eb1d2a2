"""One distributed-primitive traversal (simulated ranks) for an ncu launch list:
which kernels a level of tsmv_bfs_dist_expand / merge spends its time in.  Dev aid.

usage: python scripts/prof_dist.py [scale] [P] [source]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import dist as D  # noqa: E402

scale = int(sys.argv[1]) if len(sys.argv) > 1 else 24
P = int(sys.argv[2]) if len(sys.argv) > 2 else 1
dev = torch.device("cuda", 0)
A = synth.rmat(scale, 16, seed=1, symmetrize=True, device=dev)
src = int(sys.argv[3]) if len(sys.argv) > 3 else 0
splits = D.partition_rows(A.row_ptr, P)
engines = [D.DistTiledMatrix(D.local_rows(A, splits, r), splits, r, P, dtype="pattern",
                             sparse_tile_max_nnz=8) for r in range(P)]
deg = torch.bincount(A.col_idx.long(), minlength=A.n).to(torch.int32)
for e in engines:
    e.set_degrees(deg)
stride = engines[0].stride
gathered = torch.zeros(P * stride, dtype=torch.int32, device=dev)
for rep in range(2):
    torch.cuda.nvtx.range_push(f"traversal{rep}")
    st = [e.begin(src) for e in engines]
    lv, fprev = 0, 0
    while sum(x[0] for x in st) > 0:
        f, mf, mu = (sum(x[i] for x in st) for i in range(3))
        d = engines[0].choose(engines[0].n, f, mf, mu, fprev)
        fprev = f
        ts = []
        for p, e in enumerate(engines):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            o = e.expand(d, wide=mu * 4 < A.nnz)
            b.record()
            torch.cuda.synchronize()
            ts.append(round(a.elapsed_time(b), 4))
            gathered[p * stride:p * stride + o.numel()] = o
        st = [e.merge(gathered, stride) for e in engines]
        if rep:
            print(f"level {lv} dir {d} f {f} mf {mf} mu {mu} expand_ms {ts}", flush=True)
        lv += 1
    torch.cuda.nvtx.range_pop()
