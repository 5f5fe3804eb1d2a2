"""Per-level device times of the fused TileBFS kernel against the per-level kernels
(the distributed primitives with one rank) on R-MAT sym.  Dev aid.
usage: python scripts/cmp_fused_prim.py scale src,src,..."""
import os, sys
sys.path.insert(0, "/root/repo")
import torch, synth
from paper_conf_icpp_jisl0t022_b200 import tsmv, dist as D
dev = torch.device("cuda", 0)
sc = int(sys.argv[1]) if len(sys.argv) > 1 else 26
A = synth.rmat(sc, 16, seed=1, symmetrize=True, device=dev)
srcs = [int(s) for s in sys.argv[2].split(",")]
torch.cuda.empty_cache()
M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", sparse_tile_max_nnz=8)
for s in srcs:
    M.bfs(s); _, st = M.bfs(s)
    print("fused", s, round(st["ms"], 3), st["dirs"], [round(x, 3) for x in st.get("level_ms", [])], flush=True)
M.close(); torch.cuda.empty_cache()
splits = D.partition_rows(A.row_ptr, 1)
e = D.DistTiledMatrix(D.local_rows(A, splits, 0), splits, 0, 1, dtype="pattern", sparse_tile_max_nnz=8)
stride = e.stride
for s in srcs:
    for rep in range(2):
        st = e.begin(s); tl = []; ds = []; fprev = 0
        while st[0] > 0:
            d = e.choose(e.n, *st, fprev)
            fprev = st[0]
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); o = e.expand(d, wide=st[2] * 4 < A.nnz); st = e.merge(o, stride); b.record(); torch.cuda.synchronize()
            tl.append(round(a.elapsed_time(b), 3)); ds.append(d)
    print("prim ", s, round(sum(tl), 3), ds, tl, flush=True)
