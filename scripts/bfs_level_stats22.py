import sys; sys.path.insert(0, "/root/repo")
import torch, synth
from paper_conf_icpp_jisl0t022_b200 import tsmv
dev = torch.device("cuda", 0)
A = synth.rmat(22, 16, seed=1, symmetrize=True, device=dev)
srcs = [0] + synth.sample_sources(A, 15, seed=1)
M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", sparse_tile_max_nnz=8)
deg = (A.row_ptr[1:] - A.row_ptr[:-1])
w = torch.empty(64 << 20, dtype=torch.float32, device=dev)
for s in srcs[:4]:
    lv, st = M.bfs(s)
    w.zero_(); torch.cuda.synchronize()
    lv, st = M.bfs(s)
    mu = int(deg.sum())
    print("source", s, "deg", int(deg[s]), round(st["ms"], 3))
    for L in range(st["nlevels"]):
        fr = lv == L
        f = int(fr.sum()); mf = int(deg[fr].sum())
        print(f"  L{L} {st['dirs'][L]:9s} f {f:10d} mf {mf:12d} mu {mu:12d} ms {st['level_ms'][L]:.4f}")
        mu -= mf
