"""Per-level |F|, m_f, m_u and device time of TileBFS on R-MAT s26 (sym) for a few
bench sources: the numbers the direction rule sees.  Dev aid."""
import sys; sys.path.insert(0, "/root/repo")
import torch, synth
from paper_conf_icpp_jisl0t022_b200 import tsmv
dev = torch.device("cuda", 0)
A = synth.rmat(26, 16, seed=1, symmetrize=True, device=dev)
srcs = [0] + synth.sample_sources(A, 7, seed=1)
torch.cuda.empty_cache()
M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", sparse_tile_max_nnz=8)
deg = (A.row_ptr[1:] - A.row_ptr[:-1])
for s in srcs[2:4] + srcs[1:2]:
    lv, st = M.bfs(s)
    lv, st = M.bfs(s)
    mu = int(deg.sum())
    print("source", s, round(st["ms"], 3))
    for L in range(st["nlevels"]):
        fr = lv == L
        f = int(fr.sum()); mf = int(deg[fr].sum())
        print(f"  L{L} {st['dirs'][L]:9s} f {f:10d} mf {mf:12d} mu {mu:12d} mf/mu {mf/max(mu,1):.3f} ms {st['level_ms'][L]:.3f}")
        mu -= int(deg[fr].sum())
