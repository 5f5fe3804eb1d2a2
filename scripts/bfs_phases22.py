import sys, os; sys.path.insert(0, "/root/repo")
import torch, synth
from paper_conf_icpp_jisl0t022_b200 import tsmv
dev = torch.device("cuda", 0)
A = synth.rmat(22, 16, seed=1, symmetrize=True, device=dev)
M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", sparse_tile_max_nnz=8)
w = torch.empty(64 << 20, dtype=torch.float32, device=dev)
for s in (0, 1657212):
    M.bfs(s); w.zero_(); torch.cuda.synchronize()
    os.environ["TSMV_BFS_PHASES"] = "1"
    print("source", s, flush=True)
    lv, st = M.bfs(s)
    torch.cuda.synchronize()
    os.environ.pop("TSMV_BFS_PHASES")
    print([round(x, 4) for x in st["level_ms"]], st["dirs"], flush=True)
