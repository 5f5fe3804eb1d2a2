"""One TileBFS traversal (after a warm-up) on a named graph, for ncu launch lists.
usage: python scripts/bfs_one.py rmat22|grid3d256|band20_64 [source]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
from paper_conf_icpp_jisl0t022_b200 import tsmv
dev = torch.device("cuda", 0)
name = sys.argv[1]
if name.startswith("rmat"):
    A = synth.rmat(int(name[4:]), 16, seed=1, symmetrize=True, device=dev)
elif name.startswith("grid3d"):
    A = synth.stencil3d(int(name[6:]), device=dev).with_values(None)
else:
    n, b = name[4:].split("_")
    A = synth.banded(1 << int(n), int(b), device=dev).with_values(None)
M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", sparse_tile_max_nnz=int(os.environ.get("THR", "2")))
src = int(sys.argv[2]) if len(sys.argv) > 2 else 0
lv = torch.empty(A.n, dtype=torch.int32, device=dev)
M.bfs(src, levels=lv)
torch.cuda.synchronize()
torch.cuda.nvtx.range_push("timed")
_, st = M.bfs(src, levels=lv)
torch.cuda.nvtx.range_pop()
print(name, st["ms"], st["dirs"], st["frontier"])
