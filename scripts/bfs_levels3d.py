import sys; sys.path.insert(0, "/root/repo")
import torch, synth, os
from paper_conf_icpp_jisl0t022_b200 import tsmv
dev = torch.device("cuda", 0)
A = synth.stencil3d(256, device=dev)
M = tsmv.TiledMatrix.from_csr(A, dtype="pattern")
w = torch.empty(64 << 20, dtype=torch.float32, device=dev)
M.bfs(0); w.zero_(); torch.cuda.synchronize()
os.environ["TSMV_BFS_PHASES"] = "1"
lv, st = M.bfs(0)
os.environ.pop("TSMV_BFS_PHASES")
import collections
t = st["level_ms"]; d = st["dirs"]; f = st["frontier"] if "frontier" in st else None
print("ms", st["ms"], "levels", st["nlevels"], collections.Counter(d))
print("level ms: first 5", [round(x,4) for x in t[:5]], "mid", [round(x,4) for x in t[380:385]], "last", [round(x,4) for x in t[-5:]])
print("sum", sum(t), "max", max(t))
