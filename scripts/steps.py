import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
from paper_conf_icpp_jisl0t022_b200 import tsmv
dev = torch.device("cuda", 0)
which = sys.argv[1] if len(sys.argv) > 1 else "c1"
if which == "c1":
    A = synth.stencil2d(64, 64, device=dev); k = 41
else:
    A = synth.attach_values(synth.rmat(22, 16, seed=1, device=dev), seed=1); k = 41943
M = tsmv.TiledMatrix.from_csr(A, build_bfs=0)
buf = torch.zeros(tsmv.tsmv_trace_words(M.ctx), dtype=torch.int64, device=dev)
w = torch.empty(64 << 20, dtype=torch.float32, device=dev); r = torch.ones(64 << 20, dtype=torch.float32, device=dev)
for s in range(1, 6):
    xi, xv = synth.sample_x(A.n, k, seed=s, device=dev)
    if s == 5: tsmv.tsmv_set_trace(M.ctx, buf.data_ptr())
    w.zero_(); _ = r.sum()
    M.spmspv(xi, xv)
t = buf[200:213].cpu().tolist()
print(which, "step deltas ns:", [t[i+1]-t[i] if t[i+1] and t[i] else None for i in range(12)])
