"""Per-warp trace of phase B (multiply) of the fused SpMSpV kernel (dev aid)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
from paper_conf_icpp_jisl0t022_b200 import tsmv
scale = int(sys.argv[1]); thr = int(sys.argv[2]); d = float(sys.argv[3])
dev = torch.device("cuda", 0)
A = synth.attach_values(synth.rmat(scale, 16, seed=1, device=dev), seed=1)
M = tsmv.TiledMatrix.from_csr(A, sparse_tile_max_nnz=thr, build_bfs=0)
nw = tsmv.tsmv_trace_words(M.ctx)
buf = torch.zeros(nw, dtype=torch.int64, device=dev)
k = synth.density_k(A.n, d)
w = torch.empty(64 << 20, dtype=torch.float32, device=dev); r = torch.ones(64 << 20, dtype=torch.float32, device=dev)
for s in range(1, 4):
    xi, xv = synth.sample_x(A.n, k, seed=s, device=dev)
    if s == 3:
        tsmv.tsmv_set_trace(M.ctx, buf.data_ptr())
    w.zero_(); _ = r.sum()
    M.spmspv(xi, xv)
t = buf.view(-1, 8).cpu().double()
t0 = t[:, 0].min()
busy = t[:, 2] > 0
print(f"s{scale} thr{thr} d{d}: warps {t.shape[0]}, busy {int(busy.sum())}, chunks {int(t[:,2].sum())}")
end = (t[:, 1] - t0) / 1e3
print(f"  loop end us: max {end.max():.1f} p99 {end.quantile(0.99):.1f} median {end[busy].median():.1f}")
print(f"  chunk ns max {t[:,5].max():.0f}; tile ns/chunk mean {t[:,3].sum()/max(1,t[:,2].sum()):.0f}; side total {t[:,4].sum()/1e3:.0f}us tile total {t[:,3].sum()/1e3:.0f}us")
i = int(torch.argmax(t[:, 1]))
print(f"  slowest warp {i}: start {(t[i,0]-t0)/1e3:.1f} end {(t[i,1]-t0)/1e3:.1f} chunks {int(t[i,2])} tile {t[i,3]/1e3:.1f}us side {t[i,4]/1e3:.1f}us max {t[i,5]/1e3:.1f}us macs {int(t[i,7])} stage-of-max {t[i,6]/1e3:.1f}us")
start = (t[:, 0] - t0) / 1e3
print(f"  phase-B start skew: max {start.max():.1f} us")
if os.environ.get("TSMV_TRACE_ROUNDS_PRINT"):
    print(f"  slowest warp rounds: position {t[i,3]/1e3:.1f}us loads {t[i,4]/1e3:.1f}us atomics {t[i,6]/1e3:.1f}us")
    print(f"  all warps: position {t[:,3].sum()/1e3:.0f}us loads {t[:,4].sum()/1e3:.0f}us atomics {t[:,6].sum()/1e3:.0f}us")
