"""Quick device timing of y = A x at T (R-MAT s22, fp64, 1 %) and C1/C2 shapes,
flat kernel vs the round-1 fused kernel (TSMV_FUSED_V6=1).  Dev aid."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
from paper_conf_icpp_jisl0t022_b200 import tsmv
dev = torch.device("cuda", 0)
w = torch.empty(64 << 20, dtype=torch.float32, device=dev); r = torch.ones(64 << 20, dtype=torch.float32, device=dev)

def run(M, A, d, steps=10, label=""):
    k = max(1, synth.density_k(A.n, d))
    xs = [synth.sample_x(A.n, k, seed=s, device=dev) for s in range(1, steps + 4)]
    yi = torch.empty(A.m, dtype=torch.int32, device=dev); yv = torch.empty(A.m, dtype=torch.float64, device=dev)
    yn = torch.zeros(1, dtype=torch.int64, device=dev)
    out = {}
    for v6 in (0,):
        if v6: os.environ["TSMV_FUSED_V6"] = "1"
        else: os.environ.pop("TSMV_FUSED_V6", None)
        for xi, xv in xs[:3]: M.spmspv_async(xi, xv, yi, yv, yn)
        torch.cuda.synchronize()
        M.set_timing(True)
        ts = []
        for xi, xv in xs[3:]:
            w.zero_(); _ = r.sum()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); M.spmspv_async(xi, xv, yi, yv, yn); e1.record(); torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) * 1e3)
        kt, n = M.get_timing(); M.set_timing(False)
        ts.sort()
        out["v6" if v6 else "flat"] = (ts[len(ts) // 2], [round(x / n * 1e3, 1) for x in kt])
    os.environ.pop("TSMV_FUSED_V6", None)
    print(f"{label} d={d}: " + "  ".join(f"{kk}: median {v[0]:.1f} us phases(A,B,C,all) {v[1]}" for kk, v in out.items()), flush=True)

p = torch.cuda.get_device_properties(0); print("L2", getattr(p, "L2_cache_size", None), "persist max", getattr(p, "persisting_l2_cache_max_size", None))
A = synth.stencil2d(64, 64, device=dev); M = tsmv.TiledMatrix.from_csr(A); run(M, A, 0.01, label="C1"); M.close()
A = synth.attach_values(synth.rmat(int(sys.argv[1]) if len(sys.argv) > 1 else 22, 16, seed=1, device=dev), seed=1)
M = tsmv.TiledMatrix.from_csr(A, build_bfs=0)
for d in (0.0001, 0.001, 0.01, 0.1): run(M, A, d, label="rmat")
