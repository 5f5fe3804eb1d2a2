"""Per-CTA barrier trace of the flat SpMSpV kernel (tsmv_set_trace): arrival /
release times of each grid barrier, last arriver.  Dev aid.
usage: python scripts/trace_flat.py c1|<scale> [density]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
from paper_conf_icpp_jisl0t022_b200 import tsmv
dev = torch.device("cuda", 0)
which = sys.argv[1] if len(sys.argv) > 1 else "c1"
if which == "c1":
    A = synth.stencil2d(64, 64, device=dev); d = 0.01
else:
    A = synth.attach_values(synth.rmat(int(which), 16, seed=1, device=dev), seed=1); d = float(sys.argv[2])
M = tsmv.TiledMatrix.from_csr(A, build_bfs=0)
k = max(1, synth.density_k(A.n, d))
buf = torch.zeros(tsmv.tsmv_trace_words(M.ctx), dtype=torch.int64, device=dev)
w = torch.empty(64 << 20, dtype=torch.float32, device=dev); r = torch.ones(64 << 20, dtype=torch.float32, device=dev)
for flush in (True, False):
    for s in range(1, 7):
        xi, xv = synth.sample_x(A.n, k, seed=s, device=dev)
        if s == 6:
            tsmv.tsmv_set_trace(M.ctx, buf.data_ptr())
        if flush:
            w.zero_(); _ = r.sum()
        M.spmspv(xi, xv)
        tsmv.tsmv_set_trace(M.ctx, 0)
    G = 148
    t = buf[: G * 12].view(G, 12).cpu().double()
    t0 = t[:, 0].min()
    t = (t - t0) / 1e3
    print(f"{which} d={d} flush={flush}: start skew {t[:,0].max():.2f} us, end {t[:,9].max():.2f} us")
    for bi in range(4):
        arr, rel = t[:, 1 + 2 * bi], t[:, 2 + 2 * bi]
        print(f"  barrier {bi+1}: arrivals min {arr.min():.2f} median {arr.median():.2f} max {arr.max():.2f} (CTA {int(arr.argmax())}); "
              f"release min {rel.min():.2f} max {rel.max():.2f}")
st = buf[148 * 12: 148 * 12 + 8].cpu().tolist()
print("warp 0 step deltas ns (B1: Ct, window, masks | B2: entry->total, ->loads):", [st[i + 1] - st[i] if st[i + 1] and st[i] else None for i in range(6)])
c2 = t[:, 9] - t[:, 8]
top = torch.argsort(c2, descending=True)[:8].tolist()
print("C2 per-CTA us: median %.2f max %.2f; slowest CTAs:" % (c2.median(), c2.max()), [(i, round(float(c2[i]), 2)) for i in top])
b1 = t[:, 3] - t[:, 2]
top = torch.argsort(b1, descending=True)[:8].tolist()
print("B1 per-CTA us: median %.2f max %.2f; slowest CTAs:" % (b1.median(), b1.max()), [(i, round(float(b1[i]), 2)) for i in top])
st = buf[148 * 12 + 16: 148 * 12 + 32].cpu().tolist()
print("C2 CTA1 warp0 step deltas ns:", [st[i + 1] - st[i] if st[i + 1] and st[i] else None for i in range(15)])
b2 = t[:, 5] - t[:, 4]
top = torch.argsort(b2, descending=True)[:8].tolist()
print("B2 per-CTA us: median %.2f max %.2f; slowest CTAs:" % (b2.median(), b2.max()), [(i, round(float(b2[i]), 2)) for i in top])
