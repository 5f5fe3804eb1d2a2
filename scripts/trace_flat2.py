"""Per-CTA phase times of the flat SpMSpV kernel from tsmv_set_trace stamps
(globaltimer, ~0.25 us resolution): A (start -> reservation), A' (-> barrier 1
arrival), barrier 1 wait, B1, B2, flushes, barrier 2 wait, C.  Dev aid.
usage: python scripts/trace_flat2.py <scale> <density>"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

dev = torch.device("cuda", 0)
scale, d = int(sys.argv[1]), float(sys.argv[2])
A = synth.attach_values(synth.rmat(scale, 16, seed=1, device=dev), seed=1)
M = tsmv.TiledMatrix.from_csr(A, build_bfs=0)
k = max(1, synth.density_k(A.n, d))
buf = torch.zeros(tsmv.tsmv_trace_words(M.ctx), dtype=torch.int64, device=dev)
w = torch.empty(64 << 20, dtype=torch.float32, device=dev)
r = torch.ones(64 << 20, dtype=torch.float32, device=dev)
G = 148
acc = []
for s in range(1, 9):
    xi, xv = synth.sample_x(A.n, k, seed=s, device=dev)
    buf.zero_()
    if s >= 3:
        tsmv.tsmv_set_trace(M.ctx, buf.data_ptr())
    w.zero_(); _ = r.sum()
    M.spmspv(xi, xv)
    tsmv.tsmv_set_trace(M.ctx, 0)
    if s >= 3:
        acc.append(buf[: G * 16].view(G, 16).cpu().double())
names = [("A scan+resv", 0, 8), ("A lists", 8, 1), ("bar1 wait", 1, 2), ("B1", 2, 3), ("B2", 3, 4),
         ("flushes", 4, 7), ("bar2 arrive", 7, 5), ("bar2 wait", 5, 6), ("C", 6, 9), ("total", 0, 9)]
if any(float(t[:, 10].abs().sum()) > 0 for t in acc):  # bucketed variant: C split
    names[-1:-1] = [("C buckets", 6, 10), ("C lookback", 10, 11), ("C copy", 11, 9)]
    names[5:5] = [("fl hot", 4, 12), ("fl rank", 12, 13), ("fl resv", 13, 14), ("fl store", 14, 7)]
print(f"s{scale} d={d}: per-CTA phase durations in us (median / max over CTAs, mean over {len(acc)} calls)")
for nm, a, b in names:
    med = sum(float(((t[:, b] - t[:, a]) / 1e3).median()) for t in acc) / len(acc)
    mx = sum(float(((t[:, b] - t[:, a]) / 1e3).max()) for t in acc) / len(acc)
    print(f"  {nm:12s} median {med:6.2f}  max {mx:6.2f}")
if any(float(t[:, 15].abs().sum()) > 0 for t in acc):
    nb = [t[:, 15] / 1e3 for t in acc]
    print("  buckets met per CTA: median %.1f max %.0f" % (sum(float(x.median()) for x in nb) / len(nb),
                                                           sum(float(x.max()) for x in nb) / len(nb)))
t = acc[-1]
t0 = t[:, 0].min()
print("  last call: start skew %.2f us, barrier-1 release %.2f, barrier-2 release %.2f, end %.2f (max over CTAs)" % (
    float((t[:, 0] - t0).max() / 1e3), float((t[:, 2] - t0).max() / 1e3), float((t[:, 6] - t0).max() / 1e3),
    float((t[:, 9] - t0).max() / 1e3)))
