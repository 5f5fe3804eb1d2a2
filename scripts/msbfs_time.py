"""Multi-source TileBFS timing (dev aid).  usage: msbfs_time.py graph [nsrc]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
from paper_conf_icpp_jisl0t022_b200 import tsmv
dev = torch.device("cuda", 0)
name = sys.argv[1]; ns = int(sys.argv[2]) if len(sys.argv) > 2 else 64
if name.startswith("rmat"):
    A = synth.rmat(int(name[4:]), 16, seed=1, symmetrize=True, device=dev)
elif name.startswith("grid3d"):
    A = synth.stencil3d(int(name[6:]), device=dev).with_values(None)
else:
    n, b = name[4:].split("_"); A = synth.banded(1 << int(n), int(b), device=dev).with_values(None)
M = tsmv.TiledMatrix.from_csr(A, dtype="pattern")
src = [0] + synth.sample_sources(A, ns - 1, seed=1)
lv, st = M.msbfs(src)
lv, st = M.msbfs(src, levels=lv)
one = []
for s in src[:4]:
    _, s1 = M.bfs(s); one.append(s1["ms"])
print(f"{name} nsrc={ns}: {st['ms']:.3f} ms, levels {st['nlevels']}, pairs {st['pairs_reached']}, "
      f"edges {st['edges_traversed']}, {st['edges_traversed'] / st['ms'] / 1e6:.1f} GTEPS; "
      f"single-source TileBFS {sum(one) / len(one):.3f} ms each -> x{ns * sum(one) / len(one) / st['ms']:.2f} throughput", flush=True)
