"""TileBFS timing: fused device loop vs host loop (dev aid).  usage: bfs_cmp.py graph..."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
from paper_conf_icpp_jisl0t022_b200 import tsmv
dev = torch.device("cuda", 0)
def graph(name):
    if name.startswith("rmat"):
        return synth.rmat(int(name[4:]), 16, seed=1, symmetrize=True, device=dev)
    if name.startswith("grid3d"):
        return synth.stencil3d(int(name[6:]), device=dev).with_values(None)
    if name.startswith("grid2d"):
        return synth.stencil2d(int(name[6:]), int(name[6:]), device=dev).with_values(None)
    if name.startswith("band"):
        n, b = name[4:].split("_")
        return synth.banded(1 << int(n), int(b), device=dev).with_values(None)
for name in sys.argv[1:]:
    A = graph(name)
    M = tsmv.TiledMatrix.from_csr(A, dtype="pattern")
    lv = torch.empty(A.n, dtype=torch.int32, device=dev)
    for mode in os.environ.get("MODES", "hybrid,nolist,hostloop").split(","):
        for e in ("TSMV_BFS_HOSTLOOP", "TSMV_BFS_FUSED_ONLY", "TSMV_BFS_NO_LIST"): os.environ.pop(e, None)
        if mode == "nolist": os.environ["TSMV_BFS_NO_LIST"] = "1"
        if mode == "hostloop": os.environ["TSMV_BFS_HOSTLOOP"] = "1"
        if mode == "fusedonly": os.environ["TSMV_BFS_FUSED_ONLY"] = "1"
        M.bfs(0, levels=lv)
        res = []
        for s in [0, 1]:
            _, st = M.bfs(s, levels=lv)
            res.append(st)
        st = res[0]
        print(f"{name} {mode:8s}: {st['ms']:.3f} ms levels {st['nlevels']} GTEPS {st['edges_traversed']/st['ms']/1e6:.2f} dirs {''.join(d[5] if d!='push_csc' else 'C' for d in st['dirs'][:40])}", flush=True)
    M.close()
