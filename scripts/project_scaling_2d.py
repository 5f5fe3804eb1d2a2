"""Projected strong scaling of the 2D-partitioned TileBFS (NEXT-4, dist2d.py) from
simulated ranks on ONE B200, the counterpart of project_scaling.py (row blocks).

P = Pr x Pc contexts (dist2d.grid_shape) hold the padded blocks A_ij of the same
graph on GPU 0; every level runs exactly as P processes would (expand on every
rank, the exchanges by concatenation, merge on every rank), each rank's calls timed
with CUDA events.  A projected level = max over ranks (expand) + max over ranks
(merge) + exchange: S/8 x (Pr - 1) bytes of the processor-column all-gather,
S/8 x (Pc - 1) of the processor-row all-to-all and (direction-optimising mode) of
the processor-row all-gather, at the peer bandwidth, plus one latency per
collective (3 or 4 with the 24-byte statistics all-reduce).

usage: python scripts/project_scaling_2d.py [scale] [P,...] [--balance nnz|rows] [--permute]"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import dist2d as D2  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("scale", type=int, nargs="?", default=24)
ap.add_argument("ranks", nargs="?", default="1,2,4,8")
ap.add_argument("--nccl-us", type=float, default=20.0)
ap.add_argument("--link-gbs", type=float, default=770.0)
ap.add_argument("--sources", type=int, default=2)
ap.add_argument("--balance", default="nnz")
ap.add_argument("--permute", action="store_true")
ap.add_argument("--mode", default="dopt")
args = ap.parse_args()
dev = torch.device("cuda", 0)
A = synth.rmat(args.scale, 16, seed=1, symmetrize=True, device=dev, permute=args.permute)
srcs = [0] + synth.sample_sources(A, args.sources - 1, seed=1)
out = {"graph": f"rmat_s{args.scale}_ef16_sym" + ("_permuted" if args.permute else ""), "nnz": A.nnz,
       "balance": args.balance, "mode": args.mode, "assumptions": {"nccl_latency_us_per_collective": args.nccl_us,
                                                "link_GBps": args.link_gbs}, "runs": {}}


for P in [int(p) for p in args.ranks.split(",")]:
    Pr, Pc = D2.grid_shape(P)
    g = D2.Grid2D(A.n, Pr, Pc, row_ptr=A.row_ptr, balance=args.balance)
    E = []
    for r in range(P):
        B = D2.block_2d(A, g, *g.coords(r))
        torch.cuda.empty_cache()
        E.append(D2.Dist2DBFS(B, g, r, device=0, mode=args.mode))
        del B
        torch.cuda.empty_cache()
    D2.sim_degrees(A, E)
    torch.cuda.empty_cache()
    rp = A.row_ptr
    deg = rp[1:] - rp[:-1]
    runs = []
    for s in srcs:
        D2.sim_bfs2d(E, s)
        trace = []
        D2.sim_bfs2d(E, s, trace=trace)
        lvls = D2.gather_levels(E)
        edges = int(deg[lvls >= 0].sum())   # R16 count: in-degrees of the reached vertices
        ncoll = 4 if args.mode == "dopt" else 3
        nbytes = (g.S / 8) * ((Pr - 1) + (Pc - 1) + ((Pc - 1) if args.mode == "dopt" else 0))
        xfer = nbytes / (args.link_gbs * 1e9) * 1e3
        lat = ncoll * args.nccl_us * 1e-3 if P > 1 else 0.0
        lv = [dict(t, exchange=(xfer + lat) if P > 1 else 0.0) for t in trace]
        proj = sum(x["expand_max"] + x["merge_max"] + x["exchange"] for x in lv)
        runs.append({"source": s, "levels": len(lv), "edges": edges, "projected_ms": round(proj, 4),
                     "projected_gteps": round(edges / (proj * 1e-3) / 1e9, 2),
                     "per_level": [{k: (round(v, 4) if isinstance(v, float) else v) for k, v in x.items()}
                                   for x in lv]})
    for e in E:
        e.close()
    del E
    torch.cuda.empty_cache()
    hm = len(runs) / sum(1.0 / r["projected_gteps"] for r in runs)
    out["runs"][P] = {"grid": [Pr, Pc], "S": g.S, "gteps_hmean_projected": round(hm, 2), "runs": runs}
    print(json.dumps({"P": P, "grid": [Pr, Pc], "gteps_hmean_projected": round(hm, 2),
                      "per_source_ms": [r["projected_ms"] for r in runs]}), flush=True)
base = out["runs"].get(1)
if base:
    out["speedup_vs_P1"] = {P: round(v["gteps_hmean_projected"] / base["gteps_hmean_projected"], 2)
                            for P, v in out["runs"].items()}
print(json.dumps({k: v for k, v in out.items() if k != "runs"}))
json.dump(out, open(os.environ.get("PROJ_OUT", "/dev/null"), "w"), indent=1)
