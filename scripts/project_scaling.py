"""Projected strong scaling of the row-block TileBFS (C5) from
simulated ranks on ONE B200 (no multi-GPU box was available).

P contexts are built from the nnz-balanced row blocks of the same graph on
GPU 0.  Every level runs through the distributed primitives exactly as P
processes would (tsmv_bfs_dist_expand on every rank, the owned frontier words
exchanged by device copies, tsmv_bfs_dist_merge on every rank) and each rank's
kernels are timed separately with CUDA events.  A level of the P-GPU run is then
projected as
    max over ranks (expand) + max over ranks (merge)
    + exchange: the n/8 frontier bytes each rank receives at the measured NVLink
      peer bandwidth (770 GB/s, B200_PROFILING.md) + a per-level NCCL latency
      (default 20 us, an assumption: --nccl-us)
    + host decision: the one read of the level's statistics (measured: the host
      time of reading the ranks' device statistics after their merges).
GTEPS(P) = edges / projected time.  This is a projection, not a measurement;
bench.py --gpus N measures the real thing when a multi-GPU box runs it.

usage: python scripts/project_scaling.py [scale] [P,...] [--nccl-us 20] [--sources 4]"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import dist as D  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("scale", type=int, nargs="?", default=24)
ap.add_argument("ranks", nargs="?", default="1,2,4,8")
ap.add_argument("--nccl-us", type=float, default=20.0)
ap.add_argument("--link-gbs", type=float, default=770.0)
ap.add_argument("--sources", type=int, default=4)
ap.add_argument("--thr", type=int, default=8)
ap.add_argument("--permute", action="store_true")
args = ap.parse_args()
dev = torch.device("cuda", 0)
A = synth.rmat(args.scale, 16, seed=1, symmetrize=True, device=dev, permute=args.permute)
srcs = [0] + synth.sample_sources(A, args.sources - 1, seed=1)
out = {"graph": f"rmat_s{args.scale}_ef16_sym" + ("_permuted" if args.permute else ""), "nnz": A.nnz, "assumptions": {
    "nccl_latency_us_per_level": args.nccl_us, "link_GBps": args.link_gbs}, "runs": {}}

# one-GPU fused traversal for reference
torch.cuda.empty_cache()
M1 = tsmv.TiledMatrix.from_csr(A, dtype="pattern", sparse_tile_max_nnz=args.thr)
ref = []
for s in srcs:
    M1.bfs(s)
    _, st = M1.bfs(s)
    ref.append({"source": s, "ms": st["ms"], "edges": st["edges_traversed"], "levels": st["nlevels"]})
M1.close()
out["single_gpu_fused"] = ref


def ev():
    return torch.cuda.Event(enable_timing=True)


for P in [int(p) for p in args.ranks.split(",")]:
    splits = D.partition_rows(A.row_ptr, P, row_weight=D.BFS_ROW_WEIGHT)
    engines = [D.DistTiledMatrix(D.local_rows(A, splits, r), splits, r, P, dtype="pattern",
                                 sparse_tile_max_nnz=args.thr) for r in range(P)]
    deg = torch.bincount(A.col_idx.long(), minlength=A.n).to(torch.int32)   # global out-degrees
    for e in engines:
        e.set_degrees(deg)
    nnz = sum(e.M.nnz for e in engines)
    stride = engines[0].stride
    gathered = torch.zeros(P * stride, dtype=torch.int32, device=dev)
    runs = []
    for s in srcs:
        for rep in range(2):  # warm-up traversal, then the measured one
            st = [e.begin(s) for e in engines]
            lv_proj, nlev, edges, fprev = [], 0, 0, 0
            while sum(x[0] for x in st) > 0:
                f = sum(x[0] for x in st)
                mf = sum(x[1] for x in st)
                mu = sum(x[2] for x in st)
                edges += mf
                d = engines[0].choose(engines[0].n, f, mf, mu, fprev)
                fprev = f
                te, tm = [], []
                for p, e in enumerate(engines):
                    a, b = ev(), ev()
                    a.record()
                    o = e.expand(d, wide=mu * D.WIDE_MULT < nnz)
                    b.record()
                    torch.cuda.synchronize()
                    te.append(a.elapsed_time(b))
                    gathered[p * stride:p * stride + o.numel()] = o
                # merge with the statistics left on the device (as the collective path
                # does before its one read per level), then that one read: the level's
                # host decision term (r2 session 5; r2 timed merge() with its two host
                # round trips per rank inside the merge term)
                devs = []
                for e in engines:
                    a, b = ev(), ev()
                    a.record()
                    devs.append(e.merge_dev(gathered, stride).clone())
                    b.record()
                    torch.cuda.synchronize()
                    tm.append(a.elapsed_time(b))
                allst = torch.stack(devs)
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                st = [tuple(int(v) for v in row) for row in allst.tolist()]  # one read (each rank reads its own)
                host_ms = (time.perf_counter() - t0) * 1e3
                xfer_ms = (A.n / 8) * (P - 1) / P / (args.link_gbs * 1e9) * 1e3 if P > 1 else 0.0
                lat_ms = args.nccl_us * 1e-3 if P > 1 else 0.0
                lv_proj.append({"expand_max": max(te), "merge_max": max(tm), "exchange": xfer_ms + lat_ms,
                                "host": host_ms, "dir": d})
                nlev += 1
        proj = sum(l["expand_max"] + l["merge_max"] + l["exchange"] + l["host"] for l in lv_proj)
        runs.append({"source": s, "levels": nlev, "edges": edges, "projected_ms": round(proj, 4),
                     "per_level": [{k: (round(v, 4) if isinstance(v, float) else v) for k, v in l.items()}
                                   for l in lv_proj],
                     "projected_gteps": round(edges / (proj * 1e-3) / 1e9, 2),
                     "kernel_ms": round(sum(l["expand_max"] + l["merge_max"] for l in lv_proj), 4),
                     "exchange_ms": round(sum(l["exchange"] for l in lv_proj), 4)})
    for e in engines:
        e.M.close()
    del engines
    torch.cuda.empty_cache()
    hm = len(runs) / sum(1.0 / r["projected_gteps"] for r in runs)
    out["runs"][P] = {"gteps_hmean_projected": round(hm, 2), "runs": runs}
    print(json.dumps({"P": P, "gteps_hmean_projected": round(hm, 2),
                      "per_source_ms": [r["projected_ms"] for r in runs]}), flush=True)
base = out["runs"].get(1)
if base:
    out["speedup_vs_P1"] = {P: round(v["gteps_hmean_projected"] / base["gteps_hmean_projected"], 2)
                            for P, v in out["runs"].items()}
fused_hm = len(ref) / sum(r["ms"] * 1e-3 * 1e9 / r["edges"] for r in ref)
out["single_gpu_fused_gteps_hmean"] = round(fused_hm, 2)
print(json.dumps({k: v for k, v in out.items() if k not in ("runs", "single_gpu_fused")}))
json.dump(out, open(os.environ.get("PROJ_OUT", "/dev/null"), "w"), indent=1)
