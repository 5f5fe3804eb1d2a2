"""BASELINE config 5 (R-MAT scale 26) on ONE B200: TileSpMSpV at 1 % and TileBFS.

Checks (no CPU oracle at this size): SpMSpV y on 4096 sampled rows against the
row-wise definition y_i = sum_j a_ij x_j evaluated with torch in fp64 (and the
structural index set on those rows); BFS levels by the Graph500 rules, evaluated
on the GPU over every edge: source level 0, |level(u) - level(v)| <= 1 on every
edge with both ends reached, no edge from a reached to an unreached vertex, and
every reached v != source has an in-neighbour one level up.
usage: python scripts/c5_single.py [scale] [--no-bfs] [--no-spmspv]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

DEV = torch.device("cuda", 0)
scale = int(sys.argv[1]) if len(sys.argv) > 1 and sys.argv[1].isdigit() else 26
out = {"scale": scale}
flushbuf = torch.empty(64 << 20, dtype=torch.float32, device=DEV)


def gb():
    return round(torch.cuda.max_memory_allocated() / 2**30, 2)


if "--no-spmspv" not in sys.argv:
    t0 = time.time()
    A = synth.attach_values(synth.rmat(scale, 16, seed=1, device=DEV), seed=1)
    out["gen_s"] = round(time.time() - t0, 1)
    out["nnz"] = A.nnz
    t0 = time.time()
    M = tsmv.TiledMatrix.from_csr(A, build_bfs=0)
    out["build_wall_s"] = round(time.time() - t0, 2)
    out["info"] = {k: v for k, v in M.info().items() if k in ("n_tiles", "n_dense_tiles", "side_nnz", "build_ms",
                                                               "bytes_spmspv")}
    colcnt = torch.bincount(A.col_idx.long(), minlength=A.n)
    k = synth.density_k(A.n, 0.01)
    yi = torch.empty(A.m, dtype=torch.int32, device=DEV)
    yv = torch.empty(A.m, dtype=torch.float64, device=DEV)
    yn = torch.zeros(1, dtype=torch.int64, device=DEV)
    runs = []
    for s in range(1, 8):
        xi, xv = synth.sample_x(A.n, k, seed=s, device=DEV)
        flushbuf.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        M.spmspv_async(xi, xv, yi, yv, yn)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1)
        fl = 2 * int(colcnt[xi.long()].sum())
        if s >= 3:
            runs.append({"us": round(ms * 1e3, 1), "gflops": round(fl / ms / 1e6, 2), "y_nnz": int(yn)})
    # check the last call on sampled rows
    ny = int(yn)
    xd = torch.zeros(A.n, dtype=torch.float64, device=DEV)
    xd[xi.long()] = xv
    g = torch.Generator(device="cpu").manual_seed(7)
    rows = torch.randint(0, A.m, (4096,), generator=g).to(DEV)
    rp = A.row_ptr
    ref, present = [], []
    for r in rows.tolist():
        c = A.col_idx[rp[r]:rp[r + 1]].long()
        v = A.values[rp[r]:rp[r + 1]]
        hit = xd[c] != 0
        present.append(bool(hit.any()))
        ref.append(float((v[hit] * xd[c][hit]).sum()))
    yi_l, yv_l = yi[:ny].long(), yv[:ny]
    pos = torch.searchsorted(yi_l, rows)
    pos_c = pos.clamp(max=max(ny - 1, 0))
    found = (yi_l[pos_c] == rows) & (pos < ny)
    ok_set = all(bool(f) == p for f, p in zip(found.tolist(), present))
    got = torch.where(found, yv_l[pos_c], torch.zeros_like(yv_l[pos_c])).tolist()
    err = max((abs(a - b) / max(abs(b), 1e-300) for a, b, p in zip(got, ref, present) if p), default=0.0)
    out["spmspv"] = {"k": k, "runs": runs, "sampled_rows": 4096, "index_set_ok": ok_set,
                     "max_rel_err": err, "peak_mem_gb": gb()}
    print(json.dumps(out), flush=True)
    M.close()
    del A, M, colcnt, xd

if "--no-bfs" not in sys.argv:
    torch.cuda.reset_peak_memory_stats()
    t0 = time.time()
    A = synth.rmat(scale, 16, seed=1, symmetrize=True, device=DEV)
    gen = time.time() - t0
    torch.cuda.empty_cache()
    free, total = torch.cuda.mem_get_info()
    print(json.dumps({"bfs_graph_nnz": A.nnz, "free_gb_before_build": round(free / 2**30, 1),
                      "torch_allocated_gb": round(torch.cuda.memory_allocated() / 2**30, 1)}), flush=True)
    t0 = time.time()
    M = tsmv.TiledMatrix.from_csr(A, dtype="pattern")
    bw = time.time() - t0
    info = M.info()
    free, total = torch.cuda.mem_get_info()
    print(json.dumps({"free_gb_after_build": round(free / 2**30, 1), "info": info}), flush=True)
    lv = torch.empty(A.n, dtype=torch.int32, device=DEV)
    srcs = [0] + synth.sample_sources(A, 2, seed=1)
    M.bfs(srcs[0], levels=lv)
    runs = []
    for s in srcs:
        flushbuf.zero_()
        torch.cuda.synchronize()
        _, st = M.bfs(s, levels=lv)
        # Graph500 level rules over every edge (chunked)
        def rows_of(c0, c1):
            return torch.searchsorted(A.row_ptr, torch.arange(c0, c1, device=DEV), right=True) - 1

        okall = bool(lv[s] == 0)
        for c0 in range(0, A.nnz, 1 << 28):
            r = rows_of(c0, min(A.nnz, c0 + (1 << 28)))
            c = A.col_idx[c0:c0 + (1 << 28)].long()
            lr, lc = lv[r], lv[c]
            both = (lr >= 0) & (lc >= 0)
            okall &= bool(((lr - lc).abs()[both] <= 1).all())
            okall &= bool(((lr >= 0) == (lc >= 0)).all())   # symmetric: no reached -> unreached edge
            del r, c, lr, lc, both
        # every reached v != s has a neighbour one level up
        has = torch.zeros(A.n, dtype=torch.bool, device=DEV)
        for c0 in range(0, A.nnz, 1 << 28):
            r = rows_of(c0, min(A.nnz, c0 + (1 << 28)))
            c = A.col_idx[c0:c0 + (1 << 28)].long()
            m = (lv[c] >= 0) & (lv[c] == lv[r] - 1)
            has[r[m]] = True
        reached = lv >= 0
        reached[s] = False
        okall &= bool(has[reached].all())
        del has
        runs.append({"source": int(s), "ms": round(st["ms"], 3), "levels": st["nlevels"],
                     "gteps": round(st["edges_traversed"] / (st["ms"] * 1e-3) / 1e9, 2),
                     "dirs": "".join({"push_csc": "C", "push_csr": "R", "pull_csc": "P"}[d] for d in st["dirs"]),
                     "reached": st["reached"], "graph500_levels_ok": okall})
    out["bfs"] = {"nnz": A.nnz, "gen_s": round(gen, 1), "build_wall_s": round(bw, 2), "build_ms": info["build_ms"],
                  "bytes_bfs": info["bytes_bfs"], "runs": runs, "peak_mem_gb": gb()}
    print(json.dumps(out), flush=True)
