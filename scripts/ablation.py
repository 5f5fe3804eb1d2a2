"""The paper's own analyses on the synthetic configs, B200.

  * direction ablation (Fig 9): Push-CSC only (K1),
    Push-CSC + Push-CSR (K1+K2: the rule with pull disabled), the full rule
    (K1+K2+K3), and Pull-CSC only;
  * per-level direction and frontier size of the automatic run (Fig 10,
    P:2753-2790);
  * tile-format build time against one traversal (Fig 11);
  * very-sparse-tile extraction on/off: side threshold 0 vs 2,
    for TileBFS and for TileSpMSpV at 1 % density.

Every traversal's levels are checked against the automatic run (the levels
are direction-invariant, R9).  Writes one JSON object to stdout.
usage: python scripts/ablation.py [--out profiles/r01s3_ablation.json]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

DEV = torch.device("cuda", 0)
PAPER = {"push_csr_density": 0.01, "pull_alpha": 14.0}   # the paper's density rule + Beamer's alpha
MODES = {"K1 push-csc": {"force_dir": 1}, "K1+K2 push only": {"pull_alpha": 1e-300, "push_csr_density": 0.01},
         "K1+K2+K3 paper rule": PAPER, "K1+K2+K3 B200 defaults": {}, "K3 pull only": {"force_dir": 3}}
DCH = {"push_csc": "C", "push_csr": "R", "pull_csc": "P"}


def flush_buf():
    w = torch.empty(64 << 20, dtype=torch.float32, device=DEV)
    return lambda: w.zero_()


def graphs(quick):
    yield "C1 grid2d 64x64", synth.stencil2d(64, 64, device=DEV).with_values(None)
    yield "C3 rmat s22 sym", synth.rmat(20 if quick else 22, 16, seed=1, symmetrize=True, device=DEV)
    yield "C4 grid3d 256^3", synth.stencil3d(64 if quick else 256, device=DEV).with_values(None)
    yield "C4 band 2^20 b64", synth.banded(1 << (16 if quick else 20), 64, device=DEV).with_values(None)


def bfs_time(M, src, flush, lv):
    M.bfs(src, levels=lv)
    flush()
    torch.cuda.synchronize()
    _, st = M.bfs(src, levels=lv)
    return st


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    ap.add_argument("--quick", action="store_true")
    args = ap.parse_args()
    flush = flush_buf()
    out = {"device": torch.cuda.get_device_name(0), "graphs": {}}
    for name, A in graphs(args.quick):
        g = {"n": A.n, "nnz": A.nnz, "directions": {}}
        lv = torch.empty(A.n, dtype=torch.int32, device=DEV)
        ref = None
        for thr in (2, 0):
            M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", sparse_tile_max_nnz=thr)
            st = bfs_time(M, 0, flush, lv)
            if ref is None:
                ref = lv.clone()
            assert torch.equal(lv, ref), f"{name}: thr={thr} levels differ"
            g[f"thr{thr}"] = {"build_ms": round(M.info()["build_ms"], 3), "bfs_ms": round(st["ms"], 4),
                              "gteps": round(st["edges_traversed"] / (st["ms"] * 1e-3) / 1e9, 3),
                              "levels": st["nlevels"], "dense_tiles": M.info()["n_dense_tiles"],
                              "side_nnz": M.info()["side_nnz"]}
            if thr == 2:
                g["per_level"] = {"dirs": "".join(DCH.get(d, "?") for d in st["dirs"]),
                                  "frontier": st["frontier"] if len(st["frontier"]) <= 64 else
                                  st["frontier"][:32] + ["..."] + st["frontier"][-8:]}
                g["build_over_bfs"] = round(M.info()["build_ms"] / st["ms"], 3)
            M.close()
        for mname, opts in MODES.items():
            if name.startswith("C4") and mname.startswith("K3") and not args.quick:
                # pull-only on a 766 / 16,385-level traversal: every level reads every row tile
                g["directions"][mname] = "skipped (one full pull per level: O(levels x n))"
                continue
            M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", **opts)
            st = bfs_time(M, 0, flush, lv)
            assert torch.equal(lv, ref), f"{name}: {mname} levels differ"
            g["directions"][mname] = {"ms": round(st["ms"], 4),
                                      "gteps": round(st["edges_traversed"] / (st["ms"] * 1e-3) / 1e9, 3),
                                      "dirs": "".join(DCH.get(d, "?") for d in st["dirs"])[:64]}
            M.close()
        out["graphs"][name] = g
        print(json.dumps({name: g}), flush=True)
        del A
    # extraction on/off for TileSpMSpV at the roofline config shape (R-MAT directed, 1 %)
    s = 20 if args.quick else 22
    base = synth.attach_values(synth.rmat(s, 16, seed=1, device=DEV), seed=1, dtype="f64")
    k = synth.density_k(base.n, 0.01)
    xs = [synth.sample_x(base.n, k, seed=1 + i, device=DEV) for i in range(8)]
    yi = torch.empty(base.m, dtype=torch.int32, device=DEV)
    yv = torch.empty(base.m, dtype=torch.float64, device=DEV)
    yn = torch.zeros(1, dtype=torch.int64, device=DEV)
    sp = {}
    for thr in (0, 1, 2, 4, 8):
        M = tsmv.TiledMatrix.from_csr(base, dtype="f64", sparse_tile_max_nnz=thr, build_bfs=0)
        for xi, xv in xs[:2]:
            M.spmspv_async(xi, xv, yi, yv, yn)
        tt = 0.0
        for xi, xv in xs[2:]:
            flush()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            M.spmspv_async(xi, xv, yi, yv, yn)
            e1.record()
            torch.cuda.synchronize()
            tt += e0.elapsed_time(e1)
        sp[f"thr{thr}"] = {"us_per_call": round(1e3 * tt / len(xs[2:]), 2), "dense_tiles": M.info()["n_dense_tiles"],
                           "side_nnz": M.info()["side_nnz"], "build_ms": round(M.info()["build_ms"], 2)}
        M.close()
    out["spmspv_extraction"] = {"matrix": f"rmat s{s} directed fp64, x 1 %", "runs": sp}
    print(json.dumps({"spmspv_extraction": out["spmspv_extraction"]}), flush=True)
    if args.out:
        with open(args.out, "w") as f:
            json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
