#!/usr/bin/env python
"""Benchmark of the TileSpMSpV / TileBFS hot path (BASELINE.json metric:
"SpMSpV GFLOPS & %HBM roofline; TileBFS GTEPS").

Default workload (config T of SURVEY §8, the north_star roofline target, the
largest single-GPU case BASELINE names): R-MAT scale 22, edge factor 16,
Graph500 (0.57, 0.19, 0.19, 0.05), directed, duplicates coalesced, fp64 values
1+u; x = 1 % density (41,943 distinct uniform indices, values 1+u), a fresh x
sample per step (seeds 1..W+K).  One step = one y = A x call (x tiling, tile
intersection + multiply + side-matrix merge, y compaction: SURVEY §8(a) a2-a6);
the tile format (a1) is built once outside the timed region and timed
separately; TileBFS (a7) on the symmetrised R-MAT s22 is reported in "bfs".

Timing: inputs resident in HBM; before every step the L2 is flushed by writing
a 256 MiB buffer (outside the events); each step is bracketed by CUDA events on
the launching stream; K steps between barriers; max over ranks.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl tsmv|reference]
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402

FALLBACK_HBM = 6650.0  # GB/s, B200_PROFILING.md fallback


def parse(argv=None):
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=30)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", default="tsmv", choices=["tsmv", "reference"])
    p.add_argument("--scale", type=int, default=22)
    p.add_argument("--density", type=float, default=0.01)
    p.add_argument("--dtype", default="f64", choices=["f64", "f32"])
    p.add_argument("--tile-dim", type=int, default=16)
    p.add_argument("--thr", type=int, default=2)
    p.add_argument("--bfs-scale", type=int, default=22)
    p.add_argument("--bfs-sources", type=int, default=16,
                   help="C3: vertex 0 + (N-1) hash-ordered non-isolated sources (SURVEY §8(d) step 4)")
    p.add_argument("--bfs26-sources", type=int, default=8, help="C5 on one GPU: vertex 0 + 7 sources")
    p.add_argument("--no-bfs26", action="store_true", help="skip the R-MAT s26 TileBFS block (C5 at N=1)")
    p.add_argument("--bfs-thr", type=int, default=8,
                   help="very-sparse-tile threshold of the TileBFS contexts (DESIGN.md R25; SpMSpV keeps --thr)")
    p.add_argument("--no-bfs", action="store_true")
    p.add_argument("--no-cpu", action="store_true")
    p.add_argument("--cpu-seconds", type=float, default=12.0)
    p.add_argument("--no-configs", action="store_true", help="skip the per-config table (C1, C2, C4)")
    p.add_argument("--dist-scale", type=int, default=26,
                   help="N > 1: R-MAT scale of the strong-scaling run (C5: the same s26 matrix at every N)")
    p.add_argument("--no-s26", action="store_true", help="N = 1: skip the s26 SpMSpV / TileBFS blocks")
    p.add_argument("--persist", action="store_true",
                   help="turn on the accumulator's L2 persisting window (TSMV_PERSIST=1, opt-in in the library); "
                        "off, the flushed-L2 protocol holds for the workspace too")
    a = p.parse_args(argv)
    a.scaling = "strong"
    a.base_scale, a.base_bfs_scale = a.scale, a.bfs_scale
    return a


def peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(path))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json)"
    except Exception:
        return FALLBACK_HBM, "fallback (B200_PROFILING.md)"


class Clocks:
    """nvidia-smi sampler running during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.path = f"/tmp/tsmv_clocks_{os.getpid()}.csv"

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return None
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], 0.0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in open(self.path):
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx = max(mx, float(f[2]))
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        if not sm:
            return None
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def make_matrix(scale, dtype, device):
    base = synth.rmat(scale, 16, seed=1, device=device)
    return synth.attach_values(base, seed=1, dtype=dtype)


def x_samples(n, k, count, dtype, device):
    return [synth.sample_x(n, k, seed=1 + s, device=device, dtype=dtype) for s in range(count)]


# --------------------------------------------------------------------------- reference arm
def run_reference(args):
    """The oracle (plain single-thread C, oracle/oracle.c) timed on the host on
    the same config / metric; each step = one oracle y = A x on one x sample."""
    import oracle
    world, rank, _ = dist_env()
    if world > 1 and rank != 0:
        return
    dev = "cuda" if torch.cuda.is_available() else "cpu"
    # our arm's workload: T at N = 1, C5 (s26, strong scaling) at N > 1; at s26 each
    # step is a bounded sample of the step (every 8th x entry: still uniform columns)
    scale = args.dist_scale if world > 1 else args.scale
    stride = 8 if world > 1 else 1
    A = make_matrix(scale, args.dtype, dev).to("cpu")
    C = oracle.csc_of(A)
    del A
    colcnt = torch.from_numpy(C.col_ptr[1:] - C.col_ptr[:-1])
    k = synth.density_k(C.n, args.density)
    xs = [(xi[::stride].contiguous(), xv[::stride].contiguous())
          for xi, xv in x_samples(C.n, k, args.warmup + args.steps, args.dtype, "cpu")]
    for s in range(args.warmup):
        oracle.spmspv(C, xs[s][0], xs[s][1])
    flops, tsum, times = 0, 0.0, []
    for s in range(args.warmup, args.warmup + args.steps):
        xi, xv = xs[s]
        t0 = time.perf_counter()
        oracle.spmspv(C, xi, xv)
        dt = time.perf_counter() - t0
        times.append(dt)
        tsum += dt
        flops += 2 * int(colcnt[xi.long()].sum())
    val = flops / tsum / 1e9
    line = {"impl": "reference", "metric": "spmspv_gflops", "value": round(val, 4), "unit": "GFLOP/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(1e3 * tsum / args.steps, 4), "higher_is_better": True,
            "scaling": "strong" if world > 1 else args.scaling,
            "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
            "config": workload_config(args, scale),
            "cpu_baseline": {"value": round(val, 4), "unit": "GFLOP/s", "cores": 1, "kind": "oracle",
                             "sample": f"{args.steps} x samples of k={k} on R-MAT s{scale}"
                                       + (f", every {stride}th x entry per step" if stride > 1 else "")
                                       + " (oracle CSC built once, untimed)"},
            "e2e": {"value": round(val, 4), "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def workload_config(args, scale=None):
    scale = args.scale if scale is None else scale
    return {"workload": f"rmat_s{scale}_ef16_directed_{args.dtype}_x{args.density * 100:g}pct",
            "matrix": f"R-MAT scale {scale}, edgefactor 16, (0.57,0.19,0.19,0.05), unpermuted, coalesced",
            "x_density": args.density, "tile_dim": args.tile_dim, "sparse_tile_max_nnz": args.thr,
            "l2": "flushed before every step (256 MiB write + 256 MiB read of another buffer, outside the events); "
                  + ("accumulator L2 persisting window on (--persist)" if args.persist
                     else "no L2 persisting window: the accumulator workspace is cold too"),
            "parallelism": "single GPU",
            "multi_gpu": f"N > 1 runs C5 (R-MAT s{args.dist_scale}) as strong scaling; at N = 1 the same s26 "
                         "workloads are the spmspv_s26 / bfs_s26 blocks"}


# --------------------------------------------------------------------------- our arm
class L2Flush:
    """Cold, clean L2 before a timed step: write a 256 MiB buffer (> 126 MB L2), then
    read a second 256 MiB buffer so that the dirty lines of the first are written
    back here, outside the timed region, instead of inside the next kernels."""

    def __init__(self, dev):
        self.w = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device=dev)
        self.r = torch.ones(64 * 1024 * 1024, dtype=torch.float32, device=dev)

    def __call__(self):
        self.w.zero_()
        self.sink = self.r.sum()

def flops_of(colcnt, xi):
    return 2 * int(colcnt[xi.long()].sum())


def call_bytes(st, k, sv, nt, m):
    """Algorithmic bytes of one tsmv_spmspv call (= one launch of the SpMSpV kernel)
    for this build's data layout: every byte the method must touch
    once, at its natural width, no sector rounding.  nt = 16 contexts run the flat
    kernel (64-byte tile records, per-column records); others the round-1 kernel."""
    if nt != 16:
        return call_bytes_v6(st, k, sv, nt, m)
    segs, items, side = st["x_segments"], st["tile_items"], st["side_items"]
    hits, hcols, macs = st["hit_tiles"], st["hit_columns"], st["tile_macs"]
    ind = st.get("tile_macs_indirect", macs)
    y = st["y_nnz"]
    phase_a = (k * (4 + sv)                       # read x (index, value)
               + k * (16 + 8)                     # ColInfo of column j + side start of j+1
               + segs * (8 + 8 + 4) + k * 8       # tile-list entries + the segments' x values
               + k * 24                           # side-list entries (start, prefix, x_j)
               + (items + side) // 128 * 4)       # chunk -> entry maps
    phase_b1 = (segs * 20 + k * 24                # list windows read back
                + items * (nt // 8)               # column mask of every tile in a hit tile column
                + hits * 16                       # hit-list entries written
                + side * (4 + sv)                 # row + value of every useful side nonzero
                + side * 8)                       # accumulator update
    phase_b2 = (hits * (16 + 64)                  # hit entry + 64-byte tile record
                + hcols * 8                       # x_j of every hit column
                + ind * (1 + sv)                  # index + value of MACs not inline in the record
                + macs * 8                        # accumulator update
                + y * 4)                          # touched bit, once per output row
    phase_c = (2 * (m // 8)                       # touched bitmap: count + emit passes
               + y * (8 + 8 + 4 + sv))            # acc read + reset, y index + value
    return phase_a + phase_b1 + phase_b2 + phase_c


def call_bytes_v6(st, k, sv, nt, m):
    """Round-1 fused kernel layout (nt = 32 / 64 contexts)."""
    si = 1 if nt == 16 else 2        # packed in-tile row index
    cs = 1 if nt == 16 else 2        # column start offset inside a tile
    mask_b = nt // 8
    phase_a = (k * (4 + sv)                      # read x (index, value)
               + k * 16 + st["x_segments"] * 16  # side col_ptr pair per entry, tile col_ptr pair per segment
               + k * 8                           # scatter x_j -> xd[j]
               + st["x_segments"] * 32 + k * 24)  # segment / side list entries written
    phase_b = (st["tile_items"] * mask_b            # column mask of every tile in a hit tile column
               + st["x_segments"] * 24 + k * 16     # list entries read back
               + st["hit_tiles"] * 16               # TileDesc {off, row, nnz} of tiles whose mask meets x
               + st["hit_columns"] * (2 * cs + 8)   # column start/end + x_j for every hit column
               + st["tile_macs"] * (si + sv)        # row index + value of every useful tile nonzero
               + st["side_items"] * (4 + sv)        # row + value of every useful side nonzero
               + st["y_nnz"] * (8 + 4))             # accumulator write + touched word per output row
    phase_c = (m // 8                               # touched bitmap scan
               + st["y_nnz"] * (8 + 8 + 4 + sv))    # acc read + clear, y index + value
    return phase_a + phase_b + phase_c


def random_access(kms, nt):
    """The kernel's DRAM read sectors (ncu capture, profiles/r02_flat_traffic.json)
    per second of its device time, next to the measured rate of cold random
    sector reads (profiles/r02_random_ceiling.json, scripts/micro/randbw2.cu):
    context for the HBM fraction, not a replacement of it."""
    try:
        t = json.load(open(os.path.join(ROOT, "profiles", "r02_flat_traffic.json" if nt == 16 else "fused_traffic.json")))
        c = json.load(open(os.path.join(ROOT, "profiles", "r02_random_ceiling.json")))
        sec = t.get("dram_sectors_read") or t["dram_bytes_per_launch"] / 32
        ach = sec / (kms * 1e-3) / 1e9
        ceil = c["G_sectors_per_s"]
        return {"dram_sectors_per_launch (ncu)": int(sec), "achieved_G_sectors_per_s": round(ach, 2),
                "random_sector_rate_G_per_s": ceil, "rate_source": c.get("how"), "frac": round(ach / ceil, 4)}
    except Exception:
        return None


def traffic_of(nt, persist=False):
    """DRAM bytes (read + write) per launch of the SpMSpV kernel at T from the ncu
    capture committed under profiles/ (taken under this bench's own L2-flush
    protocol; not measured in this run)."""
    name = ("r02_flat_traffic_bench.json" if persist else "r02s5_flat_traffic_cold.json") if nt == 16 \
        else "fused_traffic.json"
    path = os.path.join(ROOT, "profiles", name)
    try:
        d = json.load(open(path))
        return d.get("dram_bytes_per_launch"), f"profiles/{name}: {d.get('how', 'ncu --set full capture')}"
    except Exception:
        return None, None


def survey_bytes(st, k, sv, nt, macs):
    """SURVEY §8(d) B_alg for the whole call (tile descriptor 4+8+nt/8 B per tile in a
    hit column; fp value + 1..2 B index per useful tile nonzero; side col_ptr pair per
    x entry; 4 B + value per useful side nonzero; read x; write y)."""
    si = 1 if nt == 16 else 2
    return (st["tile_items"] * (4 + 8 + nt // 8) + (macs - st["side_items"]) * (sv + si) + k * 16
            + st["side_items"] * (4 + sv) + k * (4 + sv) + st["y_nnz"] * (4 + sv))


def run_tsmv(args):
    world, rank, local = dist_env()
    # TSMV_DIST_BACKEND=gloo lets the N > 1 path run with several ranks on one
    # GPU (logic check only; NCCL refuses two ranks on one device)
    local = local % max(1, torch.cuda.device_count())
    if world > 1:
        import torch.distributed as dist
        be = os.environ.get("TSMV_DIST_BACKEND", "nccl")
        if be == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(be)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if args.persist:
        # opt-in L2 persisting window over the accumulator workspace (read by tsmv_create)
        os.environ["TSMV_PERSIST"] = "1"
    from paper_conf_icpp_jisl0t022_b200 import tsmv
    sv = 4 if args.dtype == "f32" else 8
    peak, peak_src = peaks()

    A = make_matrix(args.scale, args.dtype, dev)
    colcnt = torch.bincount(A.col_idx.long(), minlength=A.n)
    k = synth.density_k(A.n, args.density)
    xs = x_samples(A.n, k, args.warmup + args.steps, args.dtype, dev)
    flush = L2Flush(dev)

    if world > 1:
        from paper_conf_icpp_jisl0t022_b200 import dist as tdist
        splits = tdist.partition_rows(A.row_ptr, world)
        Al = tdist.local_rows(A, splits, rank)
        D = tdist.DistTiledMatrix(Al, splits, rank, world, dtype=args.dtype, device=local,
                                  tile_dim=args.tile_dim, sparse_tile_max_nnz=args.thr)
        M = D.M
    else:
        D = None
        M = tsmv.TiledMatrix.from_csr(A, dtype=args.dtype, tile_dim=args.tile_dim,
                                      sparse_tile_max_nnz=args.thr, build_bfs=0)
    info = M.info()
    y_idx = torch.empty(M.m, dtype=torch.int32, device=dev)
    y_val = torch.empty(M.m, dtype=torch.float32 if args.dtype == "f32" else torch.float64, device=dev)
    y_nnz = torch.zeros(1, dtype=torch.int64, device=dev)

    def step(s):
        xi, xv = xs[s]
        if D is None:
            M.spmspv_async(xi, xv, y_idx, y_val, y_nnz)
        else:
            lo, hi = D.splits[rank], D.splits[rank + 1]
            own = (xi >= lo) & (xi < hi)
            D.spmspv_async(xi[own], xv[own], y_idx, y_val, y_nnz)

    for s in range(args.warmup):
        flush()
        step(s)
    torch.cuda.synchronize()

    clocks = Clocks(local) if rank == 0 else None
    if clocks:
        clocks.start()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    flops, kexp_bytes, svy_bytes, step_stats = 0, 0, 0, []
    M.set_timing(True)
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    for i in range(args.steps):
        s = args.warmup + i
        flush()
        ev[i][0].record()
        step(s)
        ev[i][1].record()
        torch.cuda.synchronize()
        st = M.last_call_stats()
        flops += flops_of(colcnt, xs[s][0]) if world == 1 else 0
        kexp_bytes += call_bytes(st, k, sv, args.tile_dim, M.m)
        macs = flops_of(colcnt, xs[s][0]) // 2
        svy_bytes += survey_bytes(st, k, sv, args.tile_dim, macs)
        step_stats.append(st)
    torch.cuda.synchronize()
    M_parity = None
    if world == 1:
        nlast = int(y_nnz.item())
        M_parity = (xs[args.warmup + args.steps - 1], (y_idx[:nlast].clone(), y_val[:nlast].clone()))
    if world > 1:
        torch.distributed.barrier()
    kt, ncalls = M.get_timing()
    M.set_timing(False)
    clk = clocks.stop() if clocks else None
    step_ms = [e0.elapsed_time(e1) for e0, e1 in ev]
    ms = sum(step_ms)
    if world > 1:
        import torch.distributed as dist
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t)
        flops = sum(flops_of(colcnt, xs[args.warmup + i][0]) for i in range(args.steps))
    value = flops / (ms * 1e-3) / 1e9

    # roofline of the dominant (only) kernel: one cooperative launch per call.
    # achieved = SURVEY §8(d) B_alg of the call (computed per sample from the
    # call's counters, survey_bytes) / its CUDA-event duration
    kms = ms / args.steps
    achieved = (svy_bytes / args.steps) / (kms * 1e-3) / 1e9
    traffic, tsrc = traffic_of(args.tile_dim, args.persist)
    n_ = max(ncalls, 1)
    roof = {"bound": "hbm", "achieved": round(achieved, 2), "peak": peak, "unit": "GB/s",
            "frac": round(achieved / peak, 4), "traffic": traffic, "traffic_source": tsrc,
            "kernel": ("k_spmspv_flat" if args.tile_dim == 16 else "k_spmspv_fused") + " (the whole call is one cooperative launch)",
            "peak_source": peak_src,
            "B_alg_bytes_per_launch": int(svy_bytes / args.steps),
            "B_alg_definition": "SURVEY §8(d): tile descriptor (4+8+nt/8 B) per tile in a hit tile column + "
                                "(value + index) per useful tile nonzero + 16 B side col_ptr pair per x entry + "
                                "(4 + value) per useful side nonzero + read x + write y",
            "kernel_ms_per_launch": round(kms, 5),
            "ms_per_launch_median": round(statistics.median(step_ms), 5),
            "ms_per_launch_min": round(min(step_ms), 5),
            "phase_ms_per_launch (globaltimer, CTA 0)": {
                "A_x_tiling": round(kt[0] / n_, 5), "B_intersect_multiply": round(kt[1] / n_, 5),
                "C_compact": round(kt[2] / n_, 5), "whole": round(kt[3] / n_, 5)},
            "layout_bytes": {"bytes_per_launch": int(kexp_bytes / args.steps),
                             "what": "every byte of this build's own layout one call touches (64-B tile records, "
                                     "list entries, chunk maps, bitmap passes): DESIGN.md §6",
                             "frac": round(kexp_bytes / (ms * 1e-3) / 1e9 / peak, 4)},
            "random_access": random_access(kms, args.tile_dim)}

    # e2e through the public synchronous API with pinned host buffers (N = 1)
    e2e = None
    if world == 1:
        hx = [(xi.cpu().pin_memory(), xv.cpu().pin_memory()) for xi, xv in xs[args.warmup:]]
        hy_i = torch.empty(M.m, dtype=torch.int32).pin_memory()
        hy_v = torch.empty(M.m, dtype=y_val.dtype).pin_memory()
        for xi, xv in hx[:3]:
            M.spmspv(xi, xv, y_idx=hy_i, y_val=hy_v)
        t_e2e, h2d, d2h = 0.0, 0, 0
        for i, (xi, xv) in enumerate(hx):
            flush()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            yi, yv = M.spmspv(xi, xv, y_idx=hy_i, y_val=hy_v)
            t_e2e += time.perf_counter() - t0
            h2d += xi.numel() * 4 + xv.numel() * sv
            d2h += yi.numel() * (4 + sv)
        e2e = {"value": round(flops / t_e2e / 1e9, 3), "unit": "GFLOP/s",
               "h2d_bytes_per_step": int(h2d / len(hx)), "d2h_bytes_per_step": int(d2h / len(hx)),
               "ms_per_step": round(1e3 * t_e2e / len(hx), 4),
               "path": "tsmv_spmspv (C ABI) with pinned host x and y; wall clock per call"}

    bfs = None
    if not args.no_bfs and world == 1:
        bfs = run_bfs(args, dev, flush, tsmv)
    elif not args.no_bfs:
        del D, M
        bfs = run_bfs_dist(args, dev, flush, rank, world)
    configs = None
    if not args.no_configs and world == 1:
        del M
        configs = run_configs(args, dev, flush, tsmv)
    bfs26 = sp26 = None
    if world == 1 and not args.no_s26:
        torch.cuda.empty_cache()
        sp26 = run_spmspv26(args, dev, flush, tsmv)
    if world == 1 and not args.no_bfs and not args.no_bfs26 and not args.no_s26:
        torch.cuda.empty_cache()
        bfs26 = run_bfs26(args, dev, flush, tsmv)

    cpu = cpu_omp_line = parity = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cpu, cpu_omp_line, parity = cpu_baseline(args, A, colcnt, xs, M_parity)

    if rank == 0:
        mean_st = {kk: sum(s_[kk] for s_ in step_stats) / len(step_stats) for kk in step_stats[0]}
        line = {"metric": "spmspv_gflops", "value": round(value, 3), "unit": "GFLOP/s", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms / args.steps, 5),
                "higher_is_better": True, "scaling": args.scaling,
                "vs_baseline": None, "dtype": args.dtype, "data": "synthetic (seeded R-MAT, seeded x)",
                "config": workload_config(args), "roofline": roof, "cpu_baseline": cpu, "cpu_openmp": cpu_omp_line,
                "parity": parity, "e2e": e2e,
                "gpu_launches": args.steps, "clocks": clk,
                "per_step": {"k": k, "mean_flops": int(flops / args.steps),
                             **{kk: round(v, 1) for kk, v in mean_st.items() if kk != "x_nnz"}},
                "format": {kk: info[kk] for kk in ("nnz", "n_tiles", "n_dense_tiles", "dense_nnz", "side_nnz",
                                                   "build_ms", "bytes_spmspv")},
                "bfs": bfs, "spmspv_s26": sp26, "bfs_s26": bfs26, "configs": configs}
        print(json.dumps(line), flush=True)
    if world > 1:
        torch.distributed.destroy_process_group()


def run_bfs(args, dev, flush, tsmv):
    """TileBFS GTEPS on the symmetrised R-MAT (BASELINE config 3 shape)."""
    A = synth.rmat(args.bfs_scale, 16, seed=1, symmetrize=True, device=dev)
    t0 = time.perf_counter()
    M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", tile_dim=args.tile_dim, sparse_tile_max_nnz=args.bfs_thr)
    build_wall = time.perf_counter() - t0
    info = M.info()
    srcs = bfs_sources(A, args.bfs_sources)
    levels = torch.empty(A.n, dtype=torch.int32, device=dev)
    M.bfs(srcs[0], levels=levels)  # warm-up
    deg, loops = degrees_and_loops(A)
    runs, lv0 = [], None
    for s in srcs:
        flush()
        torch.cuda.synchronize()
        _, st = M.bfs(s, levels=levels)
        runs.append(bfs_run_line(s, st, levels, deg, loops))
        if lv0 is None:
            lv0 = levels.clone()
            lvl_ms = [round(x, 4) for x in st["level_ms"]]
    hm = len(runs) / sum(1.0 / r["gteps"] for r in runs if r["gteps"] > 0)
    hm500 = len(runs) / sum(1.0 / r["gteps_graph500"] for r in runs if r["gteps_graph500"] > 0)
    bpar = None
    if not args.no_cpu:
        # parity of the timed traversal from vertex 0 against the oracle's queue BFS
        import numpy as np

        import oracle
        C = oracle.csc_of(A.to("cpu"))
        ref = oracle.bfs_queue(C, srcs[0])
        bpar = {"ok": bool(np.array_equal(lv0.cpu().numpy(), ref)),
                "checked": f"levels of the timed traversal from {srcs[0]} == oracle.bfs_queue (every vertex)"}
        del C
    # min-id parents (MIN_SECOND semiring) of the last traversal, device time
    parents = torch.empty(A.n, dtype=torch.int32, device=dev)
    M.bfs_parents(levels, parents)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    flush()
    e0.record()
    M.bfs_parents(levels, parents)
    e1.record()
    torch.cuda.synchronize()
    par_ms = e0.elapsed_time(e1)
    # multi-source TileBFS (NEXT-3): 64 sources (vertex 0 + 63 hash-ordered)
    ms_src = [0] + synth.sample_sources(A, 63, seed=2)
    mlv, _ = M.msbfs(ms_src)
    flush()
    torch.cuda.synchronize()
    mlv, mst = M.msbfs(ms_src, levels=mlv)
    del mlv
    msbfs = {"sources": len(ms_src), "ms": round(mst["ms"], 4), "levels": mst["nlevels"],
             "pairs_reached": mst["pairs_reached"], "edges": mst["edges_traversed"],
             "gteps": round(mst["edges_traversed"] / (mst["ms"] * 1e-3) / 1e9, 3)}
    M.close()
    return {"graph": f"rmat_s{args.bfs_scale}_ef16_sym", "sparse_tile_max_nnz": args.bfs_thr,
            "nnz": info["nnz"], "sources": len(runs), "gteps_hmean": round(hm, 3),
            "gteps_graph500_hmean": round(hm500, 3),
            "parents_ms": round(par_ms, 4), "msbfs_64": msbfs, "parity": bpar,
            "level_ms_source0": lvl_ms,
            "build_ms": round(info["build_ms"], 2), "build_wall_s": round(build_wall, 3),
            "edge_count": EDGE_COUNT, "runs": runs}


EDGE_COUNT = ("gteps: edges = sum of out-degrees of reached vertices (R16, directed count of the "
              "symmetrised graph); gteps_graph500: undirected edges of the traversed component "
              "((sum of degrees + self loops) / 2, Graph500 TEPS)")


def bfs_sources(A, count):
    """Vertex 0 plus hash-ordered non-isolated sources (seed 1): SURVEY §8(d) step 4."""
    return [0] + synth.sample_sources(A, max(0, count - 1), seed=1)


def degrees_and_loops(A):
    rp = A.row_ptr
    deg = (rp[1:] - rp[:-1]).to(torch.int64)
    rows = torch.repeat_interleave(torch.arange(A.m, device=rp.device), deg)
    loops = torch.zeros(A.m, dtype=torch.int64, device=rp.device)
    sl = rows[A.col_idx.long() == rows]
    loops[sl] = 1
    del rows
    return deg, loops


def bfs_run_line(s, st, levels, deg, loops):
    r = levels >= 0
    und = int((deg[r].sum() + loops[r].sum()) // 2)
    ms = st["ms"]
    return {"source": int(s), "ms": round(ms, 4), "levels": st["nlevels"],
            "edges": st["edges_traversed"], "edges_graph500": und, "reached": st["reached"],
            "gteps": round(st["edges_traversed"] / (ms * 1e-3) / 1e9, 3),
            "gteps_graph500": round(und / (ms * 1e-3) / 1e9, 3),
            "dirs": "".join({"push_csc": "C", "push_csr": "R", "pull_csc": "P"}.get(d, "?") for d in st["dirs"])}


def run_spmspv26(args, dev, flush, tsmv, steps=8, warm=3):
    """C5 SpMSpV on one GPU: R-MAT s26 directed fp64, x 1 % (671 K entries), the
    N = 1 point of the strong-scaling curve bench.py --gpus N measures."""
    A = make_matrix(26, args.dtype, dev)
    M = tsmv.TiledMatrix.from_csr(A, dtype=args.dtype, tile_dim=args.tile_dim, sparse_tile_max_nnz=args.thr,
                                  build_bfs=0)
    r = spmspv_gflops(M, A, args.dtype, args.density, flush, steps=steps, warm=warm)
    M.close()
    del A
    torch.cuda.empty_cache()
    return {"graph": "rmat_s26_ef16_directed", **r}


def run_bfs26(args, dev, flush, tsmv):
    """C5 on one GPU: TileBFS on the symmetrised R-MAT s26 (2.1 G nonzeros, int64
    offsets), vertex 0 + 7 sources, the bench's BFS context settings."""
    t0 = time.perf_counter()
    A = synth.rmat(26, 16, seed=1, symmetrize=True, device=dev)
    gen = time.perf_counter() - t0
    torch.cuda.empty_cache()
    M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", tile_dim=args.tile_dim, sparse_tile_max_nnz=args.bfs_thr)
    info = M.info()
    srcs = bfs_sources(A, args.bfs26_sources)
    deg, loops = degrees_and_loops(A)
    levels = torch.empty(A.n, dtype=torch.int32, device=dev)
    M.bfs(srcs[0], levels=levels)
    runs = []
    for s in srcs:
        flush()
        torch.cuda.synchronize()
        _, st = M.bfs(s, levels=levels)
        runs.append(bfs_run_line(s, st, levels, deg, loops))
    M.close()
    hm = len(runs) / sum(1.0 / r["gteps"] for r in runs if r["gteps"] > 0)
    hm500 = len(runs) / sum(1.0 / r["gteps_graph500"] for r in runs if r["gteps_graph500"] > 0)
    return {"graph": "rmat_s26_ef16_sym", "nnz": A.nnz, "sparse_tile_max_nnz": args.bfs_thr,
            "sources": len(runs), "gteps_hmean": round(hm, 3), "gteps_graph500_hmean": round(hm500, 3),
            "gen_s": round(gen, 2), "build_ms": round(info["build_ms"], 2), "edge_count": EDGE_COUNT,
            "parity": "tests/test_gpu_bench_configs.py::test_c5_s26 (levels from vertex 0 vs oracle)", "runs": runs}


def run_bfs_dist(args, dev, flush, rank, world):
    """Row-block partitioned TileBFS on the symmetrised R-MAT: each
    rank builds its nnz-balanced row block; one NCCL all-gather of the owned
    frontier bitmaps + one all-reduce of (m_f, m_u) per level.  Time = max over
    ranks of the CUDA-event time of the traversal; edges = sum of out-degrees of
    the reached vertices (all ranks)."""
    import torch.distributed as dist
    from paper_conf_icpp_jisl0t022_b200 import dist as tdist
    A = synth.rmat(args.bfs_scale, 16, seed=1, symmetrize=True, device=dev)
    srcs = [0] + synth.sample_sources(A, max(0, args.bfs_sources - 1), seed=1)
    splits = tdist.partition_rows(A.row_ptr, world, row_weight=tdist.BFS_ROW_WEIGHT)
    Al = tdist.local_rows(A, splits, rank)
    nnz = A.nnz
    del A
    t0 = time.perf_counter()
    D = tdist.DistTiledMatrix(Al, splits, rank, world, dtype="pattern", device=dev.index,
                              tile_dim=args.tile_dim, sparse_tile_max_nnz=args.bfs_thr)
    build_wall = time.perf_counter() - t0
    rowlen = (Al.row_ptr[1:] - Al.row_ptr[:-1]).to(torch.int64)
    D.bfs(srcs[0])  # warm-up
    runs = []
    for s in srcs:
        flush()
        torch.cuda.synchronize()
        dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        lv, nl = D.bfs(s)
        e1.record()
        torch.cuda.synchronize()
        t = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        red = torch.stack([(rowlen * (lv >= 0)).sum(), (lv >= 0).sum()]).to(torch.int64)
        dist.all_reduce(red)
        ms, edges = float(t), int(red[0])
        runs.append({"source": int(s), "ms": round(ms, 4), "levels": int(nl), "edges": edges,
                     "reached": int(red[1]), "gteps": round(edges / (ms * 1e-3) / 1e9, 3)})
    hm = len(runs) / sum(1.0 / r["gteps"] for r in runs if r["gteps"] > 0)
    return {"graph": f"rmat_s{args.bfs_scale}_ef16_sym", "nnz": nnz, "gteps_hmean": round(hm, 3),
            "partition": f"row blocks x{world} (nnz + {tdist.BFS_ROW_WEIGHT:g} x rows balanced)", "build_wall_s": round(build_wall, 3),
            "edge_count": "sum of out-degrees of reached vertices (directed count of the symmetrised graph)",
            "time": "CUDA events around the whole traversal, max over ranks", "runs": runs}


def spmspv_gflops(M, A, dtype, density, flush, steps=5, warm=2):
    """Device-timed SpMSpV at `density` on context M (fresh x per step, L2 flushed)."""
    dev = A.row_ptr.device
    colcnt = torch.bincount(A.col_idx.long(), minlength=A.n)
    k = max(1, synth.density_k(A.n, density))
    xs = x_samples(A.n, k, steps + warm, dtype, dev)
    vt = torch.float32 if dtype == "f32" else torch.float64
    yi = torch.empty(A.m, dtype=torch.int32, device=dev)
    yv = torch.empty(A.m, dtype=vt, device=dev)
    yn = torch.zeros(1, dtype=torch.int64, device=dev)
    for s in range(warm):
        M.spmspv_async(xs[s][0], xs[s][1], yi, yv, yn)
    ms, flops = 0.0, 0
    for s in range(warm, warm + steps):
        flush()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        M.spmspv_async(xs[s][0], xs[s][1], yi, yv, yn)
        e1.record()
        torch.cuda.synchronize()
        ms += e0.elapsed_time(e1)
        flops += flops_of(colcnt, xs[s][0])
    return {"density": density, "k": k, "us_per_call": round(1e3 * ms / steps, 2),
            "gflops": round(flops / (ms * 1e-3) / 1e9, 3), "y_nnz": int(yn.item())}


def bfs_gteps(M, A, flush, sources):
    lv = torch.empty(A.n, dtype=torch.int32, device=A.row_ptr.device)
    M.bfs(sources[0], levels=lv)
    out = []
    for s in sources:
        flush()
        torch.cuda.synchronize()
        _, st = M.bfs(s, levels=lv)
        out.append({"source": int(s), "ms": round(st["ms"], 3), "levels": st["nlevels"],
                    "gteps": round(st["edges_traversed"] / (st["ms"] * 1e-3) / 1e9, 3)})
    return out


def run_configs(args, dev, flush, tsmv):
    """The other BASELINE.json configs (C1, C2, C4), a few device-timed calls each."""
    res = {}
    # C1: 2D 5-point 64x64, fp64, x 1 %, BFS from 0
    A = synth.stencil2d(64, 64, device=dev)
    M = tsmv.TiledMatrix.from_csr(A)
    res["C1_stencil2d_64x64"] = {"spmspv_f64": spmspv_gflops(M, A, "f64", 0.01, flush),
                                 "bfs": bfs_gteps(M, A, flush, [0])}
    M.close()
    # C2: R-MAT s20 ef16 sweep, fp64 and fp32
    base = synth.rmat(20, 16, seed=1, device=dev)
    c2 = {}
    for dt in ("f64", "f32"):
        A = synth.attach_values(base, seed=1, dtype=dt)
        M = tsmv.TiledMatrix.from_csr(A, dtype=dt, build_bfs=0)
        c2[dt] = [spmspv_gflops(M, A, dt, d, flush) for d in (0.0001, 0.001, 0.01, 0.1)]
        M.close()
    res["C2_rmat_s20_sweep"] = c2
    # Graph500-style relabelled R-MAT s22 (hubs spread over the id space): SpMSpV at
    # 1 % (directed, fp64) and TileBFS (symmetrised), to show the numbers above are
    # not an artefact of the unpermuted generator's hub locality
    A = synth.attach_values(synth.rmat(22, 16, seed=1, device=dev, permute=True), seed=1)
    M = tsmv.TiledMatrix.from_csr(A, build_bfs=0)
    sp = spmspv_gflops(M, A, "f64", 0.01, flush)
    M.close()
    del A
    A = synth.rmat(22, 16, seed=1, symmetrize=True, device=dev, permute=True)
    M = tsmv.TiledMatrix.from_csr(A, dtype="pattern", sparse_tile_max_nnz=args.bfs_thr)
    res["rmat_s22_permuted"] = {"spmspv_f64_1pct": sp,
                                "bfs": bfs_gteps(M, A, flush, [synth.sample_sources(A, 1, seed=1)[0]])}
    M.close()
    del A
    # C4: 3D 7-point 256^3 and banded (2^20, b = 64): TileBFS + SpMSpV at 1 %
    for name, A in (("C4_stencil3d_256", synth.stencil3d(256, device=dev)),
                    ("C4_banded_2e20_b64", synth.banded(1 << 20, 64, device=dev))):
        M = tsmv.TiledMatrix.from_csr(A)
        res[name] = {"nnz": A.nnz, "spmspv_f64": spmspv_gflops(M, A, "f64", 0.01, flush),
                     "bfs": bfs_gteps(M, A, flush, [0])}
        M.close()
        del A
    return res


def cpu_baseline(args, A, colcnt, xs, parity_y):
    """(1) The oracle as it stands on the host (1 core), bounded to ~cpu_seconds of
    CPU work; (2) the OpenMP speed baseline (cpu_omp/: SpMSpV-bucket column merge)
    on all host cores over the same samples; (3) parity of one timed step: y of
    the last timed sample from the CUDA path against the oracle (index set
    bit-exact, values within 1e-12 * sum_j |a_ij x_j|)."""
    import numpy as np

    import cpu_omp
    import oracle
    Ac = A.to("cpu")
    C = oracle.csc_of(Ac)
    flops, t = 0, 0.0
    used = 0
    cc = colcnt.cpu()
    for xi, xv in xs:
        xi_c, xv_c = xi.cpu(), xv.cpu()
        t0 = time.perf_counter()
        oracle.spmspv(C, xi_c, xv_c)
        t += time.perf_counter() - t0
        flops += flops_of(cc, xi_c)
        used += 1
        if t > args.cpu_seconds:
            break
    cpu = {"value": round(flops / t / 1e9, 5), "unit": "GFLOP/s", "cores": 1, "kind": "oracle",
           "sample": f"{used} x samples (k={xs[0][0].numel()}) of the same workload, oracle CSC built once untimed",
           "nproc": os.cpu_count(), "cpu_model": cpu_omp.cpu_model()}
    Co = cpu_omp.csc_of(Ac)
    nth = cpu_omp.threads()
    fo, to = 0, 0.0
    for xi, xv in xs[:used]:
        xi_c, xv_c = xi.cpu().numpy(), xv.cpu().numpy()
        t0 = time.perf_counter()
        cpu_omp.spmspv(Co, xi_c, xv_c, nthreads=nth)
        to += time.perf_counter() - t0
        fo += flops_of(cc, torch.from_numpy(xi_c))
    omp = {"value": round(fo / to / 1e9, 5), "unit": "GFLOP/s", "cores": nth, "kind": "openmp (cpu_omp/)",
           "sample": f"the same {used} samples", "cpu_model": cpu_omp.cpu_model(), "nproc": os.cpu_count()}
    parity = None
    if parity_y is not None:
        (pxi, pxv), (yi, yv) = parity_y
        ri, rv = oracle.spmspv(C, pxi.cpu().numpy(), pxv.cpu().numpy())
        Ca = oracle.CSC(C.m, C.n, C.col_ptr, C.row_idx, np.abs(C.val))
        _, mag = oracle.spmspv(Ca, pxi.cpu().numpy(), np.abs(pxv.cpu().numpy()))
        gi, gv = yi.cpu().numpy(), yv.cpu().numpy()
        same = gi.shape == ri.shape and bool(np.array_equal(gi, ri))
        ok = same and bool(np.all(np.abs(gv - rv) <= 1e-12 * mag))
        parity = {"ok": ok, "checked": "y of the last timed step vs oracle.spmspv: index set bit-exact, "
                                       "|y - y_ref| <= 1e-12 * sum_j |a_ij x_j|",
                  "y_nnz": int(gi.size), "y_nnz_oracle": int(ri.size)}
    return cpu, omp, parity


def run_dist(args):
    """N > 1 (C5): strong scaling on the same R-MAT s26 at every N.
    Every rank generates the seeded matrix, keeps its nnz-balanced row block in a
    libtsmv context that owns its NCCL communicator (bootstrap: one unique id from
    rank 0 over torch.distributed), and the timed calls are the collective
    tsmv_spmspv (owned x in, owned y out: count all-gather + x broadcasts inside
    the library) and tsmv_bfs (the level loop and the per-level frontier
    broadcasts inside the library).  Time = CUDA events around each call on every
    rank, max over ranks; value = all flops / that time."""
    import torch.distributed as dist
    world, rank, local = dist_env()
    local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist.init_process_group("nccl", device_id=dev)
    from paper_conf_icpp_jisl0t022_b200 import dist as tdist
    uid = tdist.bootstrap_unique_id()
    flush = L2Flush(dev)

    def max_over_ranks(v):
        t = torch.tensor([v], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t)

    # ---- SpMSpV, x 1 %, fp64
    A = make_matrix(args.dist_scale, args.dtype, dev)
    colcnt = torch.bincount(A.col_idx.long(), minlength=A.n)
    splits = tdist.partition_rows(A.row_ptr, world)
    t0 = time.perf_counter()
    D = tdist.DistMatrix(tdist.local_rows(A, splits, rank), splits, rank, world, uid, dtype=args.dtype,
                         device=local, tile_dim=args.tile_dim, sparse_tile_max_nnz=args.thr, build_bfs=0)
    build_s = time.perf_counter() - t0
    n = A.n
    del A
    torch.cuda.empty_cache()
    k = synth.density_k(n, args.density)
    lo, hi = splits[rank], splits[rank + 1]
    xs = []
    for xi, xv in x_samples(n, k, args.warmup + args.steps, args.dtype, dev):
        own = (xi >= lo) & (xi < hi)
        xs.append((xi[own].contiguous(), xv[own].contiguous(), 2 * int(colcnt[xi.long()].sum())))
    m_loc = hi - lo
    y_idx = torch.empty(m_loc, dtype=torch.int32, device=dev)
    y_val = torch.empty(m_loc, dtype=torch.float32 if args.dtype == "f32" else torch.float64, device=dev)
    for s in range(args.warmup):
        D.spmspv(xs[s][0], xs[s][1], y_idx=y_idx, y_val=y_val)
    clocks = Clocks(local) if rank == 0 else None
    if clocks:
        clocks.start()
    dist.barrier()
    torch.cuda.synchronize()
    step_ms, flops = [], 0
    for i in range(args.steps):
        xi, xv, fl = xs[args.warmup + i]
        flush()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        D.spmspv(xi, xv, y_idx=y_idx, y_val=y_val)
        e1.record()
        torch.cuda.synchronize()
        step_ms.append(e0.elapsed_time(e1))
        flops += fl
    torch.cuda.synchronize()
    dist.barrier()
    clk = clocks.stop() if clocks else None
    ms = max_over_ranks(sum(step_ms))
    value = flops / (ms * 1e-3) / 1e9
    # e2e: the same collective call with pinned host x and y, wall clock, max over ranks
    hx = [(xi.cpu().pin_memory(), xv.cpu().pin_memory()) for xi, xv, _ in xs[args.warmup:]]
    hy_i = torch.empty(m_loc, dtype=torch.int32).pin_memory()
    hy_v = torch.empty(m_loc, dtype=y_val.dtype).pin_memory()
    dist.barrier()
    t_e2e, h2d, d2h = 0.0, 0, 0
    for xi, xv in hx:
        flush()
        torch.cuda.synchronize()
        dist.barrier()
        t0 = time.perf_counter()
        yi, yv = D.spmspv(xi, xv, y_idx=hy_i, y_val=hy_v)
        t_e2e += time.perf_counter() - t0
        h2d += xi.numel() * 4 + xv.numel() * xv.element_size()
        d2h += yi.numel() * (4 + yv.element_size())
    t_e2e = max_over_ranks(t_e2e)
    n_e2e = len(hx)
    D.close()
    del D, y_idx, y_val, colcnt, xs, hx
    torch.cuda.empty_cache()

    # ---- TileBFS on the symmetrised s26, vertex 0 + 7 sources
    bfs = None
    if not args.no_bfs:
        A = synth.rmat(args.dist_scale, 16, seed=1, symmetrize=True, device=dev)
        torch.cuda.empty_cache()
        splits_b = tdist.partition_rows(A.row_ptr, world, row_weight=tdist.BFS_ROW_WEIGHT)
        uid_b = tdist.bootstrap_unique_id()   # a unique id serves one communicator only
        Db = tdist.DistMatrix(tdist.local_rows(A, splits_b, rank), splits_b, rank, world, uid_b, dtype="pattern",
                              device=local, tile_dim=args.tile_dim, sparse_tile_max_nnz=args.bfs_thr)
        srcs = bfs_sources(A, args.bfs26_sources)
        deg, loops = degrees_and_loops(A)
        nnz = A.nnz
        del A
        torch.cuda.empty_cache()
        lvl = torch.empty(splits_b[rank + 1] - splits_b[rank], dtype=torch.int32, device=dev)
        Db.bfs(srcs[0], levels=lvl)
        runs = []
        for s in srcs:
            flush()
            torch.cuda.synchronize()
            dist.barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            _, st = Db.bfs(s, levels=lvl)
            e1.record()
            torch.cuda.synchronize()
            tms = max_over_ranks(e0.elapsed_time(e1))
            # Graph500 count: reached rows of every rank
            r = lvl >= 0
            part = torch.stack([deg[splits_b[rank]:splits_b[rank + 1]][r].sum(),
                                loops[splits_b[rank]:splits_b[rank + 1]][r].sum()])
            dist.all_reduce(part)
            und = int((part[0] + part[1]) // 2)
            runs.append({"source": int(s), "ms": round(tms, 4), "levels": st["nlevels"],
                         "edges": st["edges_traversed"], "edges_graph500": und, "reached": st["reached"],
                         "gteps": round(st["edges_traversed"] / (tms * 1e-3) / 1e9, 3),
                         "gteps_graph500": round(und / (tms * 1e-3) / 1e9, 3),
                         "dirs": "".join({"push_csc": "C", "push_csr": "R", "pull_csc": "P"}.get(d, "?")
                                         for d in st["dirs"])})
        Db.close()
        hm = len(runs) / sum(1.0 / x["gteps"] for x in runs if x["gteps"] > 0)
        hm500 = len(runs) / sum(1.0 / x["gteps_graph500"] for x in runs if x["gteps_graph500"] > 0)
        bfs = {"graph": f"rmat_s{args.dist_scale}_ef16_sym", "nnz": nnz, "sources": len(runs),
               "gteps_hmean": round(hm, 3), "gteps_graph500_hmean": round(hm500, 3),
               "sparse_tile_max_nnz": args.bfs_thr, "partition": f"row blocks x{world} (nnz + {tdist.BFS_ROW_WEIGHT:g} x rows balanced)",
               "time": "CUDA events around the collective tsmv_bfs, max over ranks", "edge_count": EDGE_COUNT,
               "runs": runs}
    if rank == 0:
        line = {"metric": "spmspv_gflops", "value": round(value, 3), "unit": "GFLOP/s", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms / args.steps, 5),
                "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": args.dtype,
                "data": "synthetic (seeded R-MAT, seeded x)",
                "config": {"workload": f"rmat_s{args.dist_scale}_ef16_directed_{args.dtype}_x{args.density * 100:g}pct",
                           "matrix": f"R-MAT scale {args.dist_scale}, edgefactor 16, unpermuted, coalesced",
                           "x_density": args.density, "tile_dim": args.tile_dim, "sparse_tile_max_nnz": args.thr,
                           "l2": "flushed before every step (256 MiB write + 256 MiB read, outside the events)",
                           "parallelism": f"row blocks x{world} (nnz-balanced), NCCL communicator inside libtsmv",
                           "scaling_rule": "strong: the same matrix at every N (C5); N = 1: bench.py's spmspv_s26 / bfs_s26 blocks"},
                "e2e": {"value": round(flops / t_e2e / 1e9, 3), "unit": "GFLOP/s",
                        "h2d_bytes_per_step": int(h2d / n_e2e), "d2h_bytes_per_step": int(d2h / n_e2e),
                        "path": "collective tsmv_spmspv (C ABI) with pinned host owned x and y; wall clock, max over ranks"},
                "gpu_launches": args.steps, "clocks": clk,
                "comm": {"nranks": world, "backend": "NCCL (communicator owned by the libtsmv context)",
                         "nccl_version": ".".join(str(v) for v in torch.cuda.nccl.version())},
                "build_s_rank0": round(build_s, 2), "bfs": bfs}
        print(json.dumps(line), flush=True)
    dist.barrier()
    dist.destroy_process_group()


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
    elif int(os.environ.get("WORLD_SIZE", "1")) > 1 or os.environ.get("TSMV_BENCH_DIST"):
        run_dist(args)   # TSMV_BENCH_DIST=1: the N > 1 path with one rank (checks it on one GPU)
    else:
        run_tsmv(args)


if __name__ == "__main__":
    main()
