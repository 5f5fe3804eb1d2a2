"""The bench's timed SpMSpV step at T with its L2 flush before every call, for an
ncu capture with --cache-control none (DRAM traffic under the bench's own
protocol: inputs cold, the persisting accumulator window as in bench.py).  Dev aid."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import synth  # noqa: E402
from paper_conf_icpp_jisl0t022_b200 import tsmv  # noqa: E402

dev = torch.device("cuda", 0)
cfg = bench.parse([])
A = bench.make_matrix(cfg.scale, cfg.dtype, dev)
M = tsmv.TiledMatrix.from_csr(A, dtype=cfg.dtype, tile_dim=cfg.tile_dim, sparse_tile_max_nnz=cfg.thr, build_bfs=0)
flush = bench.L2Flush(dev)
k = synth.density_k(A.n, cfg.density)
yi = torch.empty(A.m, dtype=torch.int32, device=dev)
yv = torch.empty(A.m, dtype=torch.float64, device=dev)
yn = torch.zeros(1, dtype=torch.int64, device=dev)
for xi, xv in bench.x_samples(A.n, k, 8, cfg.dtype, dev):
    flush()
    M.spmspv_async(xi, xv, yi, yv, yn)
torch.cuda.synchronize()
print("done")
