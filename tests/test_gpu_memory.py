"""Device-memory hygiene of the C ABI: tsmv_create must release every builder
temporary (CUB scratch, sort keys, the symmetry check's key copies) and
tsmv_destroy everything the ctx owns; a create/destroy loop must not drift."""
import pytest
import torch

import synth

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


def test_create_destroy_does_not_leak():
    from paper_conf_icpp_jisl0t022_b200 import tsmv
    A = synth.rmat(18, 16, seed=2, symmetrize=True, device=DEV)
    Av = synth.attach_values(synth.rmat(18, 16, seed=3, device=DEV), seed=1)
    torch.cuda.synchronize()
    torch.cuda.empty_cache()

    def cycle():
        for M in (tsmv.TiledMatrix.from_csr(A, dtype="pattern"), tsmv.TiledMatrix.from_csr(Av)):
            info = M.info()
            M.close()
        torch.cuda.synchronize()
        return info

    cycle()  # first use: lazy module loading, caches
    free0, _ = torch.cuda.mem_get_info()
    for _ in range(4):
        cycle()
    torch.cuda.empty_cache()
    free1, _ = torch.cuda.mem_get_info()
    # one build of these graphs holds ~0.3 GB of temporaries: 4 leaked builds would show
    assert free0 - free1 < 32 << 20, f"device memory drift {(free0 - free1) / 2**20:.1f} MiB after 4 create/destroy"


def test_context_holds_only_its_structures():
    from paper_conf_icpp_jisl0t022_b200 import tsmv
    A = synth.rmat(18, 16, seed=2, symmetrize=True, device=DEV)
    torch.cuda.synchronize()
    torch.cuda.empty_cache()
    free0, _ = torch.cuda.mem_get_info()
    M = tsmv.TiledMatrix.from_csr(A, dtype="pattern")
    torch.cuda.synchronize()
    free1, _ = torch.cuda.mem_get_info()
    info = M.info()
    owned = info["bytes_spmspv"] + info["bytes_bfs"] + info["bytes_workspace"]
    # the ctx's own accounting plus small per-context buffers (lists, BFS vertex lists, counters)
    assert free0 - free1 < owned + 4 * A.n * 4 + (64 << 20), \
        f"ctx uses {(free0 - free1) / 2**20:.0f} MiB, accounts for {owned / 2**20:.0f} MiB"
    M.close()
