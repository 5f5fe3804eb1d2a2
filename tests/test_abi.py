"""CPU-side checks of the C-ABI boundary: libtsmv.so loads and exports every
function include/tsmv.h declares; host-only entry points behave."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "tsmv.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = set(re.findall(r"\b(tsmv_[a-z_0-9]+)\s*\(", src))
    return sorted(names)


@pytest.fixture(scope="module")
def lib():
    from paper_conf_icpp_jisl0t022_b200 import build
    build.build()
    return ctypes.CDLL(build.LIB)


def test_every_declared_symbol_exported(lib):
    names = _declared()
    assert len(names) >= 15
    for n in names:
        assert hasattr(lib, n), f"{n} declared in include/tsmv.h but not exported"


def test_binding_covers_abi():
    from paper_conf_icpp_jisl0t022_b200 import tsmv
    assert set(_declared()) == set(tsmv.EXPORTED)


def test_host_only_calls():
    from paper_conf_icpp_jisl0t022_b200 import tsmv
    assert tsmv.tsmv_version() >> 16 == 1
    o = tsmv.default_options()
    assert o.tile_dim == 16 and o.sparse_tile_max_nnz == 2 and o.nranks == 1
    assert abs(o.push_csr_density - 0.05) < 1e-15 and o.pull_alpha == 2.0   # B200 defaults
    # direction rule (reading R9) with the paper's thresholds (0.01, Beamer's 14)
    pap = tsmv.default_options(push_csr_density=0.01, pull_alpha=14.0)
    assert tsmv.choose_dir(1000, 1, 10, 10_000, pap) == tsmv.DIR_PUSH_CSC
    assert tsmv.choose_dir(1000, 10, 10, 10_000, pap) == tsmv.DIR_PUSH_CSR
    assert tsmv.choose_dir(1000, 10, 1000, 10_000, pap) == tsmv.DIR_PULL_CSC
    # B200 defaults: Push-CSR from 5 % of n, Pull-CSC when m_f > m_u / 2
    assert tsmv.choose_dir(1000, 10, 10, 10_000) == tsmv.DIR_PUSH_CSC
    assert tsmv.choose_dir(1000, 50, 10, 10_000) == tsmv.DIR_PUSH_CSR
    assert tsmv.choose_dir(1000, 10, 1000, 10_000) == tsmv.DIR_PUSH_CSC
    assert tsmv.choose_dir(1000, 10, 6000, 10_000) == tsmv.DIR_PULL_CSC
    # reading R9': Beamer's 14 on a level whose frontier grew >= 4x (defaults 14, 4)
    assert o.pull_alpha_burst == 14.0 and o.burst_growth == 4.0
    assert tsmv.choose_dir(1000, 10, 1000, 10_000, None, 2) == tsmv.DIR_PULL_CSC    # 10 >= 4 x 2: 1000 > 10000/14
    assert tsmv.choose_dir(1000, 10, 1000, 10_000, None, 3) == tsmv.DIR_PUSH_CSC    # 10 < 4 x 3: alpha 2
    assert tsmv.choose_dir(1000, 10, 1000, 10_000, None, 0) == tsmv.DIR_PUSH_CSC    # unknown previous level
    off = tsmv.default_options(pull_alpha_burst=0.0)
    assert tsmv.choose_dir(1000, 10, 1000, 10_000, off, 1) == tsmv.DIR_PUSH_CSC     # R9' off: alpha 2
    o.force_dir = tsmv.DIR_PUSH_CSR
    assert tsmv.choose_dir(1000, 1, 1000, 10, o) == tsmv.DIR_PUSH_CSR
    assert tsmv.tsmv_destroy(None) == tsmv.OK
    assert tsmv.tsmv_owned_words(None) == 0


def test_create_rejects_bad_args_without_gpu():
    from paper_conf_icpp_jisl0t022_b200 import tsmv
    ctx = ctypes.c_void_p()
    o = tsmv.default_options(tile_dim=24)
    rp = (ctypes.c_int64 * 2)(0, 0)
    st = tsmv.tsmv_create(ctypes.byref(ctx), 1, 1, ctypes.cast(rp, ctypes.c_void_p), None, None, tsmv.PATTERN,
                          ctypes.byref(o))
    assert st == tsmv.EINVAL and b"tile_dim" in tsmv.tsmv_last_error()
    assert not ctx.value


def test_nccl_unique_id_without_gpu():
    """Bootstrap of a distributed context: NCCL is loaded at run time
    and a unique id needs no GPU."""
    from paper_conf_icpp_jisl0t022_b200 import tsmv
    a, b = tsmv.nccl_unique_id(), tsmv.nccl_unique_id()
    assert len(a) == 128 and any(a) and a != b
    assert tsmv.tsmv_nccl_unique_id(None) == tsmv.EINVAL


def test_options_layout_matches_header():
    """ctypes mirror of tsmv_options has the header's field order (last: nccl_unique_id)."""
    from paper_conf_icpp_jisl0t022_b200 import tsmv
    src = open(os.path.join(ROOT, "include", "tsmv.h")).read()
    body = src[src.index("typedef struct {\n    int32_t device;"):src.index("} tsmv_options;")]
    body = re.sub(r"/\*.*?\*/", "", body, flags=re.S)
    names = re.findall(r"\b([a-z_]+)\s*(?:,\s*([a-z_]+))?\s*;", body)
    flat = [x for pair in names for x in pair if x]
    assert flat == [f for f, _ in tsmv.tsmv_options._fields_]
