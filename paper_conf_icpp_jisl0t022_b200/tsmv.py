"""Thin ctypes binding of libtsmv.so (include/tsmv.h).  Argument marshalling
only: every step of the hot path runs in the library's sm_100a kernels.

The `tsmv_*` functions mirror the C ABI one to one; `TiledMatrix` is a small
convenience wrapper that owns a context and passes torch tensors (device or
host) as raw pointers together with torch's current CUDA stream.

If libtsmv.so is missing this module raises ImportError: there is no CPU
fallback anywhere in the product path.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("TSMV_LIB") or os.path.join(_HERE, "libtsmv.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"libtsmv.so not built ({LIB_PATH}); run `python -c 'import __graft_entry__ as g; g.build()'`")

_lib = ctypes.CDLL(LIB_PATH)

# --------------------------------------------------------------------------- ABI types
OK, EINVAL, ENOMEM, ECUDA, ENCCL, ECAPACITY, EUNSUPPORTED = range(7)
DIST_WIDE = 0x100   # tsmv_bfs_dist_expand hint for late pull levels (TSMV_DIST_WIDE)
F64, F32, PATTERN = 0, 1, 2
PLUS_TIMES, OR_AND, MIN_SECOND = 0, 1, 2
DIR_AUTO, DIR_PUSH_CSC, DIR_PUSH_CSR, DIR_PULL_CSC = 0, 1, 2, 3
MAX_LEVELS = 65536
_SEMIRINGS = {"plus_times": PLUS_TIMES, "or_and": OR_AND, "min_second": MIN_SECOND}
_DTYPES = {"f64": F64, "f32": F32, "pattern": PATTERN}
DIR_NAMES = {DIR_PUSH_CSC: "push_csc", DIR_PUSH_CSR: "push_csr", DIR_PULL_CSC: "pull_csc"}


class tsmv_options(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("tile_dim", ctypes.c_int32),
                ("sparse_tile_max_nnz", ctypes.c_int32), ("build_bfs", ctypes.c_int32),
                ("push_csr_density", ctypes.c_double), ("pull_alpha", ctypes.c_double),
                ("force_dir", ctypes.c_int32), ("rank", ctypes.c_int32), ("nranks", ctypes.c_int32),
                ("row_begin", ctypes.c_int64), ("row_splits", ctypes.POINTER(ctypes.c_int64)),
                ("nccl_unique_id", ctypes.c_void_p), ("row_driven_density", ctypes.c_double),
                ("pull_alpha_burst", ctypes.c_double), ("burst_growth", ctypes.c_double)]


class tsmv_call_stats(ctypes.Structure):
    _fields_ = [("x_nnz", ctypes.c_int64), ("x_segments", ctypes.c_int64), ("tile_items", ctypes.c_int64),
                ("side_items", ctypes.c_int64), ("y_nnz", ctypes.c_int64), ("hit_tiles", ctypes.c_int64),
                ("hit_columns", ctypes.c_int64), ("tile_macs", ctypes.c_int64),
                ("tile_macs_indirect", ctypes.c_int64)]


class tsmv_info(ctypes.Structure):
    _fields_ = [("nrows", ctypes.c_int64), ("ncols", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("tile_dim", ctypes.c_int32), ("symmetric", ctypes.c_int32), ("n_tiles", ctypes.c_int64),
                ("n_dense_tiles", ctypes.c_int64), ("dense_nnz", ctypes.c_int64), ("side_nnz", ctypes.c_int64),
                ("bytes_spmspv", ctypes.c_int64), ("bytes_bfs", ctypes.c_int64),
                ("bytes_workspace", ctypes.c_int64), ("build_ms", ctypes.c_double)]


class tsmv_msbfs_stats(ctypes.Structure):
    _fields_ = [("nlevels", ctypes.c_int32), ("pairs_reached", ctypes.c_int64), ("edges_traversed", ctypes.c_int64),
                ("ms", ctypes.c_double)]


class tsmv_bfs_stats(ctypes.Structure):
    _fields_ = [("nlevels", ctypes.c_int32), ("reached", ctypes.c_int64), ("edges_traversed", ctypes.c_int64),
                ("ms", ctypes.c_double), ("dir_per_level", ctypes.c_int32 * MAX_LEVELS),
                ("frontier_per_level", ctypes.c_int64 * MAX_LEVELS), ("level_ms", ctypes.c_float * MAX_LEVELS)]


_vp, _i64, _i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
_SIGS = {
    "tsmv_default_options": (ctypes.c_int, [ctypes.POINTER(tsmv_options)]),
    "tsmv_nccl_unique_id": (ctypes.c_int, [_vp]),
    "tsmv_create": (ctypes.c_int, [ctypes.POINTER(_vp), _i64, _i64, _vp, _vp, _vp, ctypes.c_int,
                                   ctypes.POINTER(tsmv_options)]),
    "tsmv_spmspv": (ctypes.c_int, [_vp, ctypes.c_int, _i64, _vp, _vp, _i64, _vp, _vp, ctypes.POINTER(_i64), _vp]),
    "tsmv_spmspv_async": (ctypes.c_int, [_vp, ctypes.c_int, _i64, _vp, _vp, _i64, _vp, _vp, _vp, _vp]),
    "tsmv_set_timing": (ctypes.c_int, [_vp, _i32]),
    "tsmv_set_direction_rule": (ctypes.c_int, [_vp, ctypes.c_double, ctypes.c_double, _i32]),
    "tsmv_set_trace": (ctypes.c_int, [_vp, _vp]),
    "tsmv_trace_words": (_i64, [_vp]),
    "tsmv_get_timing": (ctypes.c_int, [_vp, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(_i64)]),
    "tsmv_last_call_stats": (ctypes.c_int, [_vp, ctypes.POINTER(tsmv_call_stats)]),
    "tsmv_bfs": (ctypes.c_int, [_vp, _i64, _vp, ctypes.POINTER(tsmv_bfs_stats), _vp]),
    "tsmv_bfs_parents": (ctypes.c_int, [_vp, _vp, _vp, _vp]),
    "tsmv_msbfs": (ctypes.c_int, [_vp, _i32, _vp, _vp, ctypes.POINTER(tsmv_msbfs_stats), _vp]),
    "tsmv_bfs_dist_begin": (ctypes.c_int, [_vp, _i64, _vp, ctypes.POINTER(_i64), _vp]),
    "tsmv_bfs_dist_set_degrees": (ctypes.c_int, [_vp, _vp]),
    "tsmv_bfs2d_scatter": (ctypes.c_int, [_vp, _vp, _vp, _i64, _vp, _i64, _vp]),
    "tsmv_bfs2d_merge": (ctypes.c_int, [_vp, _vp, _i32, _i64, _i64, _vp, _vp, _i32, _vp, _vp, _vp, _vp, _vp]),
    "tsmv_bfs2d_expand": (ctypes.c_int, [_vp, _i32, _vp, _vp, _vp, _vp, _vp, _i32, _vp]),
    "tsmv_bfs2d_list": (ctypes.c_int, [_vp, _vp, _i64, _vp, _vp, _vp]),
    "tsmv_bfs_dist_expand": (ctypes.c_int, [_vp, _i32, _vp, _vp]),
    "tsmv_bfs_dist_merge": (ctypes.c_int, [_vp, _vp, _i64, ctypes.POINTER(_i64), _vp]),
    "tsmv_owned_words": (_i64, [_vp]),
    "tsmv_choose_dir": (_i32, [ctypes.POINTER(tsmv_options), _i64, _i64, _i64, _i64, _i64]),
    "tsmv_get_info": (ctypes.c_int, [_vp, ctypes.POINTER(tsmv_info)]),
    "tsmv_export_csr": (ctypes.c_int, [_vp, _vp, _vp, _vp]),
    "tsmv_export_bitmask_tiles": (ctypes.c_int, [_vp, _i32, _i64, _vp, _vp, _vp, ctypes.POINTER(_i64)]),
    "tsmv_destroy": (ctypes.c_int, [_vp]),
    "tsmv_last_error": (ctypes.c_char_p, []),
    "tsmv_version": (_i32, []),
}
for _name, (_res, _args) in _SIGS.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args
    globals()[_name] = _f

EXPORTED = sorted(_SIGS)


class TsmvError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"tsmv status {status}: {msg}")
        self.status = status


def check(status, what=""):
    if status != OK:
        raise TsmvError(status, f"{what}: {tsmv_last_error().decode(errors='replace')}")


def _ptr(t: Optional[torch.Tensor]):
    if t is None:
        return None
    assert t.is_contiguous(), "tensors passed to libtsmv must be contiguous"
    return t.data_ptr() if t.numel() else None


_RAW_STREAM = getattr(torch._C, "_cuda_getCurrentRawStream", None)


def _stream(stream=None):
    if stream is not None:
        return stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)
    if torch.cuda.is_available():
        if _RAW_STREAM is not None:  # the current stream's handle without building a Stream object
            return _RAW_STREAM(torch.cuda.current_device())
        return torch.cuda.current_stream().cuda_stream
    return None


def default_options(**kw) -> tsmv_options:
    o = tsmv_options()
    check(tsmv_default_options(ctypes.byref(o)), "tsmv_default_options")
    for k, v in kw.items():
        if v is None:
            continue
        if k == "row_splits":
            arr = (ctypes.c_int64 * len(v))(*[int(x) for x in v])
            o._splits_keepalive = arr
            o.row_splits = ctypes.cast(arr, ctypes.POINTER(ctypes.c_int64))
        elif k == "nccl_unique_id":
            buf = ctypes.create_string_buffer(bytes(v), 128)
            o._nccl_keepalive = buf
            o.nccl_unique_id = ctypes.cast(buf, ctypes.c_void_p)
        else:
            setattr(o, k, v)
    return o


class TiledMatrix:
    """A matrix converted to the tiled format on one GPU (one tsmv context)."""

    def __init__(self, m, n, row_ptr, col_idx, values=None, dtype: Optional[str] = None, **opts):
        if dtype is None:
            dtype = "pattern" if values is None else ("f32" if values.dtype == torch.float32 else "f64")
        self.dtype = dtype
        self.vtype = torch.float32 if dtype == "f32" else torch.float64
        self.m, self.n = int(m), int(n)
        row_ptr = row_ptr.to(torch.int64).contiguous()
        col_idx = col_idx.to(torch.int32).contiguous()
        if values is not None:
            values = values.to(self.vtype).contiguous()
        self.opts = default_options(**opts)
        self.device = torch.device("cuda", self.opts.device) if torch.cuda.is_available() else None
        ctx = _vp()
        args = (self.m, self.n, _ptr(row_ptr) or row_ptr.data_ptr(), _ptr(col_idx),
                _ptr(values) if dtype != "pattern" else None, _DTYPES[dtype], ctypes.byref(self.opts))
        st = tsmv_create(ctypes.byref(ctx), *args)
        if st == ENOMEM and self.device is not None:
            # the library allocates with cudaMalloc: hand torch's cached blocks back and retry once
            torch.cuda.empty_cache()
            st = tsmv_create(ctypes.byref(ctx), *args)
        check(st, "tsmv_create")
        self.ctx = ctx
        self.nnz = int(col_idx.numel())

    @classmethod
    def from_csr(cls, A, dtype: Optional[str] = None, **opts):
        vals = A.values
        if dtype == "pattern":
            vals = None
        return cls(A.m, A.n, A.row_ptr, A.col_idx, vals, dtype=dtype, **opts)

    # -- SpMSpV ---------------------------------------------------------------
    def spmspv(self, x_idx: torch.Tensor, x_val: Optional[torch.Tensor] = None, semiring="plus_times",
               y_idx: Optional[torch.Tensor] = None, y_val: Optional[torch.Tensor] = None, stream=None):
        """y = A x.  x_idx strictly ascending int32.  Returns (y_idx, y_val) views of
        length y_nnz (y_val None for or_and).  Tensors may live on the GPU or the host."""
        sr = _SEMIRINGS[semiring] if isinstance(semiring, str) else int(semiring)
        dev = x_idx.device
        if x_idx.dtype != torch.int32 or not x_idx.is_contiguous():
            x_idx = x_idx.to(torch.int32).contiguous()
        if x_val is not None and (x_val.dtype != self.vtype or not x_val.is_contiguous()):
            x_val = x_val.to(self.vtype).contiguous()
        if y_idx is None:
            y_idx = torch.empty(self.m, dtype=torch.int32, device=dev)
        if y_val is None and sr != OR_AND:
            y_val = torch.empty(self.m, dtype=self.vtype, device=dev)
        ynnz = ctypes.c_int64(0)
        st = tsmv_spmspv(self.ctx, sr, x_idx.numel(), _ptr(x_idx), _ptr(x_val), y_idx.numel(), _ptr(y_idx),
                         _ptr(y_val) if sr != OR_AND else None, ctypes.byref(ynnz), _stream(stream))
        check(st, "tsmv_spmspv")
        k = ynnz.value
        return y_idx[:k], (y_val[:k] if y_val is not None and sr != OR_AND else None)

    def spmspv_async(self, x_idx: torch.Tensor, x_val: Optional[torch.Tensor], y_idx: torch.Tensor,
                     y_val: Optional[torch.Tensor], y_nnz: torch.Tensor, semiring="plus_times", stream=None):
        """Device-only, no synchronisation; y_nnz (int64[1] on the device) receives the size."""
        sr = _SEMIRINGS[semiring] if isinstance(semiring, str) else int(semiring)
        if x_idx.dtype != torch.int32 or not x_idx.is_contiguous():
            x_idx = x_idx.to(torch.int32).contiguous()
        if x_val is not None and (x_val.dtype != self.vtype or not x_val.is_contiguous()):
            x_val = x_val.to(self.vtype).contiguous()
        if y_nnz.dtype != torch.int64 or y_nnz.numel() != 1 or y_nnz.device != x_idx.device:
            raise ValueError("spmspv_async: y_nnz must be one int64 on the device of x")
        check(tsmv_spmspv_async(self.ctx, sr, x_idx.numel(), _ptr(x_idx), _ptr(x_val), y_idx.numel(), _ptr(y_idx),
                                _ptr(y_val) if sr != OR_AND else None, _ptr(y_nnz), _stream(stream)),
              "tsmv_spmspv_async")

    def set_direction_rule(self, push_csr_density: Optional[float] = None, pull_alpha: Optional[float] = None,
                           force_dir: Optional[int] = None):
        """Retune the TileBFS direction rule (R9) for the next traversals."""
        o = self.opts
        if push_csr_density is not None:
            o.push_csr_density = float(push_csr_density)
        if pull_alpha is not None:
            o.pull_alpha = float(pull_alpha)
        if force_dir is not None:
            o.force_dir = int(force_dir)
        check(tsmv_set_direction_rule(self.ctx, o.push_csr_density, o.pull_alpha, o.force_dir),
              "tsmv_set_direction_rule")

    def set_timing(self, enable: bool = True):
        check(tsmv_set_timing(self.ctx, 1 if enable else 0), "tsmv_set_timing")

    def get_timing(self):
        """(ms x-scan, ms expand, ms compact, ms whole call) summed, and the number of calls."""
        ms = (ctypes.c_double * 4)()
        n = ctypes.c_int64(0)
        check(tsmv_get_timing(self.ctx, ms, ctypes.byref(n)), "tsmv_get_timing")
        return [ms[i] for i in range(4)], n.value

    def last_call_stats(self) -> dict:
        s = tsmv_call_stats()
        check(tsmv_last_call_stats(self.ctx, ctypes.byref(s)), "tsmv_last_call_stats")
        return {f: getattr(s, f) for f, _ in s._fields_}

    # -- BFS ------------------------------------------------------------------
    def bfs(self, source: int, levels: Optional[torch.Tensor] = None, stream=None, with_stats=True):
        if levels is None:
            levels = torch.empty(self.m, dtype=torch.int32, device=self.device)
        stats = tsmv_bfs_stats() if with_stats else None
        check(tsmv_bfs(self.ctx, int(source), _ptr(levels), ctypes.byref(stats) if stats else None,
                       _stream(stream)), "tsmv_bfs")
        if not with_stats:
            return levels, None
        L = stats.nlevels
        d = {"nlevels": L, "reached": stats.reached, "edges_traversed": stats.edges_traversed, "ms": stats.ms,
             "dirs": [DIR_NAMES.get(stats.dir_per_level[i], "?") for i in range(min(L, MAX_LEVELS))],
             "frontier": [stats.frontier_per_level[i] for i in range(min(L, MAX_LEVELS))],
             "level_ms": [stats.level_ms[i] for i in range(min(L, MAX_LEVELS))]}
        return levels, d

    def bfs_parents(self, levels: torch.Tensor, parents: Optional[torch.Tensor] = None, stream=None):
        """Min-id BFS parents (min-second semiring) from the levels of a finished bfs()."""
        if parents is None:
            parents = torch.empty(self.m, dtype=torch.int32, device=self.device)
        check(tsmv_bfs_parents(self.ctx, _ptr(levels), _ptr(parents), _stream(stream)), "tsmv_bfs_parents")
        return parents

    def msbfs(self, sources, levels: Optional[torch.Tensor] = None, stream=None):
        """Multi-source TileBFS from up to 64 sources at once.  Returns (levels
        int32[m, nsrc] on the device, vertex-major, -1 = unreachable; stats)."""
        src = torch.as_tensor(list(sources), dtype=torch.int64)
        ns = int(src.numel())
        if levels is None:
            levels = torch.empty(self.m, ns, dtype=torch.int32, device=self.device)
        st = tsmv_msbfs_stats()
        check(tsmv_msbfs(self.ctx, ns, src.data_ptr(), _ptr(levels), ctypes.byref(st), _stream(stream)), "tsmv_msbfs")
        return levels, {"nlevels": st.nlevels, "pairs_reached": st.pairs_reached,
                        "edges_traversed": st.edges_traversed, "ms": st.ms}

    # -- introspection -----------------------------------------------------------
    def info(self) -> dict:
        s = tsmv_info()
        check(tsmv_get_info(self.ctx, ctypes.byref(s)), "tsmv_get_info")
        return {f: getattr(s, f) for f, _ in s._fields_}

    def export_csr(self):
        rp = torch.zeros(self.m + 1, dtype=torch.int64)
        ci = torch.zeros(max(self.nnz, 1), dtype=torch.int32)
        vals = torch.zeros(max(self.nnz, 1), dtype=self.vtype) if self.dtype != "pattern" else None
        check(tsmv_export_csr(self.ctx, rp.data_ptr(), ci.data_ptr(), vals.data_ptr() if vals is not None else None),
              "tsmv_export_csr")
        return rp, ci[:self.nnz], (vals[:self.nnz] if vals is not None else None)

    def export_bitmask_tiles(self, orient: int, max_tiles: int = 1 << 16):
        nt = self.opts.tile_dim
        tI = torch.zeros(max_tiles, dtype=torch.int64)
        tJ = torch.zeros(max_tiles, dtype=torch.int64)
        w = torch.zeros(max_tiles * nt, dtype=torch.int64)
        cnt = ctypes.c_int64(0)
        check(tsmv_export_bitmask_tiles(self.ctx, orient, max_tiles, tI.data_ptr(), tJ.data_ptr(), w.data_ptr(),
                                        ctypes.byref(cnt)), "tsmv_export_bitmask_tiles")
        out = []
        for t in range(cnt.value):
            out.append((int(tI[t]), int(tJ[t]), [int(x) & ((1 << 64) - 1) for x in w[t * nt:(t + 1) * nt]]))
        return out

    def close(self):
        if getattr(self, "ctx", None):
            tsmv_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


def nccl_unique_id() -> bytes:
    """128 bytes for tsmv_options.nccl_unique_id (call on one rank, share with all)."""
    buf = ctypes.create_string_buffer(128)
    check(tsmv_nccl_unique_id(buf), "tsmv_nccl_unique_id")
    return buf.raw


def choose_dir(n, frontier, m_f, m_u, opts: Optional[tsmv_options] = None, prev_frontier: int = 0) -> int:
    return int(tsmv_choose_dir(ctypes.byref(opts) if opts is not None else None, n, frontier, m_f, m_u,
                               prev_frontier))
