"""ctypes binding of include/npp.h — argument marshalling only.

Every step of the path (selection, kernels, Split combine) runs inside libnpp.so; this module converts
torch tensors to raw pointers and structs to dicts.  There is no CPU fallback: importing it without the
built library raises.  PyTorch provides device memory and streams only.
"""
from __future__ import annotations

import ctypes
import os

import torch

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("NPP_LIB_PATH") or os.path.join(_PKG, "libnpp.so")  # override: experiment builds

# enums (include/npp.h)
OK, ERR_INVALID_ARG, ERR_UNSUPPORTED, ERR_ALIGNMENT, ERR_WORKSPACE, ERR_NO_FEASIBLE, ERR_CUDA = 0, -1, -2, -3, -4, -5, -6
DTYPES = {"f32": 0, "i32": 1, "i64": 2, "f64": 3}
TORCH_DTYPES = {"f32": torch.float32, "i32": torch.int32, "i64": torch.int64, "f64": torch.float64}
PATTERNS = {"SUM_ROWS": 0, "SUM_COLS": 1, "KMEANS_ASSIGN": 2, "LOGREG_GRAD": 3,
            "SUM_WEIGHTED_ROWS": 4, "SUM_WEIGHTED_COLS": 5, "SUM_ROWS_COLS": 6,
            "KMEANS_UPDATE": 7, "PAGERANK": 8}
STRATEGIES = {"AUTO": 0, "LITERAL": 1, "1D": 2, "TB_T": 3, "WARP": 4}
SPAN_ONE, SPAN_ALL, SPAN_N, SPLIT_K = 0, 1, 2, 3
CLASS_RX, CLASS_MX, CLASS_KMEANS, CLASS_LOGREG, CLASS_EMPTY, CLASS_RC, CLASS_KMUPDATE, CLASS_PAGERANK = range(8)


class NppError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"npp error {status}: {msg}")
        self.status = status


class Level(ctypes.Structure):
    _fields_ = [("dim", ctypes.c_int32), ("block", ctypes.c_int32), ("span", ctypes.c_int32),
                ("reserved", ctypes.c_int32), ("factor", ctypes.c_int64), ("chunk", ctypes.c_int64),
                ("grid", ctypes.c_int64)]


class Mapping(ctypes.Structure):
    _fields_ = [("nlevels", ctypes.c_int32), ("kernel_class", ctypes.c_int32), ("vec", ctypes.c_int32),
                ("staged", ctypes.c_int32), ("level", Level * 4), ("score", ctypes.c_int64),
                ("dop", ctypes.c_int64), ("threads", ctypes.c_int64), ("grid", ctypes.c_int64),
                ("block", ctypes.c_int32 * 3), ("smem_bytes", ctypes.c_int32),
                ("workspace_bytes", ctypes.c_int64), ("claim_tiles", ctypes.c_int64),
                ("temp", ctypes.c_int32), ("reserved2", ctypes.c_int32), ("temp_stride", ctypes.c_int64 * 2),
                ("static_tiles", ctypes.c_int64)]


class Limits(ctypes.Structure):
    _fields_ = [("sm_count", ctypes.c_int32), ("max_threads_per_sm", ctypes.c_int32),
                ("max_threads_per_block", ctypes.c_int32), ("max_block_dim", ctypes.c_int32 * 3),
                ("warp_size", ctypes.c_int32), ("max_blocks_per_sm", ctypes.c_int32),
                ("regs_per_sm", ctypes.c_int32), ("regs_per_block", ctypes.c_int32),
                ("regs_per_thread", ctypes.c_int32), ("reserved", ctypes.c_int32),
                ("smem_per_block", ctypes.c_int64)]


EXEC_OVERLAP, EXEC_NO_PDL = 1, 2  # npp.h NPP_EXEC_OVERLAP / NPP_EXEC_NO_PDL
TEMP_NONE, TEMP_MALLOC, TEMP_PREALLOC = 0, 1, 2  # npp.h npp_temp

EXPORTS = ("npp_version", "npp_last_error", "npp_limits_query", "npp_select", "npp_plan",
           "npp_plan_with_mapping", "npp_plan_mapping", "npp_plan_workspace_bytes", "npp_execute",
           "npp_execute_ex", "npp_execute_host", "npp_enumerate", "npp_plan_launches", "npp_plan_destroy",
           "npp_plan_tiles", "npp_execute_traced")


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run `python -m paper_conf_micro_leebsro14_b200.build` "
                          "(no CPU fallback exists)")
    lib = ctypes.CDLL(LIB_PATH)
    P, I64P = ctypes.c_void_p, ctypes.POINTER(ctypes.c_int64)
    lib.npp_version.restype = ctypes.c_int
    lib.npp_last_error.restype = ctypes.c_char_p
    lib.npp_limits_query.argtypes = [ctypes.c_int, ctypes.POINTER(Limits)]
    lib.npp_select.argtypes = [ctypes.c_int, I64P, ctypes.c_int, ctypes.c_int, ctypes.POINTER(Limits),
                               ctypes.c_int, ctypes.POINTER(Mapping)]
    lib.npp_plan.argtypes = [ctypes.c_int, I64P, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                             ctypes.POINTER(Limits), ctypes.POINTER(P)]
    lib.npp_plan_with_mapping.argtypes = [ctypes.c_int, I64P, ctypes.c_int, ctypes.c_int,
                                          ctypes.POINTER(Mapping), ctypes.POINTER(Limits), ctypes.POINTER(P)]
    lib.npp_plan_mapping.argtypes = [P, ctypes.POINTER(Mapping)]
    lib.npp_plan_workspace_bytes.argtypes = [P]
    lib.npp_plan_workspace_bytes.restype = ctypes.c_int64
    lib.npp_execute.argtypes = [P, ctypes.POINTER(P), ctypes.c_int, P, P, P]
    lib.npp_execute_ex.argtypes = [P, ctypes.POINTER(P), ctypes.c_int, P, P, P, ctypes.c_uint]
    lib.npp_execute_host.argtypes = [P, ctypes.POINTER(P), ctypes.c_int, P, ctypes.POINTER(P), P, P, P]
    lib.npp_plan_launches.argtypes = [P]
    lib.npp_plan_tiles.argtypes = [P]
    lib.npp_plan_tiles.restype = ctypes.c_int64
    lib.npp_execute_traced.argtypes = [P, ctypes.POINTER(P), ctypes.c_int, P, P, P, P]
    lib.npp_enumerate.argtypes = [ctypes.c_int, I64P, ctypes.c_int, ctypes.c_int, ctypes.POINTER(Limits),
                                  ctypes.c_void_p, ctypes.c_int64]
    lib.npp_enumerate.restype = ctypes.c_int64
    lib.npp_plan_destroy.argtypes = [P]
    lib.npp_plan_destroy.restype = None
    return lib


_lib = _load()


def lib():
    return _lib


def _check(status: int):
    if status != OK:
        raise NppError(status, _lib.npp_last_error().decode())


def _shape_arr(shape):
    return (ctypes.c_int64 * len(shape))(*[int(s) for s in shape])


# ---------------------------------------------------------------- limits / mapping conversions

def limits_to_dict(l: Limits) -> dict:
    return dict(sm_count=l.sm_count, max_threads_per_sm=l.max_threads_per_sm,
                max_threads_per_block=l.max_threads_per_block, max_block_dim=tuple(l.max_block_dim),
                warp_size=l.warp_size, max_blocks_per_sm=l.max_blocks_per_sm, regs_per_sm=l.regs_per_sm,
                regs_per_block=l.regs_per_block, regs_per_thread=l.regs_per_thread,
                smem_per_block=l.smem_per_block)


def limits_from_dict(d: dict) -> Limits:
    l = Limits()
    for k, v in d.items():
        if k == "max_block_dim":
            l.max_block_dim = (ctypes.c_int32 * 3)(*v)
        else:
            setattr(l, k, int(v))
    return l


def mapping_to_dict(m: Mapping) -> dict:
    levels = [dict(dim=m.level[i].dim, block=m.level[i].block, span=m.level[i].span,
                   factor=m.level[i].factor, chunk=m.level[i].chunk, grid=m.level[i].grid)
              for i in range(m.nlevels)]
    return dict(nlevels=m.nlevels, kernel_class=m.kernel_class, vec=m.vec, staged=m.staged, levels=levels,
                score=m.score,
                dop=m.dop, threads=m.threads, grid=m.grid, block=list(m.block), smem_bytes=m.smem_bytes,
                workspace_bytes=m.workspace_bytes, claim_tiles=m.claim_tiles, temp=m.temp,
                temp_stride=[m.temp_stride[0], m.temp_stride[1]], static_tiles=m.static_tiles)


def mapping_from_dict(d: dict) -> Mapping:
    m = Mapping()
    m.nlevels = len(d["levels"])
    m.vec = int(d.get("vec", 1))
    for i, lv in enumerate(d["levels"]):
        m.level[i].dim = int(lv["dim"])
        m.level[i].block = int(lv["block"])
        m.level[i].span = int(lv["span"])
        m.level[i].factor = int(lv.get("factor", 1))
    m.temp = int(d.get("temp", 0))
    ts = d.get("temp_stride", (0, 0))
    m.temp_stride[0], m.temp_stride[1] = int(ts[0]), int(ts[1])
    return m


def limits_query(device: int = 0) -> dict:
    l = Limits()
    _check(_lib.npp_limits_query(device, ctypes.byref(l)))
    return limits_to_dict(l)


def select(pattern: str, shape, dtype: str, limits: dict, strategy: str = "AUTO") -> dict:
    """Pure selector (no CUDA call): the mapping record for DESIGN.md §3."""
    m = Mapping()
    l = limits_from_dict(limits)
    _check(_lib.npp_select(PATTERNS[pattern], _shape_arr(shape), len(shape), DTYPES[dtype], ctypes.byref(l),
                           STRATEGIES[strategy], ctypes.byref(m)))
    return mapping_to_dict(m)


def enumerate_mappings(pattern: str, shape, dtype: str, limits: dict) -> list:
    """npp_enumerate: every hard-feasible Algorithm 1 candidate with ControlDOP applied, as LITERAL
    records (S2-S6, S9), in enumeration order."""
    l = limits_from_dict(limits)
    n = _lib.npp_enumerate(PATTERNS[pattern], _shape_arr(shape), len(shape), DTYPES[dtype], ctypes.byref(l),
                           None, 0)
    if n < 0:
        _check(int(n))
    arr = (Mapping * max(1, n))()
    got = _lib.npp_enumerate(PATTERNS[pattern], _shape_arr(shape), len(shape), DTYPES[dtype], ctypes.byref(l),
                             arr, n)
    if got < 0:
        _check(int(got))
    return [mapping_to_dict(arr[i]) for i in range(n)]


def _ptr(t) -> ctypes.c_void_p:
    return ctypes.c_void_p(t.data_ptr() if t is not None else 0)


def _stream_handle(stream) -> ctypes.c_void_p:
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream))


class Plan:
    """An immutable plan (npp_plan / npp_plan_with_mapping) plus its workspace buffer."""

    def __init__(self, pattern: str, shape, dtype: str = "f32", strategy: str = "AUTO",
                 limits: dict | None = None, mapping: dict | None = None, device=None):
        self.pattern, self.shape, self.dtype = pattern, tuple(int(s) for s in shape), dtype
        self.strategy = strategy if mapping is None else "EXPLICIT"
        h = ctypes.c_void_p()
        lp = ctypes.byref(limits_from_dict(limits)) if limits is not None else None
        if mapping is None:
            st = _lib.npp_plan(PATTERNS[pattern], _shape_arr(self.shape), len(self.shape), DTYPES[dtype],
                               STRATEGIES[strategy], lp, ctypes.byref(h))
        else:
            fm = mapping_from_dict(mapping)
            st = _lib.npp_plan_with_mapping(PATTERNS[pattern], _shape_arr(self.shape), len(self.shape),
                                            DTYPES[dtype], ctypes.byref(fm), lp, ctypes.byref(h))
        _check(st)
        self._h = h
        m = Mapping()
        _check(_lib.npp_plan_mapping(h, ctypes.byref(m)))
        self.mapping = mapping_to_dict(m)
        self.workspace_bytes = int(_lib.npp_plan_workspace_bytes(h))
        self.launches = int(_lib.npp_plan_launches(h))
        self.device = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        # the workspace must be zero before first use; kernels leave it zero (Split tickets reset)
        self.workspace = (torch.zeros(self.workspace_bytes, dtype=torch.uint8, device=self.device)
                          if self.workspace_bytes > 0 else None)

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value and _lib is not None:  # _lib is None during interpreter shutdown
            _lib.npp_plan_destroy(h)
            self._h = None

    def out_shape(self):
        p, s = self.pattern, self.shape
        if p in ("SUM_ROWS", "SUM_WEIGHTED_ROWS"):
            return (s[0],)
        if p in ("SUM_COLS", "SUM_WEIGHTED_COLS"):
            return (s[1],)
        if p == "SUM_ROWS_COLS":
            return (s[0] + s[1],)
        if p == "KMEANS_ASSIGN":
            return (s[0],)
        if p == "KMEANS_UPDATE":
            return (s[2], s[1] + 1)
        if p == "PAGERANK":
            return (s[0],)
        return (s[0], s[2])

    def out_dtype(self):
        if self.pattern == "KMEANS_ASSIGN":
            return torch.int32
        return TORCH_DTYPES[self.dtype]

    def new_out(self):
        return torch.empty(self.out_shape(), dtype=self.out_dtype(), device=self.device)

    def execute(self, ins, out, stream=None, workspace=None, overlap=False, pdl=True):
        """Enqueue on `stream` (default: torch's current stream). Inputs must be contiguous device tensors.
        overlap=True is npp_execute_ex(NPP_EXEC_OVERLAP): the caller asserts no earlier work on the
        stream writes `ins` (the staged kernels then start while the previous kernel drains).
        pdl=False is NPP_EXEC_NO_PDL: plain stream-ordered launches (isolated kernel timing)."""
        for t in ins:
            if not t.is_contiguous():
                raise ValueError("inputs must be contiguous")
        arr = (ctypes.c_void_p * len(ins))(*[t.data_ptr() for t in ins])
        ws = workspace if workspace is not None else self.workspace
        flags = (EXEC_OVERLAP if overlap else 0) | (0 if pdl else EXEC_NO_PDL)
        _check(_lib.npp_execute_ex(self._h, arr, len(ins), _ptr(out), _ptr(ws), _stream_handle(stream), flags))
        return out

    @property
    def tiles(self) -> int:
        """npp_plan_tiles: tiles (or regions) of the plan's schedule, 0 if it has none."""
        return int(_lib.npp_plan_tiles(self._h))

    def execute_traced(self, ins, out, stream=None):
        """npp_execute_traced: execute and return (block of each tile, loads of each tile) as int32 tensors
        on the device (white-box check of the runtime rule's schedule, S8)."""
        n = self.tiles
        trace = torch.zeros(2 * max(n, 1), dtype=torch.int32, device=self.device)
        trace[:n] = -1
        arr = (ctypes.c_void_p * len(ins))(*[t.data_ptr() for t in ins])
        _check(_lib.npp_execute_traced(self._h, arr, len(ins), _ptr(out), _ptr(self.workspace),
                                       _stream_handle(stream), _ptr(trace)))
        return trace[:n], trace[n:2 * n]

    def execute_host(self, host_ins, host_out, dev_ins, dev_out, stream=None):
        """End-to-end: H2D copy of host_ins into dev_ins, execute, D2H into host_out, synchronise."""
        hi = (ctypes.c_void_p * len(host_ins))(*[t.data_ptr() for t in host_ins])
        di = (ctypes.c_void_p * len(dev_ins))(*[t.data_ptr() for t in dev_ins])
        _check(_lib.npp_execute_host(self._h, hi, len(host_ins), _ptr(host_out), di, _ptr(dev_out),
                                     _ptr(self.workspace), _stream_handle(stream)))
        return host_out


# ---------------------------------------------------------------- convenience front-ends (Fig 1)

_PLAN_CACHE: dict = {}


def _cached_plan(pattern, shape, dtype, strategy, device, stream=None):
    """One plan (and so one workspace) per (pattern, shape, dtype, strategy, device, STREAM): executes on
    one stream are ordered, so they may share a workspace; executes on different streams get their own
    (npp.h: concurrent executes need distinct workspaces)."""
    with torch.cuda.device(device):
        sh = _stream_handle(stream).value
    key = (pattern, tuple(shape), dtype, strategy, str(device), sh)
    p = _PLAN_CACHE.get(key)
    if p is None:
        p = Plan(pattern, shape, dtype, strategy, device=device)
        _PLAN_CACHE[key] = p
    return p


def _dtype_name(t: torch.Tensor) -> str:
    for k, v in TORCH_DTYPES.items():
        if v == t.dtype:
            return k
    raise TypeError(f"unsupported dtype {t.dtype}")


def sum_rows(m: torch.Tensor, strategy: str = "AUTO", out=None, stream=None) -> torch.Tensor:
    """m mapRows { r => r reduce + } (Fig 1) on a contiguous [R, C] CUDA tensor."""
    p = _cached_plan("SUM_ROWS", m.shape, _dtype_name(m), strategy, m.device, stream)
    return p.execute([m], out if out is not None else p.new_out(), stream)


def sum_cols(m: torch.Tensor, strategy: str = "AUTO", out=None, stream=None) -> torch.Tensor:
    """m mapCols { c => c reduce + } (Fig 1)."""
    p = _cached_plan("SUM_COLS", m.shape, _dtype_name(m), strategy, m.device, stream)
    return p.execute([m], out if out is not None else p.new_out(), stream)


def sum_rows_cols(m: torch.Tensor, out=None, stream=None):
    """Both Naive Bayes counts (§VI-E) in one pass over m: returns (row sums, column
    sums), views of one [R + C] output (SUM_ROWS_COLS, strategy AUTO)."""
    R = m.shape[0]
    p = _cached_plan("SUM_ROWS_COLS", m.shape, _dtype_name(m), "AUTO", m.device, stream)
    o = p.execute([m], out if out is not None else p.new_out(), stream)
    return o[:R], o[R:]


def sum_weighted_rows(m, v, strategy="AUTO", out=None, stream=None):
    p = _cached_plan("SUM_WEIGHTED_ROWS", m.shape, _dtype_name(m), strategy, m.device, stream)
    return p.execute([m, v], out if out is not None else p.new_out(), stream)


def sum_weighted_cols(m, v, strategy="AUTO", out=None, stream=None):
    p = _cached_plan("SUM_WEIGHTED_COLS", m.shape, _dtype_name(m), strategy, m.device, stream)
    return p.execute([m, v], out if out is not None else p.new_out(), stream)


def kmeans_assign(x, c, strategy="AUTO", out=None, stream=None):
    N, D = x.shape
    if c.dim() != 2 or c.shape[1] != D:
        raise ValueError("kmeans_assign: centroids must be [K, D] with the points' D")
    p = _cached_plan("KMEANS_ASSIGN", (N, D, c.shape[0]), "f32", strategy, x.device, stream)
    return p.execute([x, c], out if out is not None else p.new_out(), stream)


def kmeans_update(x, a, K, out=None, stream=None):
    """Centroid update after an assignment (groupBy a + Reduce, Table I): [K, D+1] fp32 with
    row k = (Σ_{i: a_i = k} x_i, count_k). New centroids are U[:, :D] / U[:, D:] where the count > 0."""
    N, D = x.shape
    if a.dtype != torch.int32 or a.numel() != N:
        raise ValueError("kmeans_update: keys must be an int32 vector with one key per point")
    p = _cached_plan("KMEANS_UPDATE", (N, D, int(K)), "f32", "AUTO", x.device, stream)
    return p.execute([x, a], out if out is not None else p.new_out(), stream)


def pagerank_step(rowptr, colidx, pr, outdeg, out=None, stream=None):
    """One PageRank step (Fig 5) over the CSR of in-neighbours: rowptr int64 [N+1], colidx
    int32 [E], pr f32 [N], outdeg int32 [N] -> (1-0.85)/N + 0.85 * Σ_{w in nbrs(n)} pr[w]/outdeg[w]."""
    N, E = pr.shape[0], colidx.shape[0]
    p = _cached_plan("PAGERANK", (N, E), "f32", "AUTO", pr.device, stream)
    return p.execute([rowptr, colidx, pr, outdeg], out if out is not None else p.new_out(), stream)


def pagerank_shard(local_rowptr, local_colidx, pr, outdeg, lo, hi, out=None, stream=None):
    """Rows [lo, hi) of a PageRank step: the shard's CSR (rowptr rebased to 0, hi-lo+1 entries) against the
    whole graph's pr / outdeg (PAGERANK shape {rows, E, N})."""
    p = _cached_plan("PAGERANK", (hi - lo, local_colidx.shape[0], pr.shape[0]), "f32", "AUTO", pr.device, stream)
    return p.execute([local_rowptr, local_colidx, pr, outdeg], out if out is not None else p.new_out(), stream)


def logreg_grad(x, y, w, B, strategy="AUTO", out=None, stream=None):
    """g[b, j] = Σ_{i in batch b} x_ij (σ(x_i·w) − y_i) over B equal mini-batches of the rows of x."""
    n, C = x.shape
    if B < 1 or n % B != 0:
        raise ValueError(f"logreg_grad: {n} rows do not split into {B} equal mini-batches")
    if y.numel() != n or w.numel() != C:
        raise ValueError("logreg_grad: y needs one label per row and w one weight per column")
    p = _cached_plan("LOGREG_GRAD", (B, n // B, C), "f32", strategy, x.device, stream)
    return p.execute([x, y, w], out if out is not None else p.new_out(), stream)
