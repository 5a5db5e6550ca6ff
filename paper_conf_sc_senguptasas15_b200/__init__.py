"""GraphReduce on B200 — thin Python binding of include/graphreduce.h.

Argument marshalling only: every step of the GAS superstep runs in the CUDA
library ``libgraphreduce.so`` (sm_100a). There is no CPU fallback; if the
library cannot be loaded every call raises.

Functions carry the C names (``gr_graph_load``, ``gr_run``,
``gr_fetch_vertex_values``, ...). ``GraphReduce`` is a small convenience
wrapper around a ``gr_graph`` handle.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from . import _build

_SO = _build.SO
_lib = None

GR_OK, GR_EINVAL, GR_ENOMEM, GR_ECUDA, GR_ENCCL, GR_EUNSUPPORTED, GR_ESTATE = range(7)
STATUS_NAMES = ["GR_OK", "GR_EINVAL", "GR_ENOMEM", "GR_ECUDA", "GR_ENCCL", "GR_EUNSUPPORTED", "GR_ESTATE"]
GR_FMT_COO, GR_FMT_CSR, GR_FMT_SORTED = 0, 1, 2
ALGOS = {"bfs": 0, "sssp": 1, "pagerank": 2, "cc": 3, "custom": 4, "pagerank_delta": 5}
FLOAT_ALGOS = ("pagerank", "pagerank_delta")
TRANSPORTS = {"nccl": 0, "shm": 1}
MODES = {"auto": 0, "resident": 1, "streamed": 2}
LOOPS = {"auto": 0, "host": 1, "device": 2, "persistent": 3}
BUILDS = {"auto": 0, "host": 1, "device": 2}
DIRECTIONS = {"auto": 0, "push": 1, "pull": 2, "fused": 3}
INF = 0xFFFFFFFF

EXPORTS = [
    "gr_get_unique_id", "gr_graph_load", "gr_graph_load_file", "gr_run", "gr_fetch_vertex_values", "gr_fetch_frontier_trace",
    "gr_graph_info_get", "gr_shard_info", "gr_graph_free", "gr_last_error", "gr_plan_intervals",
    "gr_host_build", "gr_host_csc", "gr_host_csr", "gr_host_shards", "gr_host_free", "gr_program_compile",
    "gr_fetch_frontier_trace_detail",
]


class GrError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS_NAMES[status] if 0 <= status < 7 else status}: {msg}")
        self.status = status


class gr_edges(ctypes.Structure):
    _fields_ = [("fmt", ctypes.c_int32), ("num_vertices", ctypes.c_uint64), ("num_edges", ctypes.c_uint64),
                ("src", ctypes.c_void_p), ("dst", ctypes.c_void_p), ("row_offsets", ctypes.c_void_p),
                ("col_idx", ctypes.c_void_p), ("weights", ctypes.c_void_p), ("in_offsets", ctypes.c_void_p),
                ("in_idx", ctypes.c_void_p), ("out_degree", ctypes.c_void_p)]


class gr_load_opts(ctypes.Structure):
    _fields_ = [("shard_edges", ctypes.c_uint64), ("device_budget_bytes", ctypes.c_uint64),
                ("mode", ctypes.c_int32), ("device", ctypes.c_int32), ("rank", ctypes.c_int32),
                ("world", ctypes.c_int32), ("nccl_unique_id", ctypes.c_void_p), ("host_threads", ctypes.c_int32),
                ("sim_ranks", ctypes.c_int32), ("build", ctypes.c_int32),
                ("transport", ctypes.c_int32), ("borrow", ctypes.c_int32)]


class gr_run_opts(ctypes.Structure):
    _fields_ = [("algo", ctypes.c_int32), ("source", ctypes.c_uint32), ("max_iters", ctypes.c_uint32),
                ("damping", ctypes.c_float), ("custom_id", ctypes.c_int32), ("loop", ctypes.c_int32),
                ("stream", ctypes.c_void_p), ("profile", ctypes.c_int32), ("direction", ctypes.c_int32),
                ("pull_div", ctypes.c_uint32), ("tolerance", ctypes.c_float), ("zero_copy", ctypes.c_int32),
                ("trace_detail", ctypes.c_int32)]


class gr_run_stats(ctypes.Structure):
    _fields_ = [("iterations", ctypes.c_uint32), ("seconds", ctypes.c_double),
                ("edges_gathered", ctypes.c_uint64), ("edges_scattered", ctypes.c_uint64),
                ("bytes_h2d", ctypes.c_uint64), ("bytes_nvlink", ctypes.c_uint64),
                ("bytes_hbm_model", ctypes.c_uint64), ("kernel_launches", ctypes.c_uint64),
                ("kernel_ms", ctypes.c_double * 4), ("pull_supersteps", ctypes.c_uint32),
                ("zero_copy_phases", ctypes.c_uint32), ("bytes_h2d_zero_copy", ctypes.c_uint64)]

    def as_dict(self):
        d = {k: getattr(self, k) for k, _ in self._fields_ if k != "kernel_ms"}
        d["kernel_ms"] = list(self.kernel_ms)
        return d


class gr_graph_info(ctypes.Structure):
    _fields_ = [("num_vertices", ctypes.c_uint64), ("num_edges", ctypes.c_uint64), ("num_shards", ctypes.c_uint32),
                ("mode", ctypes.c_int32), ("rank", ctypes.c_int32), ("world", ctypes.c_int32),
                ("sim_ranks", ctypes.c_int32), ("own_lo", ctypes.c_uint64), ("own_hi", ctypes.c_uint64),
                ("device_bytes", ctypes.c_uint64), ("pinned_bytes", ctypes.c_uint64),
                ("offsets_64bit", ctypes.c_int32), ("has_weights", ctypes.c_int32),
                ("built_on_device", ctypes.c_int32), ("reserved", ctypes.c_int32)]


class gr_shard_desc(ctypes.Structure):
    _fields_ = [("v_lo", ctypes.c_uint64), ("v_hi", ctypes.c_uint64), ("in_begin", ctypes.c_uint64),
                ("in_end", ctypes.c_uint64), ("out_begin", ctypes.c_uint64), ("out_end", ctypes.c_uint64)]


def lib():
    """Load libgraphreduce.so (built in-tree for sm_100a); raise if unavailable."""
    global _lib
    if _lib is not None:
        return _lib
    so = os.environ.get("GR_LIB")  # experiments: an alternative in-tree build of the same library
    if not so:
        so = _SO
        if not os.path.exists(_SO) or _build.stale():
            if not os.path.exists(_build.NVCC):
                raise GrError(GR_EUNSUPPORTED, f"{_SO} is missing and nvcc is unavailable to build it")
            _build.build()
    L = ctypes.CDLL(so)
    vp, u64, u32, i32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int32
    u64p = ctypes.POINTER(ctypes.c_uint64)
    sig = {
        "gr_get_unique_id": (i32, [vp]),
        "gr_graph_load": (i32, [ctypes.POINTER(gr_edges), ctypes.POINTER(gr_load_opts), ctypes.POINTER(vp)]),
        "gr_graph_load_file": (i32, [ctypes.c_char_p, ctypes.POINTER(gr_load_opts), ctypes.POINTER(vp)]),
        "gr_run": (i32, [vp, ctypes.POINTER(gr_run_opts), ctypes.POINTER(gr_run_stats)]),
        "gr_fetch_vertex_values": (i32, [vp, vp, u64]),
        "gr_fetch_frontier_trace": (i32, [vp, u64p, u64, u64p]),
        "gr_fetch_frontier_trace_detail": (i32, [vp, u64p, u64, u64p]),
        "gr_graph_info_get": (i32, [vp, ctypes.POINTER(gr_graph_info)]),
        "gr_program_compile": (i32, [ctypes.c_char_p, ctypes.c_char_p, ctypes.POINTER(i32)]),
        "gr_shard_info": (i32, [vp, u32, ctypes.POINTER(gr_shard_desc)]),
        "gr_graph_free": (None, [vp]),
        "gr_last_error": (ctypes.c_char_p, []),
        "gr_plan_intervals": (i32, [u64, u64p, u32, u64p]),
        "gr_host_build": (i32, [ctypes.POINTER(gr_edges), ctypes.POINTER(gr_load_opts), ctypes.POINTER(vp)]),
        "gr_host_csc": (i32, [vp, ctypes.POINTER(u64p), ctypes.POINTER(ctypes.POINTER(u32)),
                              ctypes.POINTER(ctypes.POINTER(ctypes.c_uint8))]),
        "gr_host_csr": (i32, [vp, ctypes.POINTER(u64p), ctypes.POINTER(ctypes.POINTER(u32)),
                              ctypes.POINTER(ctypes.POINTER(ctypes.c_uint8))]),
        "gr_host_shards": (i32, [vp, ctypes.POINTER(u32), ctypes.POINTER(u64p)]),
        "gr_host_free": (None, [vp]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return L


def _check(status: int):
    if status != GR_OK:
        raise GrError(status, lib().gr_last_error().decode(errors="replace"))


def _u32(a):
    return None if a is None else np.ascontiguousarray(a, dtype=np.uint32)


def _edges(n, src=None, dst=None, weights=None, row_offsets=None, col_idx=None):
    keep = []
    e = gr_edges()
    e.num_vertices = int(n)
    if row_offsets is not None:
        ro = np.ascontiguousarray(row_offsets, dtype=np.uint64)
        ci = _u32(col_idx)
        keep += [ro, ci]
        e.fmt, e.num_edges = GR_FMT_CSR, int(ci.shape[0])
        e.row_offsets, e.col_idx = ro.ctypes.data, ci.ctypes.data
    else:
        s, d = _u32(src), _u32(dst)
        keep += [s, d]
        e.fmt, e.num_edges = GR_FMT_COO, int(s.shape[0])
        e.src, e.dst = s.ctypes.data, d.ctypes.data
    if weights is not None:
        w = _u32(weights)
        keep.append(w)
        e.weights = w.ctypes.data
    return e, keep


def _load_opts(shard_edges=0, device_budget_bytes=0, mode="auto", device=0, rank=0, world=1,
               nccl_unique_id=None, host_threads=0, sim_ranks=0, build="auto", transport="nccl", borrow=False):
    o = gr_load_opts()
    o.shard_edges, o.device_budget_bytes = int(shard_edges), int(device_budget_bytes)
    o.mode = MODES[mode] if isinstance(mode, str) else int(mode)
    o.device, o.rank, o.world = int(device), int(rank), int(world)
    uid = None
    if nccl_unique_id is not None:
        uid = ctypes.create_string_buffer(bytes(nccl_unique_id), 128)
        o.nccl_unique_id = ctypes.cast(uid, ctypes.c_void_p)
    o.host_threads, o.sim_ranks = int(host_threads), int(sim_ranks)
    o.build = BUILDS[build] if isinstance(build, str) else int(build)
    o.transport = TRANSPORTS[transport] if isinstance(transport, str) else int(transport)
    o.borrow = 1 if borrow else 0
    return o, uid


# ----------------------------------------------------------------- C names
def gr_get_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(lib().gr_get_unique_id(buf))
    return buf.raw


def gr_graph_load(n, src=None, dst=None, weights=None, row_offsets=None, col_idx=None, **opts):
    """Partition + lay out + place the graph; returns an opaque handle (c_void_p)."""
    e, keep = _edges(n, src, dst, weights, row_offsets, col_idx)
    o, uid = _load_opts(**opts)
    h = ctypes.c_void_p()
    _check(lib().gr_graph_load(ctypes.byref(e), ctypes.byref(o), ctypes.byref(h)))
    del keep, uid
    return h


GRAPH_FILE_MAGIC = b"GRGRAPH1"


def write_graph_file(path, n, src=None, dst=None, weights=None, row_offsets=None, col_idx=None):
    """Write the canonical graph file read by gr_graph_load_file (layout in
    include/graphreduce.h): 32-byte header, then COO src/dst (or CSR
    row_offsets/col_idx), then optional uint32 weights."""
    if row_offsets is not None:
        ro = np.ascontiguousarray(row_offsets, dtype=np.uint64)
        ci = np.ascontiguousarray(col_idx, dtype=np.uint32)
        fmt, m, arrays = GR_FMT_CSR, ci.shape[0], [ro, ci]
    else:
        s_, d_ = np.ascontiguousarray(src, dtype=np.uint32), np.ascontiguousarray(dst, dtype=np.uint32)
        if s_.shape != d_.shape:
            raise ValueError("src and dst lengths differ")
        fmt, m, arrays = GR_FMT_COO, s_.shape[0], [s_, d_]
    flags = 0
    if weights is not None:
        w = np.ascontiguousarray(weights, dtype=np.uint32)
        if w.shape[0] != m:
            raise ValueError("weights length != number of edges")
        arrays.append(w)
        flags = 1
    hdr = GRAPH_FILE_MAGIC + np.array([n, m], np.uint64).tobytes() + np.array([fmt, flags], np.uint32).tobytes()
    with open(path, "wb") as f:
        f.write(hdr)
        for a in arrays:
            a.tofile(f)


def gr_graph_load_sorted(n, m, in_offsets=None, in_idx=None, row_offsets=None, col_idx=None, out_degree=None,
                         **opts):
    """GR_FMT_SORTED: load the already-sorted layout (in-CSC and/or out-CSR). With
    borrow=True the adjacency arrays are used in place: they must hold m + 4
    entries and outlive the handle (GraphReduce.from_sorted keeps them)."""
    e = gr_edges()
    e.fmt, e.num_vertices, e.num_edges = GR_FMT_SORTED, int(n), int(m)
    keep = []
    for name, arr, dt in (("in_offsets", in_offsets, np.uint64), ("in_idx", in_idx, np.uint32),
                          ("row_offsets", row_offsets, np.uint64), ("col_idx", col_idx, np.uint32),
                          ("out_degree", out_degree, np.uint32)):
        if arr is None:
            continue
        if arr.dtype != dt or not arr.flags["C_CONTIGUOUS"]:
            if opts.get("borrow"):
                raise ValueError(f"{name}: borrowed arrays must be C-contiguous {np.dtype(dt).name}")
            arr = np.ascontiguousarray(arr, dtype=dt)
        keep.append(arr)
        setattr(e, name, arr.ctypes.data)
    o, uid = _load_opts(**opts)
    h = ctypes.c_void_p()
    _check(lib().gr_graph_load(ctypes.byref(e), ctypes.byref(o), ctypes.byref(h)))
    return h


def gr_graph_load_file(path, **opts):
    """gr_graph_load from a canonical graph file (memory-mapped by the library)."""
    o, uid = _load_opts(**opts)
    h = ctypes.c_void_p()
    _check(lib().gr_graph_load_file(os.fsencode(path), ctypes.byref(o), ctypes.byref(h)))
    del uid
    return h


def gr_run(h, algo, source=0, max_iters=0, damping=0.85, custom_id=0, loop="auto", stream=None,
           profile=False, direction="auto", pull_div=0, zero_copy=0, tolerance=1e-4, trace_detail=False) -> dict:
    o = gr_run_opts()
    o.algo = ALGOS[algo] if isinstance(algo, str) else int(algo)
    o.source, o.max_iters, o.damping, o.custom_id = int(source), int(max_iters), float(damping), int(custom_id)
    o.loop = LOOPS[loop] if isinstance(loop, str) else int(loop)
    o.stream = stream
    o.profile = 1 if profile else 0
    o.direction = DIRECTIONS[direction] if isinstance(direction, str) else int(direction)
    o.pull_div = int(pull_div)
    o.zero_copy = int(zero_copy)
    o.tolerance = float(tolerance)
    o.trace_detail = 1 if trace_detail else 0
    st = gr_run_stats()
    _check(lib().gr_run(h, ctypes.byref(o), ctypes.byref(st)))
    return st.as_dict()


def gr_program_compile(source: str, struct_name: str) -> int:
    """Compile a GAS program at run time (NVRTC) and return its custom_id
    (include/graphreduce.h gr_program_compile)."""
    cid = ctypes.c_int32(0)
    _check(lib().gr_program_compile(source.encode(), struct_name.encode(), ctypes.byref(cid)))
    return int(cid.value)


def gr_graph_info_get(h) -> dict:
    i = gr_graph_info()
    _check(lib().gr_graph_info_get(h, ctypes.byref(i)))
    return {k: getattr(i, k) for k, _ in i._fields_}


def gr_fetch_vertex_values(h, out: np.ndarray | None = None, dtype=np.uint32) -> np.ndarray:
    n = gr_graph_info_get(h)["num_vertices"]
    if out is None:
        out = np.empty(n, dtype)
    _check(lib().gr_fetch_vertex_values(h, out.ctypes.data, out.nbytes))
    return out


def gr_fetch_frontier_trace(h, max_rows: int = 1 << 20) -> np.ndarray:
    buf = np.zeros((max_rows, 4), np.uint64)
    rows = ctypes.c_uint64(0)
    _check(lib().gr_fetch_frontier_trace(h, buf.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)), max_rows,
                                         ctypes.byref(rows)))
    return buf[: rows.value].copy()


def gr_fetch_frontier_trace_detail(h, max_rows: int = 1 << 20) -> np.ndarray:
    """(active_shards, S_t) per superstep of the last run (run with trace_detail=True)."""
    buf = np.zeros((max_rows, 2), np.uint64)
    rows = ctypes.c_uint64(0)
    _check(lib().gr_fetch_frontier_trace_detail(h, buf.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)), max_rows,
                                                ctypes.byref(rows)))
    return buf[: rows.value].copy()


def gr_shard_info(h, s: int) -> dict:
    d = gr_shard_desc()
    _check(lib().gr_shard_info(h, s, ctypes.byref(d)))
    return {k: getattr(d, k) for k, _ in d._fields_}


def gr_graph_free(h):
    if h:
        lib().gr_graph_free(h)


def gr_plan_intervals(weight_prefix, P: int) -> np.ndarray:
    wp = np.ascontiguousarray(weight_prefix, dtype=np.uint64)
    b = np.zeros(P + 1, np.uint64)
    u64p = ctypes.POINTER(ctypes.c_uint64)
    _check(lib().gr_plan_intervals(len(wp) - 1, wp.ctypes.data_as(u64p), P, b.ctypes.data_as(u64p)))
    return b


class HostLayout:
    """gr_host_build: the host-side sharded layout, copied out to numpy (CPU only)."""

    def __init__(self, n, src, dst, weights=None, **opts):
        e, keep = _edges(n, src, dst, weights)
        o, uid = _load_opts(**opts)
        h = ctypes.c_void_p()
        L = lib()
        _check(L.gr_host_build(ctypes.byref(e), ctypes.byref(o), ctypes.byref(h)))
        try:
            info = self._copy(L, h, int(n), weights is not None)
        finally:
            L.gr_host_free(h)
        self.__dict__.update(info)

    @classmethod
    def from_sorted(cls, n, m, in_offsets, in_idx, row_offsets, col_idx, **opts):
        """gr_host_build of a GR_FMT_SORTED input (both halves), copied out like __init__."""
        self = cls.__new__(cls)
        e = gr_edges()
        e.fmt, e.num_vertices, e.num_edges = GR_FMT_SORTED, int(n), int(m)
        keep = [np.ascontiguousarray(in_offsets, dtype=np.uint64), np.ascontiguousarray(in_idx, dtype=np.uint32),
                np.ascontiguousarray(row_offsets, dtype=np.uint64), np.ascontiguousarray(col_idx, dtype=np.uint32)]
        e.in_offsets, e.in_idx, e.row_offsets, e.col_idx = (a.ctypes.data for a in keep)
        o, uid = _load_opts(**opts)
        h = ctypes.c_void_p()
        L = lib()
        _check(L.gr_host_build(ctypes.byref(e), ctypes.byref(o), ctypes.byref(h)))
        try:
            info = self._copy(L, h, int(n), False)
        finally:
            L.gr_host_free(h)
        self.__dict__.update(info)
        return self

    @staticmethod
    def _copy(L, h, n, has_w):
        u64p, u32p, u8p = (ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_uint32),
                           ctypes.POINTER(ctypes.c_uint8))
        nshard = ctypes.c_uint32()
        bp = u64p()
        _check(L.gr_host_shards(h, ctypes.byref(nshard), ctypes.byref(bp)))
        bounds = np.ctypeslib.as_array(bp, (nshard.value + 1,)).copy()
        off, idx, w = u64p(), u32p(), u8p()
        _check(L.gr_host_csc(h, ctypes.byref(off), ctypes.byref(idx), ctypes.byref(w)))
        own_n = int(bounds[-1] - bounds[0])
        in_off = np.ctypeslib.as_array(off, (own_n + 1,)).copy()
        m_in = int(in_off[-1])
        in_src = np.ctypeslib.as_array(idx, (max(m_in, 1),))[:m_in].copy()
        in_w = np.ctypeslib.as_array(w, (max(m_in, 1),))[:m_in].copy() if has_w and m_in else None
        _check(L.gr_host_csr(h, ctypes.byref(off), ctypes.byref(idx), ctypes.byref(w)))
        out_off = np.ctypeslib.as_array(off, (n + 1,)).copy()
        out_dst = np.ctypeslib.as_array(idx, (max(m_in, 1),))[:m_in].copy()
        out_w = np.ctypeslib.as_array(w, (max(m_in, 1),))[:m_in].copy() if has_w and m_in else None
        return dict(bounds=bounds, in_off=in_off, in_src=in_src, in_w=in_w, out_off=out_off, out_dst=out_dst,
                    out_w=out_w)


class GraphReduce:
    """Convenience wrapper: load once, run many programs, fetch results."""

    def __init__(self, n, src=None, dst=None, weights=None, **opts):
        self.n = int(n)
        self.h = gr_graph_load(n, src, dst, weights, **opts)

    @classmethod
    def from_sorted(cls, n, m, **kw):
        """GR_FMT_SORTED load (gr_graph_load_sorted); borrowed arrays are kept alive here."""
        self = cls.__new__(cls)
        self._borrowed = [v for v in kw.values() if isinstance(v, np.ndarray)]
        self.h = gr_graph_load_sorted(n, m, **kw)
        self.n = int(n)
        return self

    @classmethod
    def from_file(cls, path, **opts):
        self = cls.__new__(cls)
        self.h = gr_graph_load_file(path, **opts)
        self.n = gr_graph_info_get(self.h)["num_vertices"]
        return self

    def run(self, algo, **kw) -> dict:
        return gr_run(self.h, algo, **kw)

    def values(self, algo=None):
        dt = np.float32 if algo in FLOAT_ALGOS else np.uint32
        return gr_fetch_vertex_values(self.h, dtype=dt)

    def trace(self):
        return gr_fetch_frontier_trace(self.h)

    def trace_detail(self):
        return gr_fetch_frontier_trace_detail(self.h)

    def info(self):
        return gr_graph_info_get(self.h)

    def close(self):
        if self.h:
            gr_graph_free(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
