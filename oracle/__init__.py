"""GAS oracle — TEST INFRASTRUCTURE ONLY.

A plain single-threaded C engine (oracle.c) that follows the paper's GAS
superstep step by step (§2.1, §4.4, §5.2, §5.3
L274-276, Fig. 6), PageRank in fp64. Only ``tests/``,
``__graft_entry__.smoke()`` and ``bench.py`` (cpu_baseline and ``--impl
reference``) may import this module. It shares no code with the CUDA path.

Pins: tests/test_oracle_pins.py (all four programs are pinned; no function is
"parity unpinned").
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.c")
_lib = None

ALGOS = {"bfs": 0, "sssp": 1, "pagerank": 2, "cc": 3, "widest": 4, "pagerank_delta": 5, "sssp_msg": 6, "heat": 7}
HEAT_H0 = 0x40000000
INF = 0xFFFFFFFF


def build(force: bool = False) -> str:
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < max(
        os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "oracle.h"))
    ):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fPIC", "-shared", "-o", tmp, _SRC], cwd=_HERE)
        os.replace(tmp, _SO)
    return _SO


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        u32p = ctypes.POINTER(ctypes.c_uint32)
        L.or_graph_build.restype = ctypes.c_void_p
        L.or_graph_build.argtypes = [ctypes.c_uint64, ctypes.c_uint64, u32p, u32p, u32p]
        L.or_graph_free.restype = None
        L.or_graph_free.argtypes = [ctypes.c_void_p]
        L.or_run.restype = ctypes.c_int64
        L.or_run.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_uint32, ctypes.c_uint32,
                             ctypes.c_double, ctypes.c_double, ctypes.c_void_p, ctypes.POINTER(ctypes.c_uint64),
                             ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint64)]
        L.or_run_detail.restype = ctypes.c_int64
        L.or_run_detail.argtypes = L.or_run.argtypes + [ctypes.POINTER(ctypes.c_uint64), ctypes.c_uint32,
                                                        ctypes.POINTER(ctypes.c_uint64)]
        _lib = L
    return _lib


def _u32(a):
    if a is None:
        return None
    a = np.ascontiguousarray(a, dtype=np.uint32)
    return a


class OracleGraph:
    """The oracle's own CSC/CSR built from a COO edge list."""

    def __init__(self, n: int, src, dst, w=None):
        self.n = int(n)
        self._src, self._dst, self._w = _u32(src), _u32(dst), _u32(w)
        self.m = int(self._src.shape[0])
        P = ctypes.POINTER(ctypes.c_uint32)
        h = lib().or_graph_build(
            self.n, self.m, self._src.ctypes.data_as(P), self._dst.ctypes.data_as(P),
            self._w.ctypes.data_as(P) if self._w is not None else None)
        if not h:
            raise ValueError("or_graph_build failed (bad ids or out of memory)")
        self._h = h

    def run(self, algo: str, source: int = 0, max_iters: int = 0, damping: float = 0.85,
            trace_cap: int = 1 << 20, tolerance: float = 1e-4):
        """Return (values, trace[rows,4], iterations). pagerank_delta values are
        float32 (the fp32 ranks); pagerank values are float64."""
        a = ALGOS[algo]
        if algo == "pagerank" and max_iters == 0:
            max_iters = 30
        vals = np.empty(self.n, np.float64 if algo == "pagerank" else np.uint32)
        tr = np.zeros((trace_cap, 4), np.uint64)
        rows = ctypes.c_uint64(0)
        it = lib().or_run(self._h, a, source, max_iters, damping, tolerance, vals.ctypes.data_as(ctypes.c_void_p),
                          tr.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)), trace_cap,
                          ctypes.byref(rows))
        if it < 0:
            raise ValueError(f"or_run failed rc={it}")
        if algo == "pagerank_delta":
            vals = vals.view(np.float32)
        return vals, tr[: min(rows.value, trace_cap)].copy(), int(it)

    def run_detail(self, algo: str, shard_bounds=None, source: int = 0, max_iters: int = 0,
                   damping: float = 0.85, trace_cap: int = 1 << 16, tolerance: float = 1e-4):
        """Like run(), plus detail[rows, 2] = (active_shards, S_t) per superstep."""
        a = ALGOS[algo]
        if algo == "pagerank" and max_iters == 0:
            max_iters = 30
        vals = np.empty(self.n, np.float64 if algo == "pagerank" else np.uint32)
        tr = np.zeros((trace_cap, 4), np.uint64)
        det = np.zeros((trace_cap, 2), np.uint64)
        rows = ctypes.c_uint64(0)
        P64 = ctypes.POINTER(ctypes.c_uint64)
        b = None if shard_bounds is None else np.ascontiguousarray(shard_bounds, dtype=np.uint64)
        nb = 0 if b is None else len(b) - 1
        it = lib().or_run_detail(self._h, a, source, max_iters, damping, tolerance,
                                 vals.ctypes.data_as(ctypes.c_void_p), tr.ctypes.data_as(P64), trace_cap,
                                 ctypes.byref(rows), None if b is None else b.ctypes.data_as(P64), nb,
                                 det.ctypes.data_as(P64))
        if it < 0:
            raise ValueError(f"or_run_detail failed rc={it}")
        r = min(rows.value, trace_cap)
        if algo == "pagerank_delta":
            vals = vals.view(np.float32)
        return vals, tr[:r].copy(), det[:r].copy(), int(it)

    def close(self):
        if getattr(self, "_h", None):
            lib().or_graph_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def run(n, src, dst, algo, w=None, **kw):
    g = OracleGraph(n, src, dst, w)
    try:
        return g.run(algo, **kw)
    finally:
        g.close()
