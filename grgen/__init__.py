"""Seeded synthetic graph inputs shared by the CUDA path and the oracle.

This module holds none of the GAS method's arithmetic: it only
produces canonical COO edge lists from counter-based random draws, shaped like
the paper's benchmark graphs (Table 1) as SURVEY.md §8(d)
specifies for BASELINE.json configs 1-5.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libgrgen.so")
_SRC = os.path.join(_HERE, "grgen.c")
_lib = None

THREADS = max(1, min(32, os.cpu_count() or 1))


def build(force: bool = False) -> str:
    """Compile libgrgen.so (plain C, OpenMP) if missing or stale."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < max(
        os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "grgen.h"))
    ):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(
            ["gcc", "-O3", "-fopenmp", "-fPIC", "-shared", "-o", tmp, _SRC, "-lm"], cwd=_HERE
        )
        os.replace(tmp, _SO)
    return _SO


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        u32p = ctypes.POINTER(ctypes.c_uint32)
        L.grgen_hash.restype = ctypes.c_uint64
        L.grgen_hash.argtypes = [ctypes.c_uint64] * 3
        L.grgen_rmat.restype = ctypes.c_int
        L.grgen_rmat.argtypes = [ctypes.c_uint32, ctypes.c_uint64, ctypes.c_double, ctypes.c_double,
                                 ctypes.c_double, ctypes.c_uint64, u32p, u32p, ctypes.c_int]
        L.grgen_weights.restype = ctypes.c_int
        L.grgen_weights.argtypes = [ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint64,
                                    u32p, ctypes.c_int]
        L.grgen_grid.restype = ctypes.c_int64
        L.grgen_grid.argtypes = [ctypes.c_uint32, ctypes.c_uint32, ctypes.c_double, ctypes.c_uint32,
                                 ctypes.c_uint64, u32p, u32p, u32p, ctypes.c_uint64]
        L.grgen_web.restype = ctypes.c_int64
        L.grgen_web.argtypes = [ctypes.c_uint64, ctypes.c_double, ctypes.c_double, ctypes.c_uint32,
                                ctypes.c_double, ctypes.c_double, ctypes.c_uint32, ctypes.c_double,
                                ctypes.c_uint64, u32p, u32p, ctypes.c_uint64, ctypes.c_int]
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32))


class Graph(dict):
    """dict with keys n, src, dst, [w], name — attribute access for convenience."""

    __getattr__ = dict.__getitem__

    @property
    def m(self) -> int:
        return int(self["src"].shape[0])


def rmat(scale: int, edgefactor: int = 16, seed: int = 1, a: float = 0.57, b: float = 0.19,
         c: float = 0.19, m: int | None = None) -> Graph:
    """R-MAT (Graph500 kron parameters), no noise, no permutation (vertex 0 is the hub)."""
    m = int(edgefactor) << scale if m is None else int(m)
    src = np.empty(m, np.uint32)
    dst = np.empty(m, np.uint32)
    rc = lib().grgen_rmat(scale, m, a, b, c, seed, _p(src), _p(dst), THREADS)
    if rc != 0:
        raise ValueError(f"grgen_rmat rc={rc}")
    return Graph(n=1 << scale, src=src, dst=dst, name=f"rmat{scale}_ef{edgefactor}_s{seed}")


_SO_GPU = os.path.join(_HERE, "libgrgen_gpu.so")
_SRC_GPU = os.path.join(_HERE, "grgen_gpu.cu")
_lib_gpu = None


def build_gpu(force: bool = False) -> str:
    """Compile libgrgen_gpu.so (nvcc, sm_100a): the GPU generator of the sorted R-MAT layout."""
    if force or not os.path.exists(_SO_GPU) or os.path.getmtime(_SO_GPU) < os.path.getmtime(_SRC_GPU):
        tmp = _SO_GPU + f".tmp{os.getpid()}"
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3",
                               "-Xcompiler", "-fPIC", "-shared", "-o", tmp, _SRC_GPU], cwd=_HERE)
        os.replace(tmp, _SO_GPU)
    return _SO_GPU


def rmat_sorted_gpu(scale: int, edgefactor: int = 16, seed: int = 1, by_src: bool = False, device: int = 0,
                    a: float = 0.57, b: float = 0.19, c: float = 0.19, other_degrees: bool = True,
                    budget_bytes: int = 0, adj: np.ndarray | None = None):
    """grgen.rmat(scale, edgefactor, seed)'s edge multiset as a sorted adjacency, generated on
    a GPU without materialising the COO (cfg5 at scale): by_src=False gives the in-CSC
    (offsets by destination, sources sorted), True the out-CSR. Returns (off, adj, other_deg)."""
    global _lib_gpu
    if _lib_gpu is None:
        build_gpu()
        L = ctypes.CDLL(_SO_GPU)
        L.grgen_rmat_sorted_gpu.restype = ctypes.c_int
        L.grgen_rmat_sorted_gpu.argtypes = [ctypes.c_uint32, ctypes.c_uint64, ctypes.c_double, ctypes.c_double,
                                            ctypes.c_double, ctypes.c_uint64, ctypes.c_int, ctypes.c_int,
                                            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64]
        _lib_gpu = L
    n = 1 << scale
    m = int(edgefactor) << scale
    off = np.empty(n + 1, np.uint64)
    if adj is None:
        adj = np.empty(m + 4, np.uint32)
    deg = np.empty(n, np.uint32) if other_degrees else None
    rc = _lib_gpu.grgen_rmat_sorted_gpu(scale, m, a, b, c, seed, 1 if by_src else 0, device, off.ctypes.data,
                                        adj.ctypes.data, deg.ctypes.data if deg is not None else None,
                                        budget_bytes)
    if rc != 0:
        raise ValueError(f"grgen_rmat_sorted_gpu rc={rc}")
    return off, adj, deg


def weights(m: int, lo: int = 1, hi: int = 64, seed: int = 1) -> np.ndarray:
    w = np.empty(m, np.uint32)
    rc = lib().grgen_weights(m, lo, hi, seed, _p(w), THREADS)
    if rc != 0:
        raise ValueError(f"grgen_weights rc={rc}")
    return w


def grid_road(W: int, H: int, p: float = 0.58, wmax: int = 64, seed: int = 3) -> Graph:
    """Road-like lattice: p-kept lattice edges + seeded connectivity repair, symmetric weights."""
    L = lib()
    m = L.grgen_grid(W, H, p, wmax, seed, None, None, None, 0)
    if m < 0:
        raise ValueError(f"grgen_grid rc={m}")
    src = np.empty(m, np.uint32)
    dst = np.empty(m, np.uint32)
    w = np.empty(m, np.uint32)
    m2 = L.grgen_grid(W, H, p, wmax, seed, _p(src), _p(dst), _p(w), m)
    if m2 != m:
        raise ValueError(f"grgen_grid rc={m2}")
    return Graph(n=W * H, src=src, dst=dst, w=w, name=f"grid{W}x{H}_s{seed}")


def heat_grid(W: int, H: int, p: float = 0.58, wmax: int = 60, seed: int = 6) -> Graph:
    """Heat-simulation input (§2.1): the road-like lattice with symmetric
    conductances w in [1, wmax] plus one self-loop per vertex whose weight makes every
    vertex's out-weights satisfy sum (w + 1) = 256 (the heat a vertex keeps). Needs
    4 * (wmax + 1) <= 255."""
    assert 4 * (wmax + 1) <= 255
    g = grid_road(W, H, p=p, wmax=wmax, seed=seed)
    out = np.bincount(g.src, weights=g.w.astype(np.float64) + 1.0, minlength=g.n).astype(np.int64)
    self_w = (255 - out).astype(np.uint32)
    v = np.arange(g.n, dtype=np.uint32)
    return Graph(n=g.n, src=np.concatenate([g.src, v]), dst=np.concatenate([g.dst, v]),
                 w=np.concatenate([g.w, self_w]), name=f"heat{W}x{H}_s{seed}")


WEB_DEFAULTS = dict(xmin=2.8, zexp=2.5, dmax=1 << 20, p_local=0.75, geo_p=1.0 / 64,
                    local_cap=4096, rank_exp=0.8)


def web(n: int, seed: int = 4, **kw) -> Graph:
    """Web-like power law (uk-2002 shape), symmetrized, self-loops dropped."""
    prm = dict(WEB_DEFAULTS)
    prm.update(kw)
    args = (n, prm["xmin"], prm["zexp"], prm["dmax"], prm["p_local"], prm["geo_p"],
            prm["local_cap"], prm["rank_exp"], seed)
    L = lib()
    m = L.grgen_web(*args, None, None, 0, THREADS)
    if m < 0:
        raise ValueError(f"grgen_web rc={m}")
    src = np.empty(m, np.uint32)
    dst = np.empty(m, np.uint32)
    m2 = L.grgen_web(*args, _p(src), _p(dst), m, THREADS)
    if m2 != m:
        raise ValueError(f"grgen_web rc={m2}")
    return Graph(n=n, src=src, dst=dst, name=f"web{n}_s{seed}")


# --------------------------------------------------------------------------
# BASELINE.json configs; `reduced` gives the parity-test
# sizes with the same shape.
# --------------------------------------------------------------------------
def config(i: int, reduced: bool = False) -> tuple[Graph, dict]:
    """Return (graph, run) for BASELINE.json configs[i-1]."""
    if i == 1:
        g = rmat(12 if reduced else 16, edgefactor=38, seed=1)
        return g, dict(algo="bfs", source=0)
    if i == 2:
        g = rmat(16 if reduced else 22, edgefactor=16, seed=2)
        return g, dict(algo="pagerank", max_iters=30, damping=0.85)
    if i == 3:
        W = 300 if reduced else 4894
        g = grid_road(W, W, p=0.58, wmax=64, seed=3)
        return g, dict(algo="sssp", source=0)
    if i == 4:
        g = web(200_000 if reduced else 18_520_486, seed=4)
        return g, dict(algo="cc")
    if i == 5:
        # cfg5 shape (R-MAT ef16); scale chosen by the caller's memory budget
        g = rmat(18 if reduced else 31, edgefactor=16, seed=5)
        return g, dict(algo="pagerank", max_iters=30, damping=0.85)
    raise ValueError(i)
