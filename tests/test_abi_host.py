"""CPU tests of the product library: it loads, exports every symbol that
include/graphreduce.h declares, and its host logic (Shard Creator + Graph
Layout Engine, §4.2) is correct. No compute
call needs a GPU here."""
import os
import re

import numpy as np
import pytest

import grgen
import paper_conf_sc_senguptasas15_b200 as gr

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    src = open(os.path.join(ROOT, "include", "graphreduce.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:gr_status|void|const char \*)\s*(gr_\w+)\s*\(", src, flags=re.M)))


def test_library_exports_every_header_symbol():
    L = gr.lib()
    names = header_functions()
    assert len(names) >= 15
    for name in names:
        assert hasattr(L, name), name
    assert set(names) == set(gr.EXPORTS)


def test_no_gpu_fails_cleanly():
    import torch

    if torch.cuda.is_available():
        pytest.skip("GPU present")
    src = np.array([0, 1], np.uint32)
    with pytest.raises(gr.GrError) as ei:
        gr.gr_graph_load(2, src, src[::-1].copy())
    assert ei.value.status == gr.GR_ECUDA


def test_program_compile_argument_errors():
    """gr_program_compile rejects bad arguments before doing
    any work, and without a GPU fails with a status instead of crashing."""
    import torch

    for name in ("", "1abc", "bad name", "a;b"):
        with pytest.raises(gr.GrError) as ei:
            gr.gr_program_compile("struct X {};", name)
        assert ei.value.status == gr.GR_EINVAL
    if not torch.cuda.is_available():
        with pytest.raises(gr.GrError) as ei:
            gr.gr_program_compile("struct X {};", "X")
        assert ei.value.status in (gr.GR_ECUDA, gr.GR_EUNSUPPORTED)


@pytest.mark.parametrize("P_target", [1 << 26, 5000, 700])
def test_host_layout_invariants(P_target):
    g = grgen.rmat(12, 16, seed=21)
    w = grgen.weights(g.m, 1, 64, seed=3)
    H = gr.HostLayout(g.n, g.src, g.dst, w, shard_edges=P_target)
    # intervals partition V
    b = H.bounds.astype(np.int64)
    assert b[0] == 0 and b[-1] == g.n and np.all(np.diff(b) >= 0)
    # CSC: each edge exactly once, segments sorted by (src, w)
    indeg = np.bincount(g.dst, minlength=g.n)
    np.testing.assert_array_equal(np.diff(H.in_off.astype(np.int64)), indeg)
    dst_of = np.repeat(np.arange(g.n, dtype=np.uint64), indeg)
    key_layout = np.sort((dst_of << 40) | (H.in_src.astype(np.uint64) << 8) | H.in_w.astype(np.uint64))
    key_input = np.sort((g.dst.astype(np.uint64) << 40) | (g.src.astype(np.uint64) << 8) | w.astype(np.uint64))
    np.testing.assert_array_equal(key_layout, key_input)
    layout_keys = (dst_of << 40) | (H.in_src.astype(np.uint64) << 8) | H.in_w.astype(np.uint64)
    assert np.all(np.diff(layout_keys.astype(np.float64)) >= 0) or np.all(layout_keys[1:] >= layout_keys[:-1])
    # CSR: each edge exactly once, sorted by (src, dst, w)
    outdeg = np.bincount(g.src, minlength=g.n)
    np.testing.assert_array_equal(np.diff(H.out_off.astype(np.int64)), outdeg)
    src_of = np.repeat(np.arange(g.n, dtype=np.uint64), outdeg)
    k2 = (src_of << 40) | (H.out_dst.astype(np.uint64) << 8) | H.out_w.astype(np.uint64)
    assert np.all(k2[1:] >= k2[:-1])
    np.testing.assert_array_equal(
        np.sort(k2), np.sort((g.src.astype(np.uint64) << 40) | (g.dst.astype(np.uint64) << 8) | w.astype(np.uint64)))
    # balance on in+out degree (L208): every shard <= ideal + max vertex weight
    wt = indeg + outdeg
    P = len(b) - 1
    per = np.array([wt[b[i]:b[i + 1]].sum() for i in range(P)])
    assert per.sum() == 2 * g.m
    assert per.max() <= 2 * g.m / P + wt.max()


def test_host_layout_deterministic_and_csr_input():
    g = grgen.rmat(10, 8, seed=5)
    H1 = gr.HostLayout(g.n, g.src, g.dst, host_threads=1)
    H8 = gr.HostLayout(g.n, g.src, g.dst, host_threads=8)
    np.testing.assert_array_equal(H1.in_src, H8.in_src)
    np.testing.assert_array_equal(H1.out_dst, H8.out_dst)
    # CSR input gives the same layout as COO input
    order = np.lexsort((g.dst, g.src))
    ro = np.zeros(g.n + 1, np.uint64)
    ro[1:] = np.cumsum(np.bincount(g.src, minlength=g.n))
    L = gr.lib()
    e, keep = gr._edges(g.n, row_offsets=ro, col_idx=g.dst[order])
    assert e.fmt == gr.GR_FMT_CSR
    H2 = gr.HostLayout.__new__(gr.HostLayout)
    import ctypes

    o, _ = gr._load_opts()
    h = ctypes.c_void_p()
    gr._check(L.gr_host_build(ctypes.byref(e), ctypes.byref(o), ctypes.byref(h)))
    try:
        H2.__dict__.update(gr.HostLayout._copy(L, h, g.n, False))
    finally:
        L.gr_host_free(h)
    np.testing.assert_array_equal(H1.in_src, H2.in_src)
    np.testing.assert_array_equal(H1.in_off, H2.in_off)


def test_host_build_rejects_bad_input():
    s = np.array([0, 9], np.uint32)
    with pytest.raises(gr.GrError) as ei:
        gr.HostLayout(4, s, s)
    assert ei.value.status == gr.GR_EINVAL
    with pytest.raises(gr.GrError):
        gr.HostLayout(4, np.array([0], np.uint32), np.array([1], np.uint32), np.array([300], np.uint32))


def test_plan_intervals():
    rng = np.random.default_rng(1)
    wts = rng.integers(0, 50, 1000)
    wts[17] = 10_000  # hub heavier than a shard
    pre = np.concatenate([[0], np.cumsum(wts)]).astype(np.uint64)
    for P in (1, 2, 7, 64, 2000):
        b = gr.gr_plan_intervals(pre, P).astype(np.int64)
        assert b[0] == 0 and b[-1] == 1000 and np.all(np.diff(b) >= 0)
        per = np.array([wts[b[i]:b[i + 1]].sum() for i in range(P)])
        assert per.max() <= wts.sum() / P + wts.max()


def test_multirank_owner_ranges_partition_edges():
    g = grgen.rmat(11, 8, seed=2)
    parts = [gr.HostLayout(g.n, g.src, g.dst, world=3, rank=r) for r in range(3)]
    lo = [int(p.bounds[0]) for p in parts]
    hi = [int(p.bounds[-1]) for p in parts]
    assert lo[0] == 0 and hi[-1] == g.n and lo[1] == hi[0] and lo[2] == hi[1]
    total_in = sum(len(p.in_src) for p in parts)
    assert total_in == g.m
    for r, p in enumerate(parts):
        # activation CSR holds exactly the edges whose destination is owned
        assert np.all((p.out_dst >= lo[r]) & (p.out_dst < hi[r]))
        owned = (g.dst >= lo[r]) & (g.dst < hi[r])
        assert len(p.out_dst) == owned.sum()


def test_graph_file_validation(tmp_path):
    """gr_graph_load_file parses the canonical file before touching the device:
    malformed files are GR_EINVAL; well-formed ones reach the device stage
    (GR_ECUDA here, without a GPU)."""
    import torch

    g = grgen.rmat(8, 4, seed=1)
    w = grgen.weights(g.m, 1, 64, seed=1)
    good = tmp_path / "g.bin"
    gr.write_graph_file(good, g.n, g.src, g.dst, w)
    raw = good.read_bytes()
    assert len(raw) == 32 + 12 * g.m and raw[:8] == b"GRGRAPH1"
    hdr = np.frombuffer(raw[8:24], np.uint64)
    assert hdr[0] == g.n and hdr[1] == g.m
    np.testing.assert_array_equal(np.frombuffer(raw[32:32 + 4 * g.m], np.uint32), g.src)
    np.testing.assert_array_equal(np.frombuffer(raw[32 + 8 * g.m:], np.uint32), w)
    bad = {
        "magic": b"XXGRAPH1" + raw[8:],
        "truncated": raw[:-4],
        "extra": raw + b"\0\0\0\0",
        "fmt": raw[:24] + np.array([7, 1], np.uint32).tobytes() + raw[32:],
        "flags": raw[:24] + np.array([0, 6], np.uint32).tobytes() + raw[32:],
        "tiny": raw[:16],
    }
    for name, data in bad.items():
        p = tmp_path / f"bad_{name}.bin"
        p.write_bytes(data)
        with pytest.raises(gr.GrError) as ei:
            gr.gr_graph_load_file(p)
        assert ei.value.status == gr.GR_EINVAL, name
    with pytest.raises(gr.GrError) as ei:
        gr.gr_graph_load_file(tmp_path / "missing.bin")
    assert ei.value.status == gr.GR_EINVAL
    # CSR form: header + row offsets + col idx
    order = np.lexsort((g.dst, g.src))
    ro = np.zeros(g.n + 1, np.uint64)
    ro[1:] = np.cumsum(np.bincount(g.src, minlength=g.n))
    csr = tmp_path / "csr.bin"
    gr.write_graph_file(csr, g.n, row_offsets=ro, col_idx=g.dst[order])
    assert csr.stat().st_size == 32 + 8 * (g.n + 1) + 4 * g.m
    if not torch.cuda.is_available():
        for p in (good, csr):
            with pytest.raises(gr.GrError) as ei:
                gr.gr_graph_load_file(p)
            assert ei.value.status == gr.GR_ECUDA


def _sorted_halves(g):
    n = g.n
    oi = np.lexsort((g.src, g.dst))
    in_off = np.zeros(n + 1, np.uint64)
    in_off[1:] = np.cumsum(np.bincount(g.dst, minlength=n))
    oo = np.lexsort((g.dst, g.src))
    out_off = np.zeros(n + 1, np.uint64)
    out_off[1:] = np.cumsum(np.bincount(g.src, minlength=n))
    return in_off, g.src[oi], out_off, g.dst[oo]


@pytest.mark.parametrize("shard_edges", [0, 3000])
def test_sorted_input_layout_equals_coo_layout(shard_edges):
    """GR_FMT_SORTED (the cfg5-at-scale input: an already-sorted in-CSC + out-CSR)
    gives the host builder's layout of the same edge multiset exactly."""
    g = grgen.rmat(12, 16, seed=23)
    a = gr.HostLayout(g.n, g.src, g.dst, shard_edges=shard_edges)
    b = gr.HostLayout.from_sorted(g.n, g.m, *_sorted_halves(g), shard_edges=shard_edges)
    for k in ("bounds", "in_off", "in_src", "out_off", "out_dst"):
        np.testing.assert_array_equal(getattr(a, k), getattr(b, k), err_msg=k)


def test_sorted_input_is_validated():
    g = grgen.rmat(8, 8, seed=24)
    in_off, in_src, out_off, out_dst = _sorted_halves(g)
    bad = in_src.copy()
    bad[5] = g.n  # id out of range
    with pytest.raises(gr.GrError) as ei:
        gr.HostLayout.from_sorted(g.n, g.m, in_off, bad, out_off, out_dst)
    assert ei.value.status == gr.GR_EINVAL
    # a row whose first two sources differ, swapped into descending order
    starts = in_off[:-1].astype(np.int64)
    two = (np.diff(in_off.astype(np.int64)) >= 2)
    cand = [int(b) for b in starts[two] if in_src[b] != in_src[b + 1]]
    b0 = cand[0]
    uns = in_src.copy()
    uns[b0], uns[b0 + 1] = in_src[b0 + 1], in_src[b0]
    with pytest.raises(gr.GrError) as ei:
        gr.HostLayout.from_sorted(g.n, g.m, in_off, uns, out_off, out_dst)
    assert ei.value.status == gr.GR_EINVAL
    short = out_off.copy()
    short[-1] -= 1  # does not span [0, m]
    with pytest.raises(gr.GrError) as ei:
        gr.HostLayout.from_sorted(g.n, g.m, in_off, in_src, short, out_dst)
    assert ei.value.status == gr.GR_EINVAL
