"""cfg5 at scale (BASELINE.json configs[4]; §3.2): the
R-MAT input generated on the GPU straight into the sorted layout (no COO ever
materialised) and loaded with GR_FMT_SORTED — one half alone when only one
direction fits host memory (PageRank: in-CSC, BFS: out-CSR), borrowed in
place. At test sizes: the generator's layout equals the CPU generator's edge
multiset sorted, and every load equals the oracle."""
import numpy as np
import pytest

import grgen
import oracle
import paper_conf_sc_senguptasas15_b200 as gr
from test_gpu_parity import check_pr

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("scale,seed", [(10, 5), (15, 5), (16, 7)])
def test_gpu_generator_equals_cpu_generator(scale, seed):
    g = grgen.rmat(scale, 16, seed=seed)
    n, m = g.n, g.m
    for by_src in (False, True):
        key, oth = (g.src, g.dst) if by_src else (g.dst, g.src)
        order = np.lexsort((oth, key))
        ref_off = np.zeros(n + 1, np.uint64)
        ref_off[1:] = np.cumsum(np.bincount(key, minlength=n))
        # a small device budget forces several key-range passes
        off, adj, deg = grgen.rmat_sorted_gpu(scale, 16, seed=seed, by_src=by_src, budget_bytes=24 << 20)
        np.testing.assert_array_equal(off, ref_off)
        np.testing.assert_array_equal(adj[:m], oth[order])
        np.testing.assert_array_equal(deg, np.bincount(oth, minlength=n).astype(np.uint32))


def _layouts(scale, seed):
    ci_off, ci, od = grgen.rmat_sorted_gpu(scale, 16, seed=seed, by_src=False)
    co_off, co, _ = grgen.rmat_sorted_gpu(scale, 16, seed=seed, by_src=True, other_degrees=False)
    return ci_off, ci, od, co_off, co


def test_sorted_load_both_halves_equals_oracle():
    scale, seed = 14, 5
    g = grgen.rmat(scale, 16, seed=seed)
    ci_off, ci, od, co_off, co = _layouts(scale, seed)
    og = oracle.OracleGraph(g.n, g.src, g.dst)
    for mode in ("resident", "streamed"):
        with gr.GraphReduce.from_sorted(g.n, g.m, in_offsets=ci_off, in_idx=ci, row_offsets=co_off, col_idx=co,
                                        mode=mode, shard_edges=1 << 16) as G:
            for algo in ("bfs", "cc", "pagerank", "pagerank_delta"):
                ref, rtr, rit = og.run(algo, source=0)
                st = G.run(algo, source=0)
                assert st["iterations"] == rit
                if algo == "pagerank":
                    check_pr(G.values(algo), ref, g.n)
                else:
                    got = G.values(algo)
                    np.testing.assert_array_equal(got.view(np.uint32), ref.view(np.uint32))
                    np.testing.assert_array_equal(G.trace(), rtr)
    og.close()


@pytest.mark.parametrize("pinned", [False, True])
def test_sorted_one_direction_streamed_borrowed(pinned):
    """PageRank from the in-CSC alone and BFS from the out-CSR alone, streamed, the
    caller's arrays used in place (pageable, or already page-locked by the caller)."""
    import torch

    scale, seed = 15, 5
    g = grgen.rmat(scale, 16, seed=seed)
    ci_off, ci, od, co_off, co = _layouts(scale, seed)
    if pinned:
        ci = torch.from_numpy(ci).pin_memory().numpy()
        co = torch.from_numpy(co).pin_memory().numpy()
    og = oracle.OracleGraph(g.n, g.src, g.dst)
    pr, _, _ = og.run("pagerank", max_iters=30)
    bfs, btr, bit = og.run("bfs", source=0)
    og.close()
    with gr.GraphReduce.from_sorted(g.n, g.m, in_offsets=ci_off, in_idx=ci, out_degree=od, mode="streamed",
                                    shard_edges=1 << 17, borrow=True) as G:
        assert G.info()["num_shards"] > 4
        st = G.run("pagerank")
        assert st["bytes_h2d"] >= 30 * 4 * g.m
        check_pr(G.values("pagerank"), pr, g.n)
        with pytest.raises(gr.GrError) as ei:
            G.run("bfs", source=0)
        assert ei.value.status == gr.GR_EUNSUPPORTED
    with gr.GraphReduce.from_sorted(g.n, g.m, row_offsets=co_off, col_idx=co, mode="streamed",
                                    shard_edges=1 << 17, borrow=True) as G:
        st = G.run("bfs", source=0)
        assert st["iterations"] == bit
        np.testing.assert_array_equal(G.values("bfs"), bfs)
        np.testing.assert_array_equal(G.trace(), btr)
        with pytest.raises(gr.GrError) as ei:
            G.run("pagerank")
        assert ei.value.status == gr.GR_EUNSUPPORTED


def test_sorted_input_validation():
    n = 4
    off = np.array([0, 1, 2, 3, 3], np.uint64)
    bad = np.array([3, 0, 9, 0, 0, 0, 0], np.uint32)  # id 9 >= n
    with pytest.raises(gr.GrError) as ei:
        gr.gr_graph_load_sorted(n, 3, in_offsets=off, in_idx=bad, mode="streamed")
    assert ei.value.status == gr.GR_EINVAL
    unsorted = np.array([3, 2, 1, 0, 0, 0, 0], np.uint32)
    off2 = np.array([0, 2, 2, 3, 3], np.uint64)  # row 0 = [3, 2]: not ascending
    with pytest.raises(gr.GrError) as ei:
        gr.gr_graph_load_sorted(n, 3, in_offsets=off2, in_idx=unsorted, mode="streamed")
    assert ei.value.status == gr.GR_EINVAL
    ok = np.array([1, 2, 3, 0, 0, 0, 0], np.uint32)
    with pytest.raises(gr.GrError) as ei:  # one half must be streamed
        gr.gr_graph_load_sorted(n, 3, in_offsets=off, in_idx=ok, mode="resident")
    assert ei.value.status == gr.GR_EUNSUPPORTED
