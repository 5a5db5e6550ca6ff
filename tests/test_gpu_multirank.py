"""GPU parity of the partitioned (multi-GPU) path with SIMULATED ranks: G owner
partitions on one device, one host thread each, exchanging through device
copies — the same per-superstep protocol NCCL runs across GPUs.
Results must equal the single-threaded oracle exactly (BFS/SSSP/CC, traces
summed over ranks) or within the PageRank tolerance."""
import numpy as np
import pytest

import grgen
import oracle
import paper_conf_sc_senguptasas15_b200 as gr
from test_gpu_parity import check_pr, hub_graph

pytestmark = pytest.mark.gpu


# ------------------------------------------------- partitioned (simulated ranks)
def run_sim_ranks(n, src, dst, w, G, algo, source=0, max_iters=0, custom_id=0):
    """G owner partitions on ONE device, one host thread each, exchanging through
    device copies (the same protocol NCCL runs across GPUs)."""
    import os
    import threading

    key = os.urandom(128)
    out, errs = [None] * G, []

    def worker(r):
        h = None
        try:
            h = gr.gr_graph_load(n, src, dst, w, world=G, rank=r, sim_ranks=G, nccl_unique_id=key)
            st = gr.gr_run(h, algo, source=source, max_iters=max_iters, custom_id=custom_id)
            vals = gr.gr_fetch_vertex_values(h, dtype=np.float32 if algo in gr.FLOAT_ALGOS else np.uint32)
            tr = gr.gr_fetch_frontier_trace(h)
            out[r] = (st, vals, tr, gr.gr_graph_info_get(h))
        except Exception as e:  # pragma: no cover - surfaced below
            errs.append(e)
        finally:
            if h:
                gr.gr_graph_free(h)

    th = [threading.Thread(target=worker, args=(r,)) for r in range(G)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=600)
    assert not errs, errs
    return out


@pytest.mark.timeout(900)
@pytest.mark.parametrize("exchange", ["fused", "nccl"])
@pytest.mark.parametrize("G", [2, 3])
@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc", "pagerank", "pagerank_delta"])
def test_sim_ranks_equal_oracle(G, algo, exchange, monkeypatch):
    """fused: the changed set is stored into every rank's exchange buffer by the
    gather's own appends (peer mappings; same-device buffers for simulated ranks);
    nccl: the allgatherv of the changed set after the gather."""
    if exchange == "nccl":
        monkeypatch.setenv("GR_FRONTIER_EXCHANGE", "nccl")
    g = grgen.rmat(13, 16, seed=8)
    src, dst = g.src, g.dst
    if algo == "cc":
        src, dst = np.concatenate([g.src, g.dst]), np.concatenate([g.dst, g.src])
    w = grgen.weights(len(src), 1, 64, seed=9)
    ref, rtr, rit = oracle.run(g.n, src, dst, algo, w=w, source=0)
    res = run_sim_ranks(g.n, src, dst, w, G, algo, source=0)
    lo = [r[3]["own_lo"] for r in res]
    hi = [r[3]["own_hi"] for r in res]
    assert lo[0] == 0 and hi[-1] == g.n and all(lo[i + 1] == hi[i] for i in range(G - 1))
    for st, vals, tr, info in res:
        assert info["world"] == G and info["sim_ranks"] == G
        assert st["iterations"] == rit
        if algo == "pagerank":
            check_pr(vals, ref, g.n)
        else:
            np.testing.assert_array_equal(vals, ref)
            np.testing.assert_array_equal(tr, rtr)
            assert st["edges_gathered"] == int(rtr[:, 2].sum())


@pytest.mark.timeout(900)
def test_sim_ranks_hubs_and_configs():
    n, src, dst, w = hub_graph()
    for algo in ("bfs", "sssp", "cc", "pagerank"):
        ref, rtr, rit = oracle.run(n, src, dst, algo, w=w, source=0)
        for st, vals, tr, info in run_sim_ranks(n, src, dst, w, 4, algo, source=0):
            if algo == "pagerank":
                check_pr(vals, ref, n)
            else:
                np.testing.assert_array_equal(vals, ref)
                np.testing.assert_array_equal(tr, rtr)
    g = grgen.grid_road(120, 120, seed=3)
    ref, rtr, rit = oracle.run(g.n, g.src, g.dst, "sssp", w=g.w, source=0)
    for st, vals, tr, info in run_sim_ranks(g.n, g.src, g.dst, g.w, 2, "sssp", source=0):
        np.testing.assert_array_equal(vals, ref)
        np.testing.assert_array_equal(tr, rtr)


@pytest.mark.timeout(600)
@pytest.mark.parametrize("prog", [(0, "widest"), (1, "sssp_msg")])
def test_sim_ranks_custom_program(prog):
    """Registered programs over owner partitions; id 1 (SSSP by edge messages)
    keeps its edge states on the rank that owns the edge's destination."""
    pid, oname = prog
    g = grgen.rmat(12, 16, seed=3)
    w = grgen.weights(g.m, 1, 64, seed=4)
    ref, rtr, rit = oracle.run(g.n, g.src, g.dst, oname, w=w, source=0)
    import os
    import threading

    key = os.urandom(128)
    out, errs = [None] * 2, []

    def worker(r):
        h = None
        try:
            h = gr.gr_graph_load(g.n, g.src, g.dst, w, world=2, rank=r, sim_ranks=2, nccl_unique_id=key)
            gr.gr_run(h, "custom", custom_id=pid, source=0)
            out[r] = (gr.gr_fetch_vertex_values(h), gr.gr_fetch_frontier_trace(h))
        except Exception as e:
            errs.append(e)
        finally:
            if h:
                gr.gr_graph_free(h)

    th = [threading.Thread(target=worker, args=(r,)) for r in range(2)]
    [t.start() for t in th]
    [t.join(timeout=300) for t in th]
    assert not errs, errs
    for vals, tr in out:
        np.testing.assert_array_equal(vals, ref)
        np.testing.assert_array_equal(tr, rtr)


@pytest.mark.timeout(900)
@pytest.mark.parametrize("G", [2, 4])
@pytest.mark.parametrize("exchange", ["p2p", "nccl"])
@pytest.mark.parametrize("hot_min", ["0", "default"])
def test_sim_ranks_pagerank_exchange(G, exchange, hot_min, monkeypatch):
    """Partitioned PageRank, both exchanges: the apply's fused stores into every
    peer replica (p2p; same-device buffers of the simulated ranks stand in for
    the NVLink peer mappings) and the allgatherv of the owned slices (nccl);
    with the hot-table edge-segmented tiles (hot_min 0) and the plain warp tiles."""
    monkeypatch.setenv("GR_PR_EXCHANGE", exchange)
    if hot_min != "default":
        monkeypatch.setenv("GR_PR_HOT_MIN_EDGES", hot_min)
    g = grgen.rmat(14, 16, seed=11)
    ref, _, _ = oracle.run(g.n, g.src, g.dst, "pagerank", max_iters=30)
    res = run_sim_ranks(g.n, g.src, g.dst, None, G, "pagerank", max_iters=30)
    for st, vals, tr, info in res:
        check_pr(vals, ref, g.n)
        assert st["iterations"] == 30
        own = info["own_hi"] - info["own_lo"]
        assert st["bytes_nvlink"] == 29 * 4 * (g.n - own)  # every other rank's slice, once per exchange
