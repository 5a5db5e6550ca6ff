"""GPU parity: the CUDA path through the C ABI vs the oracle.

BFS / SSSP / CC bit-exact, frontier traces identical; PageRank within
max|dR| <= 1e-6 and L1 <= 1e-5 of the fp64 oracle (BASELINE.json north_star),
plus the internal gates of SURVEY §8(c): relative error <= 1e-4 where
R >= 1/n and |sum R - sum R_oracle| <= 1e-5.
"""
import numpy as np
import pytest

import grgen
import oracle
import paper_conf_sc_senguptasas15_b200 as gr

pytestmark = pytest.mark.gpu

PR_MAX, PR_L1 = 1e-6, 1e-5


def check_pr(got, ref, n):
    got = got.astype(np.float64)
    err = np.abs(got - ref)
    assert err.max() <= PR_MAX, err.max()
    assert err.sum() <= PR_L1, err.sum()
    big = ref >= 1.0 / n
    if big.any():
        assert (err[big] / ref[big]).max() <= 1e-4
    assert abs(got.sum() - ref.sum()) <= 1e-5


DIRS = ("auto", "push", "pull", "fused")


def compare(n, src, dst, w, algo, source=0, max_iters=0, loops=("auto", "device", "host"), directions=DIRS,
            run_kw=None, **load):
    """Every loop driver x every FrontierActivate direction (push / pull / the
    size heuristic) must reproduce the oracle's values and trace."""
    og = oracle.OracleGraph(n, src, dst, w)
    ref, rtr, rit = og.run(algo, source=source, max_iters=max_iters)
    og.close()
    with gr.GraphReduce(n, src, dst, w, **load) as G:
        resident1 = G.info()["mode"] == gr.MODES["resident"] and G.info()["world"] == 1
        for loop in loops:
            for d in (directions if algo != "pagerank" else ("auto",)):
                st = G.run(algo, source=source, max_iters=max_iters, loop=loop, direction=d, **(run_kw or {}))
                got = G.values(algo)
                tr = G.trace()
                assert st["iterations"] == rit, (loop, d, st["iterations"], rit)
                if algo == "pagerank":
                    check_pr(got, ref, n)
                    continue
                np.testing.assert_array_equal(got, ref, err_msg=f"{loop} {d}")
                np.testing.assert_array_equal(tr, rtr, err_msg=f"{loop} {d}")
                assert st["edges_gathered"] == int(rtr[:, 2].sum())
                assert st["edges_scattered"] == int(rtr[:, 3].sum())
                if resident1:  # bytes model from the device's running sums of |A_t|, |C_t|
                    wb = 5 if algo == "sssp" else 4
                    sa, sc = int(rtr[:, 0].sum()), int(rtr[:, 1].sum())
                    sg, ss = int(rtr[:, 2].sum()), int(rtr[:, 3].sum())
                    assert st["bytes_hbm_model"] in (wb * sg + 12 * sa + 4 * ss + 12 * sc,
                                                     16 * sa + wb * ss + 12 * sc), (loop, d)
                if d == "push" or not resident1:
                    assert st["pull_supersteps"] == 0
                elif d == "pull" and rtr[:, 1].sum() > 0:
                    assert st["pull_supersteps"] > 0
    return st


def rand_graph(seed, n, m, sym=False, wmax=64):
    rng = np.random.default_rng(seed)
    src = rng.integers(0, n, m).astype(np.uint32)
    dst = rng.integers(0, n, m).astype(np.uint32)
    w = rng.integers(1, wmax + 1, m).astype(np.uint32)
    if sym:
        src, dst, w = np.concatenate([src, dst]), np.concatenate([dst, src]), np.concatenate([w, w])
    return src, dst, w


ALGOS = ["bfs", "sssp", "cc", "pagerank", "pagerank_delta"]


@pytest.mark.parametrize("algo", ALGOS)
@pytest.mark.parametrize("seed,n,m", [(1, 1, 0), (2, 7, 20), (3, 200, 900), (4, 5000, 3000), (5, 3001, 40000)])
def test_random_graphs(algo, seed, n, m):
    src, dst, w = rand_graph(seed, n, m, sym=(algo == "cc"))
    compare(n, src, dst, w, algo, source=seed % n)


def hub_graph(k=5000, extra=3000, seed=9):
    """Star hubs above the CTA-per-vertex threshold plus random edges (both directions)."""
    rng = np.random.default_rng(seed)
    n = k + 10
    s = [np.zeros(k, np.uint32), np.arange(1, k + 1, dtype=np.uint32)]
    d = [np.arange(1, k + 1, dtype=np.uint32), np.zeros(k, np.uint32)]
    s.append(np.full(2000, 3, np.uint32))
    d.append(rng.integers(0, n, 2000).astype(np.uint32))
    s.append(rng.integers(0, n, extra).astype(np.uint32))
    d.append(rng.integers(0, n, extra).astype(np.uint32))
    src, dst = np.concatenate(s), np.concatenate(d)
    src, dst = np.concatenate([src, dst]), np.concatenate([dst, src])
    w = rng.integers(1, 65, len(src)).astype(np.uint32)
    return n, src, dst, w


@pytest.mark.parametrize("algo", ALGOS)
def test_hubs(algo):
    n, src, dst, w = hub_graph()
    for s in (0, 5, n - 1):
        compare(n, src, dst, w, algo, source=s)


@pytest.mark.parametrize("cfg", [1, 2, 3, 4])
def test_reduced_configs(cfg):
    g, run = grgen.config(cfg, reduced=True)
    w = g.get("w")
    if run["algo"] == "sssp" and w is None:
        w = grgen.weights(g.m, 1, 64, seed=cfg)
    compare(g.n, g.src, g.dst, w, run["algo"], source=run.get("source", 0), max_iters=run.get("max_iters", 0))


def test_sssp_unit_weights_equals_bfs_and_rmat_weights():
    g = grgen.rmat(14, 16, seed=7)
    w = np.ones(g.m, np.uint32)
    with gr.GraphReduce(g.n, g.src, g.dst, w) as G:
        G.run("bfs", source=0)
        b = G.values()
        G.run("sssp", source=0)
        s = G.values()
    np.testing.assert_array_equal(b, s)
    w = grgen.weights(g.m, 1, 64, seed=11)
    compare(g.n, g.src, g.dst, w, "sssp", source=0)


def test_repeated_runs_and_epochs():
    g = grgen.rmat(13, 8, seed=3)
    w = grgen.weights(g.m, 1, 64, seed=1)
    og = oracle.OracleGraph(g.n, g.src, g.dst, w)
    with gr.GraphReduce(g.n, g.src, g.dst, w) as G:
        for algo, s in [("bfs", 0), ("bfs", 17), ("sssp", 5), ("cc", 0), ("bfs", 0), ("pagerank", 0), ("sssp", 0)]:
            G.run(algo, source=s)
            ref, rtr, _ = og.run(algo, source=s)
            if algo == "pagerank":
                check_pr(G.values(algo), ref, g.n)
            else:
                np.testing.assert_array_equal(G.values(), ref)
                np.testing.assert_array_equal(G.trace(), rtr)
    og.close()


def test_pr_iteration_counts_and_closed_form_cycle():
    n = 1000
    src = np.arange(n, dtype=np.uint32)
    dst = ((src + 1) % n).astype(np.uint32)
    with gr.GraphReduce(n, src, dst) as G:
        for it in (1, 2, 30, 50):
            st = G.run("pagerank", max_iters=it)
            assert st["iterations"] == it
            np.testing.assert_allclose(G.values("pagerank"), 1.0 / n, rtol=1e-6)


def test_max_iters_truncates_frontier_programs():
    g = grgen.grid_road(60, 60, seed=3)
    compare(g.n, g.src, g.dst, g.w, "sssp", source=0, max_iters=7)
    compare(g.n, g.src, g.dst, g.w, "bfs", source=0, max_iters=3)


def test_errors_through_abi():
    src = np.array([0, 1, 2], np.uint32)
    dst = np.array([1, 2, 0], np.uint32)
    with gr.GraphReduce(3, src, dst) as G:
        with pytest.raises(gr.GrError) as ei:
            G.run("sssp", source=0)  # no weights
        assert ei.value.status == gr.GR_EINVAL
        with pytest.raises(gr.GrError) as ei:
            gr.gr_fetch_vertex_values(G.h)
        assert ei.value.status == gr.GR_ESTATE
        with pytest.raises(gr.GrError):
            G.run("bfs", source=3)
        with pytest.raises(gr.GrError):
            G.run("pagerank", damping=1.5)
        G.run("bfs", source=0)
        with pytest.raises(gr.GrError):
            gr.gr_fetch_vertex_values(G.h, np.empty(2, np.uint32))
        with pytest.raises(gr.GrError) as ei:
            G.run("custom", custom_id=77)
        assert ei.value.status == gr.GR_EUNSUPPORTED


# ---------------------------------------------------------------- streamed mode
@pytest.mark.parametrize("algo", ALGOS)
@pytest.mark.parametrize("shard_edges", [3000, 40000])
@pytest.mark.parametrize("zero_copy", [-1, 0, 1])
def test_streamed_equals_oracle(algo, shard_edges, zero_copy):
    """Whole-shard DMA (-1), in-place reads over the host link (1) and the
    per-phase choice (0) all reproduce the oracle."""
    g = grgen.rmat(13, 16, seed=4)
    src, dst = g.src, g.dst
    if algo == "cc":
        src, dst = np.concatenate([g.src, g.dst]), np.concatenate([g.dst, g.src])
    w = grgen.weights(len(src), 1, 64, seed=5)
    st = compare(g.n, src, dst, w, algo, source=1, loops=("host",), mode="streamed", shard_edges=shard_edges,
                 run_kw={"zero_copy": zero_copy})
    assert st["bytes_h2d"] > 0
    if zero_copy < 0:
        assert st["bytes_h2d_zero_copy"] == 0 and st["zero_copy_phases"] == 0
    if zero_copy > 0:  # nothing staged: every byte was read in place
        assert st["bytes_h2d"] == st["bytes_h2d_zero_copy"] > 0
        wb = 5 if algo == "sssp" else 4
        if algo == "pagerank":
            assert st["bytes_h2d"] == 4 * len(src) * st["iterations"]
        else:
            assert st["bytes_h2d"] == wb * st["edges_gathered"] + 4 * st["edges_scattered"]


@pytest.mark.parametrize("algo", ALGOS)
def test_streamed_hub_larger_than_shard(algo):
    n, src, dst, w = hub_graph()
    compare(n, src, dst, w, algo, source=0, loops=("host",), mode="streamed", shard_edges=2000)


@pytest.mark.parametrize("cfg", [1, 3, 4])
def test_streamed_reduced_configs(cfg):
    g, run = grgen.config(cfg, reduced=True)
    w = g.get("w")
    compare(g.n, g.src, g.dst, w, run["algo"], source=run.get("source", 0), loops=("host",), mode="streamed",
            shard_edges=max(1000, g.m // 16))


def test_streamed_frontier_skips_inactive_shards():
    # two disjoint directed paths: BFS from the first never copies a shard of the second
    k = 20000
    a = np.arange(k - 1, dtype=np.uint32)
    src = np.concatenate([a, a + k])
    dst = np.concatenate([a + 1, a + 1 + k])
    with gr.GraphReduce(2 * k, src, dst, mode="streamed", shard_edges=4000) as G:
        info = G.info()
        assert info["mode"] == 2 and info["num_shards"] > 4
        shards = [gr.gr_shard_info(G.h, s) for s in range(info["num_shards"])]
        first = [s for s in shards if s["v_lo"] < k]
        max_first = max(4 * (s["out_end"] - s["out_begin"]) for s in first)
        st = G.run("bfs", source=0, zero_copy=-1)
        assert st["iterations"] == k
        # one changed vertex per superstep => at most one shard's out-edges copied per superstep
        assert st["bytes_h2d"] <= st["iterations"] * max_first
        # and in total never more than the first path's shards once per superstep they were active
        whole = 4 * (len(src))
        assert st["bytes_h2d"] < st["iterations"] * whole / 4
        d = G.values()
        assert d[k - 1] == k - 1 and d[k] == gr.INF
        # f1: with one frontier vertex per superstep the auto policy reads its
        # single out-edge in place instead of DMA-ing a shard
        st2 = G.run("bfs", source=0, zero_copy=0)
        assert st2["zero_copy_phases"] == st2["iterations"]  # one (activation) phase per superstep
        assert st2["bytes_h2d"] == st2["bytes_h2d_zero_copy"] == 4 * (k - 1)
        np.testing.assert_array_equal(G.values(), d)


@pytest.mark.parametrize("variant", ["block", "warp", "warphot", "seg", "seg-launches"])
def test_pagerank_kernel_variants(variant, monkeypatch):
    """Every PageRank gather the library still selects (CTA merge-path tiles when
    no shared-memory table fits, warp merge-path tiles for small partitions, the
    same with the hot-source table when the seg layout's indices would
    overflow; the edge-segmented tiles in the persistent loop or one launch per
    phase) meets the PageRank bar."""
    if variant == "seg-launches":
        monkeypatch.setenv("GR_PR_LOOP", "0")
    variant = variant.split("-")[0]
    monkeypatch.setenv("GR_PR_KERNEL", variant)
    g = grgen.rmat(17, 16, seed=12)  # > 2^20 edges so the hot table engages
    ref, _, _ = oracle.run(g.n, g.src, g.dst, "pagerank", max_iters=30)
    with gr.GraphReduce(g.n, g.src, g.dst) as G:
        st = G.run("pagerank")
        assert st["kernel_ms"][3] == {"block": 0, "warp": 2, "warphot": 3, "seg": 7}[variant]
        check_pr(G.values("pagerank"), ref, g.n)
    n, src, dst, _ = hub_graph(k=70000, extra=1_200_000)
    ref, _, _ = oracle.run(n, src, dst, "pagerank", max_iters=30)
    with gr.GraphReduce(n, src, dst) as G:
        G.run("pagerank")
        check_pr(G.values("pagerank"), ref, n)


def test_pagerank_tma_stream(monkeypatch):
    """The persistent PageRank loop with its item / head-bit streams moved by TMA
    bulk copies into per-warp staging (GR_PR_TMA=1, cp.async.bulk + mbarrier)
    sums in exactly the order of the load path (GR_PR_TMA=0): bit-identical
    ranks, both within the PageRank bar of the oracle. Graphs with hub rows
    spanning many tiles and with more tiles than warps (several tiles per warp,
    both staging buffers reused across supersteps)."""
    for g in (grgen.rmat(17, 16, seed=12), grgen.rmat(16, 24, seed=13)):
        ref, _, _ = oracle.run(g.n, g.src, g.dst, "pagerank", max_iters=30)
        got = {}
        for tma in ("1", "0"):
            monkeypatch.setenv("GR_PR_TMA", tma)
            with gr.GraphReduce(g.n, g.src, g.dst) as G:
                st = G.run("pagerank")
                assert st["kernel_ms"][3] == 7
                got[tma] = G.values("pagerank").copy()
                G.run("pagerank")  # a second run reuses the mbarriers' phases from zero
                np.testing.assert_array_equal(G.values("pagerank").view(np.uint32), got[tma].view(np.uint32))
            check_pr(got[tma], ref, g.n)
        np.testing.assert_array_equal(got["1"].view(np.uint32), got["0"].view(np.uint32))


@pytest.mark.parametrize("block_v,policy", [(10000, "1"), (10000, "0"), (40000, "1"), (1 << 16, "1")])
def test_pagerank_source_blocked(block_v, policy, monkeypatch):
    """the source-blocked layout (sources cut into blocks whose
    contributions fit in L2; one run per (destination, block); per-block
    reduction phases + an apply phase) meets the PageRank bar, with and without
    the L2 cache-policy hints, for block counts 2..14, on an R-MAT graph and on
    a hub graph whose runs span many tiles."""
    monkeypatch.setenv("GR_PR_BLOCK_V", str(block_v))
    monkeypatch.setenv("GR_PR_BLOCK_POLICY", policy)
    g = grgen.rmat(17, 16, seed=12)
    ref, _, _ = oracle.run(g.n, g.src, g.dst, "pagerank", max_iters=30)
    with gr.GraphReduce(g.n, g.src, g.dst) as G:
        st = G.run("pagerank")
        assert st["kernel_ms"][3] == 8
        first = G.values("pagerank")
        check_pr(first, ref, g.n)
        G.run("pagerank")
        np.testing.assert_array_equal(G.values("pagerank"), first)  # fixed summation order
    n, src, dst, _ = hub_graph(k=70000, extra=1_200_000)
    ref, _, _ = oracle.run(n, src, dst, "pagerank", max_iters=30)
    with gr.GraphReduce(n, src, dst) as G:
        G.run("pagerank", max_iters=30)
        check_pr(G.values("pagerank"), ref, n)


@pytest.mark.parametrize("seed", [1, 2])
def test_device_build_matches_host_build(seed):
    """The GPU shard builder produces the host builder's layout exactly: every
    program (PageRank included, same fp32 summation order) is bit-identical,
    and the shard tables agree."""
    g = grgen.rmat(14, 16, seed=seed)
    w = grgen.weights(g.m, 1, 64, seed=seed)
    src = np.concatenate([g.src, g.src[:5000]])  # extra duplicates with other weights
    dst = np.concatenate([g.dst, g.dst[:5000]])
    w = np.concatenate([w, (w[:5000] % 7) + 1]).astype(np.uint32)
    res = {}
    for build in ("host", "device"):
        with gr.GraphReduce(g.n, src, dst, w, build=build, shard_edges=50000) as G:
            info = G.info()
            shards = [gr.gr_shard_info(G.h, s) for s in range(info["num_shards"])]
            out = {"shards": shards}
            for algo in ("bfs", "sssp", "cc", "pagerank"):
                G.run(algo, source=3)
                out[algo] = (G.values(algo), G.trace())
            res[build] = out
    assert res["host"]["shards"] == res["device"]["shards"]
    for algo in ("bfs", "sssp", "cc", "pagerank"):
        np.testing.assert_array_equal(res["host"][algo][0], res["device"][algo][0])
        np.testing.assert_array_equal(res["host"][algo][1], res["device"][algo][1])
    with pytest.raises(gr.GrError):
        gr.GraphReduce(4, np.array([0, 9], np.uint32), np.array([1, 2], np.uint32), build="device")


@pytest.mark.parametrize("mode", ["resident", "streamed"])
def test_custom_program_widest_path(mode):
    """A user program registered with GR_CUSTOM_PROGRAMS (include/gr/program.cuh)
    runs through the same engine and equals the oracle's widest path exactly."""
    for seed in (1, 2):
        g = grgen.rmat(12, 16, seed=seed)
        w = grgen.weights(g.m, 1, 64, seed=seed + 7)
        ref, rtr, rit = oracle.run(g.n, g.src, g.dst, "widest", w=w, source=0)
        kw = dict(mode=mode, shard_edges=6000) if mode == "streamed" else {}
        with gr.GraphReduce(g.n, g.src, g.dst, w, **kw) as G:
            for loop in (("auto", "device", "host") if mode == "resident" else ("host",)):
                st = G.run("custom", custom_id=0, source=0, loop=loop)
                assert st["iterations"] == rit
                np.testing.assert_array_equal(G.values(), ref)
                np.testing.assert_array_equal(G.trace(), rtr)
    n, src, dst, w = hub_graph()
    ref, rtr, _ = oracle.run(n, src, dst, "widest", w=w, source=5)
    with gr.GraphReduce(n, src, dst, w) as G:
        G.run("custom", custom_id=0, source=5)
        np.testing.assert_array_equal(G.values(), ref)
        np.testing.assert_array_equal(G.trace(), rtr)


# Run-time programs: the paper's GAS functors (§4.1
# L196, Fig. 6) written as source strings, compiled by gr_program_compile.
JIT_SSSP = r"""
struct JitSSSP {
  using GatherT = uint32_t;
  static constexpr bool kHasGather = true;
  static constexpr bool kUsesWeights = true;
  static constexpr int kInit = kInitSourceChanged;
  __device__ static uint32_t initValue(uint32_t v, const Ctx &c) { return v == c.source ? 0u : 0xFFFFFFFFu; }
  __host__ __device__ static GatherT identity() { return 0xFFFFFFFFu; }
  static GatherT identity_host() { return 0xFFFFFFFFu; }
  __device__ static GatherT gatherMap(uint32_t, uint32_t s, uint32_t w, uint32_t, const Ctx &) {
    const uint32_t r = s + w;
    return (s == 0xFFFFFFFFu || r < s || r == 0xFFFFFFFFu) ? 0xFFFFFFFFu : r;
  }
  __device__ static GatherT gatherReduce(GatherT a, GatherT b) { return a < b ? a : b; }
  __device__ static void atomicGather(GatherT *acc, GatherT r) { atomicMin(acc, r); }
  __device__ static bool apply(uint32_t *cur, GatherT r, const Ctx &) {
    const bool changed = r < *cur;
    if (changed) *cur = r;
    return changed;
  }
};
"""

JIT_CC64 = r"""
// connected components with a 64-bit gather type (exercises GatherT = 8 bytes)
struct JitCC64 {
  using GatherT = unsigned long long;
  static constexpr bool kHasGather = true;
  static constexpr bool kUsesWeights = false;
  static constexpr int kInit = kInitAll;
  __device__ static uint32_t initValue(uint32_t v, const Ctx &) { return v; }
  __host__ __device__ static GatherT identity() { return ~0ull; }
  static GatherT identity_host() { return ~0ull; }
  __device__ static GatherT gatherMap(uint32_t, uint32_t s, uint32_t, uint32_t, const Ctx &) { return s; }
  __device__ static GatherT gatherReduce(GatherT a, GatherT b) { return a < b ? a : b; }
  __device__ static void atomicGather(GatherT *acc, GatherT r) { atomicMin(acc, r); }
  __device__ static bool apply(uint32_t *cur, GatherT r, const Ctx &) {
    const bool changed = r < *cur;
    if (changed) *cur = (uint32_t)r;
    return changed;
  }
};
"""

JIT_WIDEST = r"""
struct JitWidest {
  using GatherT = uint32_t;
  static constexpr bool kHasGather = true;
  static constexpr bool kUsesWeights = true;
  static constexpr int kInit = kInitSourceChanged;
  __device__ static uint32_t initValue(uint32_t v, const Ctx &c) { return v == c.source ? 0xFFFFFFFFu : 0u; }
  __host__ __device__ static GatherT identity() { return 0u; }
  static GatherT identity_host() { return 0u; }
  __device__ static GatherT gatherMap(uint32_t, uint32_t s, uint32_t w, uint32_t, const Ctx &) { return s < w ? s : w; }
  __device__ static GatherT gatherReduce(GatherT a, GatherT b) { return a > b ? a : b; }
  __device__ static void atomicGather(GatherT *acc, GatherT r) { atomicMax(acc, r); }
  __device__ static bool apply(uint32_t *cur, GatherT r, const Ctx &) {
    const bool changed = r > *cur;
    if (changed) *cur = r;
    return changed;
  }
};
"""

_jit_ids = {}


def jit_id(src, name):
    if name not in _jit_ids:
        _jit_ids[name] = gr.gr_program_compile(src, name)
    return _jit_ids[name]


@pytest.mark.parametrize("prog", ["sssp", "cc64", "widest"])
def test_runtime_program_equals_oracle(prog):
    """a program compiled at run time through the C ABI runs the
    library's own frontier engine and equals the oracle exactly (values, trace)."""
    src, name, algo = {"sssp": (JIT_SSSP, "JitSSSP", "sssp"), "cc64": (JIT_CC64, "JitCC64", "cc"),
                       "widest": (JIT_WIDEST, "JitWidest", "widest")}[prog]
    cid = jit_id(src, name)
    assert cid >= 1000
    for seed in (1, 2):
        g = grgen.rmat(13, 16, seed=seed)
        w = grgen.weights(g.m, 1, 64, seed=seed + 7)
        s, d = g.src, g.dst
        if prog == "cc64":
            s, d = np.concatenate([g.src, g.dst]), np.concatenate([g.dst, g.src])
            w = None
        ref, rtr, rit = oracle.run(g.n, s, d, algo, w=w, source=0)
        with gr.GraphReduce(g.n, s, d, w) as G:
            for direction in ("auto", "push"):
                st = G.run("custom", custom_id=cid, source=0, direction=direction)
                assert st["iterations"] == rit
                np.testing.assert_array_equal(G.values(), ref)
                np.testing.assert_array_equal(G.trace(), rtr)
    n, src, dst, w = hub_graph()
    ref, rtr, _ = oracle.run(n, src, dst, algo if prog != "cc64" else "cc", w=w if prog != "cc64" else None,
                             source=5)
    with gr.GraphReduce(n, src, dst, w) as G:
        G.run("custom", custom_id=cid, source=5)
        np.testing.assert_array_equal(G.values(), ref)
        np.testing.assert_array_equal(G.trace(), rtr)


def test_runtime_program_errors():
    """Compile errors carry the NVRTC log; a program reading weights needs them."""
    with pytest.raises(gr.GrError) as ei:
        gr.gr_program_compile("struct Broken { this is not C++ };", "Broken")
    assert ei.value.status == gr.GR_ECUDA and "NVRTC" in str(ei.value)
    cid = jit_id(JIT_SSSP, "JitSSSP")
    g = grgen.rmat(10, 8, seed=3)
    with gr.GraphReduce(g.n, g.src, g.dst) as G:  # no weights
        with pytest.raises(gr.GrError) as ei:
            G.run("custom", custom_id=cid)
        assert ei.value.status == gr.GR_EINVAL


@pytest.mark.parametrize("fmt", ["coo", "csr"])
def test_load_from_file(tmp_path, fmt):
    """gr_graph_load_file (mmap of the canonical file) == in-memory load, both formats."""
    g = grgen.rmat(13, 8, seed=4)
    w = grgen.weights(g.m, 1, 64, seed=4)
    path = tmp_path / "g.bin"
    if fmt == "coo":
        gr.write_graph_file(path, g.n, g.src, g.dst, w)
    else:
        order = np.lexsort((g.dst, g.src))
        ro = np.zeros(g.n + 1, np.uint64)
        ro[1:] = np.cumsum(np.bincount(g.src, minlength=g.n))
        gr.write_graph_file(path, g.n, row_offsets=ro, col_idx=g.dst[order], weights=w[order])
    og = oracle.OracleGraph(g.n, g.src, g.dst, w)
    with gr.GraphReduce.from_file(path) as G:
        assert G.n == g.n and G.info()["num_edges"] == g.m
        for algo in ("bfs", "sssp", "pagerank"):
            G.run(algo, source=1)
            ref, rtr, _ = og.run(algo, source=1)
            if algo == "pagerank":
                check_pr(G.values(algo), ref, g.n)
            else:
                np.testing.assert_array_equal(G.values(algo), ref)
                np.testing.assert_array_equal(G.trace(), rtr)
    og.close()


@pytest.mark.parametrize("tol", [0.0, 1e-6, 1e-3])
def test_pagerank_delta_rmat_tolerances(tol):
    """Tolerance-driven PageRank: ranks bit-identical to the
    oracle (exact fixed-point gather) and the shrinking frontier trace equal,
    on an R-MAT with hubs above the chunk threshold; with a tolerance the
    supersteps activate ever fewer vertices."""
    g = grgen.rmat(15, 16, seed=21)
    mi = 40 if tol == 0.0 else 0
    ref, rtr, rit = oracle.run(g.n, g.src, g.dst, "pagerank_delta", tolerance=tol, max_iters=mi)
    with gr.GraphReduce(g.n, g.src, g.dst) as G:
        for d in DIRS:
            st = G.run("pagerank_delta", tolerance=tol, max_iters=mi, direction=d)
            np.testing.assert_array_equal(G.values("pagerank_delta").view(np.uint32), ref.view(np.uint32))
            np.testing.assert_array_equal(G.trace(), rtr)
            assert st["iterations"] == rit
        if tol > 0:  # the frontier shrinks (Figs. 16-17): late supersteps gather a fraction of V
            assert rtr[-1, 0] < g.n // 4 and rtr[:, 0].min() < g.n


def test_custom_program_edge_messages():
    """Mutable edge state (the paper's Scatter phase, §2.1, §4.4
    L253): ProgSSSPMsg (custom id 1) keeps a message on every edge, written by
    scatter after the commit and read by the gather; bit-exact values and
    traces against the oracle's OR_SSSPMSG in every loop."""
    cases = []
    for seed in (1, 2):
        g = grgen.rmat(12, 16, seed=seed)
        cases.append((g.n, g.src, g.dst, grgen.weights(g.m, 1, 64, seed=seed + 7), 0))
    n, src, dst, w = hub_graph()
    cases.append((n, src, dst, w, 5))
    g = grgen.grid_road(80, 80, seed=3)
    cases.append((g.n, g.src, g.dst, g.w, 0))
    for (n, src, dst, w, s) in cases:
        ref, rtr, rit = oracle.run(n, src, dst, "sssp_msg", w=w, source=s)
        with gr.GraphReduce(n, src, dst, w) as G:
            for loop in ("auto", "device", "host"):
                for _ in range(2):  # edge states are reset per run
                    st = G.run("custom", custom_id=1, source=s, loop=loop)
                    assert st["iterations"] == rit
                    np.testing.assert_array_equal(G.values(), ref)
                    np.testing.assert_array_equal(G.trace(), rtr)
                    assert st["pull_supersteps"] == 0


@pytest.mark.parametrize("zero_copy", [-1, 0, 1])
def test_edge_messages_streamed(zero_copy):
    """Streamed (out-of-core) runs of the scatter program: the edge states live in
    mapped pinned host memory and are read by the gathers and rewritten by the
    scatters in place over the host link; shards copied or read in place."""
    g = grgen.rmat(11, 16, seed=5)
    w = grgen.weights(g.m, 1, 64, seed=6)
    ref, rtr, rit = oracle.run(g.n, g.src, g.dst, "sssp_msg", w=w, source=0)
    with gr.GraphReduce(g.n, g.src, g.dst, w, mode="streamed", shard_edges=3000) as G:
        assert G.info()["mode"] == gr.MODES["streamed"]
        for _ in range(2):
            st = G.run("custom", custom_id=1, source=0, zero_copy=zero_copy)
            assert st["iterations"] == rit
            np.testing.assert_array_equal(G.values(), ref)
            np.testing.assert_array_equal(G.trace(), rtr)


@pytest.mark.parametrize("force", ["1", "0"])
@pytest.mark.parametrize("algo", ["sssp", "cc", "pagerank_delta"])
def test_dense_tile_gather_forced(algo, force, monkeypatch):
    """Dense (pull) supersteps on edge-segmented tiles (GR_DENSE_SEG=1, the
    default only for 64-bit gathers) and on the vertex path (GR_DENSE_SEG=0):
    identical values and traces, including hubs whose rows span many tiles."""
    monkeypatch.setenv("GR_DENSE_SEG", force)
    g = grgen.rmat(13, 16, seed=21)
    src, dst = g.src, g.dst
    if algo == "cc":
        src, dst = np.concatenate([g.src, g.dst]), np.concatenate([g.dst, g.src])
    w = grgen.weights(len(src), 1, 64, seed=22)
    compare(g.n, src, dst, w, algo, loops=("auto",), directions=("pull", "auto"))
    n, s2, d2, w2 = hub_graph()
    compare(n, s2, d2, w2, algo, loops=("auto",), directions=("pull",))


def _oracle_run(n, src, dst, w, algo, source, max_iters=0):
    if algo == "widest":
        return oracle.run(n, src, dst, "widest", w=w, source=source)
    if algo == "heat":
        return oracle.run(n, src, dst, "heat", w=w, source=source, max_iters=max_iters)
    og = oracle.OracleGraph(n, src, dst, w)
    try:
        return og.run(algo, source=source, max_iters=max_iters)
    finally:
        og.close()


@pytest.mark.parametrize("force", ["1", "1out", "1nosym", "0"])
@pytest.mark.parametrize("algo", ["sssp", "cc", "widest", "heat"])
def test_vertex_records_forced(algo, force, monkeypatch):
    """Vertex records (GR_REC=1: one 32-byte record per vertex with its first
    kRecDeg = 4 neighbours, weights, degree and offset; the default for graphs
    whose vertices nearly all have degree <= 4, e.g. the cfg3 road grid) against
    the CSR/CSC path (GR_REC=0), with and without the activation records
    (GR_REC_OUT), and with the in-records serving the activation of symmetric
    graphs (the road grid, the hub graph; GR_REC_SYM): identical values and
    traces in every loop and direction. The R-MAT graph mixes record lanes (degree <= 4) with packed,
    warp-cooperative and hub lanes in one warp; the road grid is all records;
    heat diffusion reads its edge states through the record's offset."""
    monkeypatch.setenv("GR_REC", force[0])
    monkeypatch.setenv("GR_REC_OUT", "1" if force == "1out" else "0")  # activation records too
    monkeypatch.setenv("GR_REC_SYM", "0" if force == "1nosym" else "1")  # symmetric graphs: in-records activate
    cases = []
    road = grgen.grid_road(70, 61, seed=44)
    cases.append((road.n, road.src, road.dst, road.w))
    if algo != "heat":
        g = grgen.rmat(12, 8, seed=45)
        src, dst = g.src, g.dst
        if algo == "cc":
            src, dst = np.concatenate([g.src, g.dst]), np.concatenate([g.dst, g.src])
        cases.append((g.n, src, dst, grgen.weights(len(src), 1, 64, seed=46)))
        cases.append(hub_graph())
    else:
        h = grgen.heat_grid(40, 33, seed=47)
        cases = [(h.n, h.src, h.dst, h.w)]
    for n, src, dst, w in cases:
        mi = 60 if algo == "heat" else 0
        ref, rtr, rit = _oracle_run(n, src, dst, w, algo, 3, mi)
        with gr.GraphReduce(n, src, dst, w) as G:
            for loop in ("auto", "device", "host"):
                for d in (("push", "pull", "auto") if algo in ("sssp", "cc") else ("auto",)):
                    if algo in ("widest", "heat"):
                        cid = 0 if algo == "widest" else 2
                        st = G.run("custom", custom_id=cid, source=3, loop=loop, direction=d, max_iters=mi)
                    else:
                        st = G.run(algo, source=3, loop=loop, direction=d)
                    assert st["iterations"] == rit, (loop, d)
                    np.testing.assert_array_equal(G.values(), ref, err_msg=f"{loop} {d}")
                    np.testing.assert_array_equal(G.trace(), rtr, err_msg=f"{loop} {d}")


@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc", "pagerank", "pagerank_delta"])
def test_trace_detail_equals_oracle(algo):
    """the detail columns of the trace — shards holding an
    active vertex and distinct sources read by the gather — equal the oracle's
    (or_run_detail, pinned by brute force), with the graph's own shard bounds."""
    g = grgen.rmat(12, 16, seed=31)
    src, dst = g.src, g.dst
    if algo == "cc":
        src, dst = np.concatenate([g.src, g.dst]), np.concatenate([g.dst, g.src])
    w = grgen.weights(len(src), 1, 64, seed=32) if algo == "sssp" else None
    mi = 30 if algo == "pagerank" else (40 if algo == "pagerank_delta" else 0)
    for shard_edges in (0, 6000):
        with gr.GraphReduce(g.n, src, dst, w, shard_edges=shard_edges) as G:
            P = G.info()["num_shards"]
            bounds = np.array([gr.gr_shard_info(G.h, s)["v_lo"] for s in range(P)] + [g.n], np.uint64)
            og = oracle.OracleGraph(g.n, src, dst, w)
            ref, rtr, rdet, rit = og.run_detail(algo, shard_bounds=bounds, source=0, max_iters=mi)
            og.close()
            st = G.run(algo, source=0, max_iters=mi, trace_detail=True)
            assert st["iterations"] == rit
            det = G.trace_detail()
            if algo != "pagerank":
                np.testing.assert_array_equal(G.trace(), rtr)
            np.testing.assert_array_equal(det, rdet)
            if shard_edges:
                assert P > 4
