"""GPU parity of user GAS programs (§4.1, Fig. 6) with mutable edge
state (the Scatter phase, §2.1) in EVERY mode — resident, streamed and
partitioned — both compiled into the library (GR_CUSTOM_PROGRAMS) and compiled
at run time through the C ABI (gr_program_compile). The
workload is the paper's heat simulation (§2.1): oracle OR_HEAT, pinned in
tests/test_oracle_pins.py to the full fixed-point heat step and the fp64
matrix power. Values and traces must be bit-exact."""
import numpy as np
import pytest

import grgen
import oracle
import paper_conf_sc_senguptasas15_b200 as gr
from test_gpu_multirank import run_sim_ranks
from test_gpu_parity import JIT_SSSP, hub_graph, jit_id

pytestmark = pytest.mark.gpu

HEAT_ID = 2  # ProgHeat in GR_CUSTOM_PROGRAMS

JIT_HEAT = r"""
// heat diffusion with the heat flow stored on the edges (written as a user would)
struct JitHeat {
  using GatherT = uint32_t;
  static constexpr bool kHasGather = true;
  static constexpr bool kUsesWeights = true;
  static constexpr bool kHasScatter = true;
  static constexpr int kInit = kInitSourceChanged;
  __device__ static uint32_t initValue(uint32_t v, const Ctx &c) { return v == c.source ? 0x40000000u : 0u; }
  __host__ __device__ static GatherT identity() { return 0u; }
  static GatherT identity_host() { return 0u; }
  __device__ static uint32_t initEdge(uint32_t, const Ctx &) { return 0u; }
  __device__ static GatherT gatherMap(uint32_t, uint32_t, uint32_t heat, uint32_t, const Ctx &) { return heat; }
  __device__ static GatherT gatherReduce(GatherT a, GatherT b) { return a + b; }
  __device__ static void atomicGather(GatherT *acc, GatherT r) { atomicAdd(acc, r); }
  __device__ static bool apply(uint32_t *cur, GatherT r, const Ctx &) {
    const bool changed = r != *cur;
    *cur = r;
    return changed;
  }
  __device__ static void scatter(uint32_t s, uint32_t, uint32_t w, uint32_t *edge, const Ctx &) {
    *edge = (uint32_t)(((unsigned long long)s * (w + 1u)) >> 8);
  }
};
"""


def heat_cases():
    out = []
    for W, H, seed, s in ((40, 30, 6, 0), (70, 70, 7, 123)):
        g = grgen.heat_grid(W, H, seed=seed)
        out.append((g.n, g.src, g.dst, g.w, s))
    # a power-law graph with hubs: conductances that sum to 256 per vertex on a
    # symmetrized R-MAT (w = 0 on the lattice-free edges, the rest on a self-loop)
    n, src, dst, w = hub_graph()
    keep = src != dst
    src, dst = src[keep], dst[keep]
    deg = np.bincount(src, minlength=n)
    ok = deg[src] <= 255  # every vertex must keep (w + 1) <= 255 in total
    src, dst = src[ok], dst[ok]
    out_sum = np.bincount(src, minlength=n)
    v = np.arange(n, dtype=np.uint32)
    out.append((n, np.concatenate([src, v]), np.concatenate([dst, v]),
                np.concatenate([np.zeros(len(src), np.uint32), (255 - out_sum).astype(np.uint32)]), 0))
    return out


def _prog_id(kind):
    return HEAT_ID if kind == "builtin" else jit_id(JIT_HEAT, "JitHeat")


@pytest.mark.parametrize("kind", ["builtin", "jit"])
def test_heat_resident(kind):
    cid = _prog_id(kind)
    for n, src, dst, w, s in heat_cases():
        ref, rtr, rit = oracle.run(n, src, dst, "heat", w=w, source=s, max_iters=150)
        with gr.GraphReduce(n, src, dst, w) as G:
            for loop in (("auto", "device", "host") if kind == "builtin" else ("auto",)):
                for _ in range(2):  # edge states are reset per run
                    st = G.run("custom", custom_id=cid, source=s, max_iters=150, loop=loop)
                    assert st["iterations"] == rit
                    np.testing.assert_array_equal(G.values(), ref)
                    np.testing.assert_array_equal(G.trace(), rtr)


@pytest.mark.parametrize("zero_copy", [-1, 0, 1])
@pytest.mark.parametrize("kind", ["builtin", "jit"])
def test_heat_streamed(kind, zero_copy):
    cid = _prog_id(kind)
    n, src, dst, w, s = heat_cases()[1]
    ref, rtr, rit = oracle.run(n, src, dst, "heat", w=w, source=s, max_iters=120)
    with gr.GraphReduce(n, src, dst, w, mode="streamed", shard_edges=4000) as G:
        assert G.info()["mode"] == gr.MODES["streamed"] and G.info()["num_shards"] > 2
        st = G.run("custom", custom_id=cid, source=s, max_iters=120, zero_copy=zero_copy)
        assert st["iterations"] == rit
        np.testing.assert_array_equal(G.values(), ref)
        np.testing.assert_array_equal(G.trace(), rtr)


@pytest.mark.timeout(900)
@pytest.mark.parametrize("G", [2, 3])
@pytest.mark.parametrize("kind", ["builtin", "jit"])
def test_heat_partitioned(kind, G):
    cid = _prog_id(kind)
    for n, src, dst, w, s in heat_cases()[::2]:
        ref, rtr, rit = oracle.run(n, src, dst, "heat", w=w, source=s, max_iters=100)
        res = run_sim_ranks(n, src, dst, w, G, "custom", source=s, max_iters=100, custom_id=cid)
        for st, vals, tr, info in res:
            assert st["iterations"] == rit
            np.testing.assert_array_equal(vals, ref)
            np.testing.assert_array_equal(tr, rtr)


def test_runtime_program_streamed_and_partitioned():
    """A run-time program without scatter runs the streamed and partitioned drivers
    with its own kernel table (prog_desc.h) and equals the oracle exactly."""
    cid = jit_id(JIT_SSSP, "JitSSSP")
    g = grgen.rmat(12, 16, seed=3)
    w = grgen.weights(g.m, 1, 64, seed=4)
    ref, rtr, rit = oracle.run(g.n, g.src, g.dst, "sssp", w=w, source=0)
    with gr.GraphReduce(g.n, g.src, g.dst, w, mode="streamed", shard_edges=20000) as G:
        for zc in (-1, 0, 1):
            st = G.run("custom", custom_id=cid, source=0, zero_copy=zc)
            assert st["iterations"] == rit
            np.testing.assert_array_equal(G.values(), ref)
            np.testing.assert_array_equal(G.trace(), rtr)
    for st, vals, tr, info in run_sim_ranks(g.n, g.src, g.dst, w, 2, "custom", source=0, custom_id=cid):
        assert st["iterations"] == rit
        np.testing.assert_array_equal(vals, ref)
        np.testing.assert_array_equal(tr, rtr)


def test_runtime_program_loop_refused():
    """Resident run-time programs run the persistent loop; other loop requests are refused."""
    cid = jit_id(JIT_SSSP, "JitSSSP")
    g = grgen.rmat(10, 8, seed=3)
    w = grgen.weights(g.m, 1, 64, seed=3)
    with gr.GraphReduce(g.n, g.src, g.dst, w) as G:
        for loop in ("host", "device"):
            with pytest.raises(gr.GrError) as ei:
                G.run("custom", custom_id=cid, loop=loop)
            assert ei.value.status == gr.GR_EUNSUPPORTED
        G.run("custom", custom_id=cid, loop="persistent")
