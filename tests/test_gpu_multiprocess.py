"""The partitioned path across REAL processes (§8
L390): two ranks as two OS processes on one GPU, exchanging
through the shared-memory transport (GR_TRANSPORT_SHM) — POSIX shared memory
for the host collectives and real cross-process cudaIpc mappings for the device
data (the fused PageRank and frontier exchanges store into the peer process's
buffers from the kernels). Every rank must equal the oracle (integer programs
bit-exact with the trace; PageRank within the north_star tolerance)."""
import json
import os
import subprocess
import sys

import numpy as np
import pytest

import grgen
import oracle
from test_gpu_parity import check_pr

pytestmark = pytest.mark.gpu

HERE = os.path.dirname(os.path.abspath(__file__))


def run_ranks(tmp_path, n, src, dst, w, algo, world=2, source=0, max_iters=0, custom_id=0, env=None):
    inp = tmp_path / "g.npz"
    kw = dict(n=n, src=src, dst=dst, source=source, max_iters=max_iters)
    if w is not None:
        kw["w"] = w
    np.savez(inp, **kw)
    hexid = os.urandom(128).hex()
    procs, outs = [], []
    for r in range(world):
        out = tmp_path / f"r{r}.npz"
        outs.append(out)
        e = dict(os.environ, **(env or {}))
        procs.append(subprocess.Popen([sys.executable, os.path.join(HERE, "_mp_rank.py"), str(r), str(world), hexid,
                                       str(inp), str(out), algo, str(custom_id)], env=e,
                                      stdout=subprocess.PIPE, stderr=subprocess.STDOUT))
    logs = []
    for p in procs:
        try:
            o, _ = p.communicate(timeout=600)
        except subprocess.TimeoutExpired:
            for q in procs:
                q.kill()
            raise
        logs.append(o.decode(errors="replace"))
    for p, log in zip(procs, logs):
        assert p.returncode == 0, log[-4000:]
    res = []
    for out in outs:
        d = np.load(out)
        res.append(dict(vals=[d["vals0"], d["vals1"]], tr=[d["tr0"], d["tr1"]], st=json.loads(str(d["st"])),
                        info=json.loads(str(d["info"]))))
    return res


CASES = {
    "bfs": lambda: (grgen.rmat(13, 16, seed=8), None),
    "sssp": lambda: (grgen.rmat(13, 16, seed=8), "w"),
    "cc": lambda: (grgen.rmat(13, 16, seed=8), "sym"),
    "pagerank": lambda: (grgen.rmat(14, 16, seed=8), None),
    "pagerank_delta": lambda: (grgen.rmat(13, 16, seed=8), None),
}


@pytest.mark.timeout(900)
@pytest.mark.parametrize("exchange", ["fused", "fused-hostcounts", "allgatherv"])
@pytest.mark.parametrize("algo", list(CASES))
def test_two_processes_equal_oracle(tmp_path, algo, exchange):
    g, kind = CASES[algo]()
    src, dst, w = g.src, g.dst, None
    if kind == "sym":
        src, dst = np.concatenate([g.src, g.dst]), np.concatenate([g.dst, g.src])
    if kind == "w":
        w = grgen.weights(g.m, 1, 64, seed=9)
    # fused: changed sets stored into the peers by the gather, counts exchanged and the
    # PageRank supersteps separated on the device (k_part_publish / k_part_wait / k_xbar);
    # fused-hostcounts: the counts allgathered through the host, the communicator's barrier
    env = {"GR_FRONTIER_EXCHANGE": "nccl", "GR_PR_EXCHANGE": "nccl"} if exchange == "allgatherv" else \
        {"GR_COUNT_EXCHANGE": "host", "GR_PR_BARRIER": "comm"} if exchange == "fused-hostcounts" else {}
    mi = 30 if algo == "pagerank" else 0
    ref, rtr, rit = oracle.run(g.n, src, dst, algo, w=w, source=0, max_iters=mi)
    res = run_ranks(tmp_path, g.n, src, dst, w, algo, source=0, max_iters=mi, env=env)
    owned = 0
    for r in res:
        assert r["info"]["world"] == 2 and r["info"]["sim_ranks"] == 1
        owned += r["info"]["own_hi"] - r["info"]["own_lo"]
        for k in range(2):
            assert r["st"][k]["iterations"] == rit
            if algo == "pagerank":
                check_pr(r["vals"][k], ref, g.n)
            else:
                vals = r["vals"][k]
                if algo == "pagerank_delta":
                    vals, ref_ = vals.view(np.uint32), ref.view(np.uint32)
                else:
                    ref_ = ref
                np.testing.assert_array_equal(vals, ref_)
                np.testing.assert_array_equal(r["tr"][k], rtr)
        if exchange.startswith("fused") and algo != "pagerank":
            assert r["st"][0]["bytes_nvlink"] > 0  # the peers' changed sets arrived
    assert owned == g.n


@pytest.mark.timeout(900)
def test_two_processes_heat_scatter(tmp_path):
    """A scatter program (mutable edge state on the destination owner's edges)."""
    g = grgen.heat_grid(50, 40, seed=6)
    ref, rtr, rit = oracle.run(g.n, g.src, g.dst, "heat", w=g.w, source=17, max_iters=80)
    res = run_ranks(tmp_path, g.n, g.src, g.dst, g.w, "custom", source=17, max_iters=80, custom_id=2)
    for r in res:
        for k in range(2):
            assert r["st"][k]["iterations"] == rit
            np.testing.assert_array_equal(r["vals"][k], ref)
            np.testing.assert_array_equal(r["tr"][k], rtr)
