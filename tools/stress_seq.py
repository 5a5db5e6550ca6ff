import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np
import grgen
import oracle
import paper_conf_sc_senguptasas15_b200 as gr
from test_gpu_parity import hub_graph
g = grgen.rmat(17, 16, seed=12)
ref1, _, _ = oracle.run(g.n, g.src, g.dst, "pagerank", max_iters=30)
n, src, dst, _ = hub_graph(k=70000, extra=1_200_000)
ref2, _, _ = oracle.run(n, src, dst, "pagerank", max_iters=30)
fails = 0
for rep in range(int(sys.argv[1]) if len(sys.argv) > 1 else 8):
    for variant in ["block", "warp", "warphot", "range", "rangehot"]:
        os.environ["GR_PR_KERNEL"] = variant
        for name, (nn, s_, d_, ref) in (("rmat17", (g.n, g.src, g.dst, ref1)), ("hub", (n, src, dst, ref2))):
            with gr.GraphReduce(nn, s_, d_) as G:
                st = G.run("pagerank")
                got = G.values("pagerank").astype(np.float64)
                info = G.info()
            err = np.abs(got - ref)
            if err.max() > 1e-6:
                fails += 1
                bad = np.nonzero(err > 1e-6)[0]
                print("FAIL rep", rep, variant, name, "kernel", st["kernel_ms"][3], "max", err.max(), "nbad", len(bad),
                      "bad", bad[:6], "got", got[bad[:3]], "ref", ref[bad[:3]], flush=True)
print("fails", fails, flush=True)
