import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import oracle
import paper_conf_sc_senguptasas15_b200 as gr
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
from test_gpu_parity import hub_graph
n, src, dst, _ = hub_graph(k=70000, extra=1_200_000)
ref, _, _ = oracle.run(n, src, dst, "pagerank", max_iters=30)
for v in ["block", "warp", "warphot", "range", "rangehot"]:
    os.environ["GR_PR_KERNEL"] = v
    for it in (1, 2, 30):
        r1, _, _ = oracle.run(n, src, dst, "pagerank", max_iters=it)
        with gr.GraphReduce(n, src, dst) as G:
            G.run("pagerank", max_iters=it)
            got = G.values("pagerank").astype(np.float64)
        err = np.abs(got - r1)
        bad = np.argsort(-err)[:3]
        print(v, it, "max", err.max(), "at", bad, "vals", got[bad], r1[bad])
