import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np
import oracle
import paper_conf_sc_senguptasas15_b200 as gr
from test_gpu_parity import hub_graph
os.environ["GR_PR_KERNEL"] = sys.argv[1] if len(sys.argv) > 1 else "warphot"
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 2
n, src, dst, _ = hub_graph(k=70000, extra=1_200_000)
ref, _, _ = oracle.run(n, src, dst, "pagerank", max_iters=iters)
with gr.GraphReduce(n, src, dst) as G:
    G.run("pagerank", max_iters=iters)
    got = G.values("pagerank").astype(np.float64)
print("max err", np.abs(got - ref).max())
