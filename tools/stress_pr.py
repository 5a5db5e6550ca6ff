import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np
import oracle
import paper_conf_sc_senguptasas15_b200 as gr
from test_gpu_parity import hub_graph
n, src, dst, _ = hub_graph(k=70000, extra=1_200_000)
ref, _, _ = oracle.run(n, src, dst, "pagerank", max_iters=30)
for variant in sys.argv[1:]:
    os.environ["GR_PR_KERNEL"] = variant
    for prof in (False, True):
        fails = 0
        for rep in range(12):
            with gr.GraphReduce(n, src, dst) as G:
                for it in range(3):
                    G.run("pagerank", profile=prof)
                    got = G.values("pagerank").astype(np.float64)
                    err = np.abs(got - ref)
                    if err.max() > 1e-6:
                        fails += 1
                        bad = np.nonzero(err > 1e-6)[0]
                        print(variant, "prof", prof, "rep", rep, "run", it, "max", err.max(), "nbad", len(bad),
                              "bad", bad[:8], "got", got[bad[:3]], "ref", ref[bad[:3]], flush=True)
        print(variant, "prof", prof, "fails", fails, "of 36", flush=True)
