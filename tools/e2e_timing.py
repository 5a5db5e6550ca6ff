import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["GR_TIMING"] = "1"
import numpy as np, torch
import grgen
import paper_conf_sc_senguptasas15_b200 as gr
g = grgen.rmat(22, 16, seed=2)
src = torch.from_numpy(g.src).pin_memory().numpy(); dst = torch.from_numpy(g.dst).pin_memory().numpy()
out = torch.empty(g.n, dtype=torch.float32).pin_memory().numpy()
for i in range(3):
    t0 = time.perf_counter()
    h = gr.gr_graph_load(g.n, src, dst)
    t1 = time.perf_counter()
    gr.gr_run(h, "pagerank")
    t2 = time.perf_counter()
    gr.gr_fetch_vertex_values(h, out)
    t3 = time.perf_counter()
    gr.gr_graph_free(h)
    t4 = time.perf_counter()
    print(f"load {1e3*(t1-t0):.1f} ms  run {1e3*(t2-t1):.1f}  fetch {1e3*(t3-t2):.1f}  free {1e3*(t4-t3):.1f}", file=sys.stderr, flush=True)
