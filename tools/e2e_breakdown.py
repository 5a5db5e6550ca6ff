"""End-to-end breakdown (load / run / fetch) through the C ABI with pinned host
buffers, with the library's internal load marks (GR_TIMING=1) — cfg2 or cfg4."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["GR_TIMING"] = "1"
import torch  # noqa: E402

import grgen  # noqa: E402
import paper_conf_sc_senguptasas15_b200 as gr  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
g, run = grgen.config(cfg)
src = torch.from_numpy(g.src).pin_memory().numpy()
dst = torch.from_numpy(g.dst).pin_memory().numpy()
out = torch.empty(g.n, dtype=torch.float32).pin_memory().numpy()
for i in range(3):
    t0 = time.perf_counter()
    h = gr.gr_graph_load(g.n, src, dst)
    t1 = time.perf_counter()
    gr.gr_run(h, run["algo"])
    t2 = time.perf_counter()
    gr.gr_fetch_vertex_values(h, out.view("uint32") if run["algo"] != "pagerank" else out)
    t3 = time.perf_counter()
    gr.gr_graph_free(h)
    t4 = time.perf_counter()
    print(f"cfg{cfg} load {1e3*(t1-t0):.1f} ms  run {1e3*(t2-t1):.1f}  fetch {1e3*(t3-t2):.1f}  free {1e3*(t4-t3):.1f}",
          file=sys.stderr, flush=True)
