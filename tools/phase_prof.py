"""Per-phase device time of a frontier run (gr_run_opts.profile: %globaltimer
spans of the gather/apply phase [0] and the activate / BFS phase [1], summed
over supersteps) next to the event-timed run. Usage:
python tools/phase_prof.py CONFIG [ALGO] [REPS]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import grgen  # noqa: E402
import paper_conf_sc_senguptasas15_b200 as gr  # noqa: E402

cfg = int(sys.argv[1])
g, run = grgen.config(cfg)
algo = sys.argv[2] if len(sys.argv) > 2 else run["algo"]
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
w = g.get("w")
if algo == "sssp" and w is None:
    w = grgen.weights(g.m, 1, 64, seed=3)
with gr.GraphReduce(g.n, g.src, g.dst, w) as G:
    for prof in (False, True):
        for r in range(reps):
            t0 = time.perf_counter()
            st = G.run(algo, source=0, profile=prof)
            dt = (time.perf_counter() - t0) * 1e3
            print(f"cfg{cfg} {algo} profile={int(prof)} wall {dt:.2f} ms iters {st['iterations']} "
                  f"pull {st['pull_supersteps']} kernel_ms {[round(x, 3) for x in st['kernel_ms'][:2]]}", flush=True)
