"""One frontier run of a BASELINE config (for ncu captures): python tools/run_once.py CONFIG ALGO LOOP [DIRECTION]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import grgen  # noqa: E402
import paper_conf_sc_senguptasas15_b200 as gr  # noqa: E402

cfg, algo, loop = int(sys.argv[1]), sys.argv[2], sys.argv[3]
direction = sys.argv[4] if len(sys.argv) > 4 else "auto"
g, run = grgen.config(cfg)
w = g.get("w")
if algo == "sssp" and w is None:
    w = grgen.weights(g.m, 1, 64, seed=3)
with gr.GraphReduce(g.n, g.src, g.dst, w) as G:
    st = G.run(algo, source=0, loop=loop, direction=direction)
    print(cfg, algo, loop, st["iterations"], st["pull_supersteps"])
