"""Cost of per-phase kernel timing (profile=True) on the frontier loops: cfg3 SSSP and cfg4 CC."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import grgen
import paper_conf_sc_senguptasas15_b200 as gr

for cfg in (3, 4, 1):
    g, run = grgen.config(cfg)
    w = g.get("w")
    if run["algo"] == "sssp" and w is None:
        w = grgen.weights(g.m, 1, 64, seed=cfg)
    with gr.GraphReduce(g.n, g.src, g.dst, w) as G:
        s = torch.cuda.current_stream()
        for loop in ("auto", "device"):
            for prof in (False, True, False, True):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                st = G.run(run["algo"], source=run.get("source", 0), stream=s.cuda_stream, profile=prof, loop=loop)
                e1.record(s)
                torch.cuda.synchronize()
                print(f"cfg{cfg} {loop:7s} profile={prof!s:5s} {e0.elapsed_time(e1):9.3f} ms  iters {st['iterations']}"
                      f"  kernel_ms {st['kernel_ms'][0]:.3f} {st['kernel_ms'][1]:.3f}", flush=True)
