"""Where the cfg1 BFS run time goes: event span of gr_run vs host wall vs the persistent kernel's own clock."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import grgen
import paper_conf_sc_senguptasas15_b200 as gr

g, run = grgen.config(1)
scratch = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
with gr.GraphReduce(g.n, g.src, g.dst, None) as G:
    s = torch.cuda.current_stream()
    for flush in (False, True):
        for prof in (False, True):
            ev, wall, kern = [], [], []
            for i in range(23):
                if flush:
                    scratch.fill_(1)
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                t0 = time.perf_counter()
                e0.record(s)
                st = G.run("bfs", source=0, stream=s.cuda_stream, profile=prof)
                e1.record(s)
                t1 = time.perf_counter()
                torch.cuda.synchronize()
                if i >= 3:
                    ev.append(e0.elapsed_time(e1)); wall.append((t1 - t0) * 1e3); kern.append(st["kernel_ms"][1])
            print(f"flush={flush!s:5s} profile={prof!s:5s} event {np.median(ev):.4f} ms  host wall {np.median(wall):.4f} ms"
                  f"  bfs phase {np.median(kern):.4f} ms", flush=True)
