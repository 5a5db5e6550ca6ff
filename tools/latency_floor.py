"""Per-superstep latency floor: a path graph (one active vertex per superstep)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sc_senguptasas15_b200 as gr

n = 20000
a = np.arange(n - 1, dtype=np.uint32)
src = np.concatenate([a, a + 1]); dst = np.concatenate([a + 1, a]); w = np.ones(len(src), np.uint32)
cta = os.environ.get("GR_PERSIST_CTAS_PER_SM", "4")
with gr.GraphReduce(n, src, dst, w) as G:
    s = torch.cuda.current_stream()
    for algo in ("bfs", "sssp"):
        for loop in ("auto", "device"):
            for prof in (False, True):
                best = 1e9
                for _ in range(3):
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(s)
                    st = G.run(algo, source=0, stream=s.cuda_stream, profile=prof, loop=loop)
                    e1.record(s)
                    torch.cuda.synchronize()
                    best = min(best, e0.elapsed_time(e1))
                it = st["iterations"]
                print(f"ctas/SM={cta} {algo:5s} {loop:7s} profile={prof!s:5s} {1e3 * best / it:7.2f} us/superstep"
                      f"  phases {1e3 * st['kernel_ms'][0] / it:6.2f} {1e3 * st['kernel_ms'][1] / it:6.2f}", flush=True)
