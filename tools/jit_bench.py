"""a run-time compiled program (gr_program_compile, NVRTC) vs
the same program built into the library, on a BASELINE config's graph: the
kernels are the same templates, so time per run must match. Prints one JSON
line per program with compile time, ms/run and GTEPS (edges traversed)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import grgen  # noqa: E402
import paper_conf_sc_senguptasas15_b200 as gr  # noqa: E402
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
from test_gpu_parity import JIT_CC64, JIT_SSSP  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 3
g, run = grgen.config(cfg)
w = g.get("w")
algo = run["algo"]
if algo == "sssp" and w is None:
    w = grgen.weights(g.m, 1, 64, seed=cfg)
t = time.perf_counter()
src, name = (JIT_SSSP, "JitSSSP") if algo == "sssp" else (JIT_CC64, "JitCC64")
cid = gr.gr_program_compile(src, name)
t_compile = time.perf_counter() - t
stream = torch.cuda.current_stream()
with gr.GraphReduce(g.n, g.src, g.dst, w) as G:
    ref = None
    for label, kw in (("built-in", dict(algo=algo)), ("run-time (NVRTC)", dict(algo="custom", custom_id=cid))):
        a = kw.pop("algo")
        for _ in range(2):
            G.run(a, source=0, stream=stream.cuda_stream, **kw)
        ms = []
        for _ in range(3):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            st = G.run(a, source=0, stream=stream.cuda_stream, **kw)
            e1.record(stream)
            torch.cuda.synchronize()
            ms.append(e0.elapsed_time(e1))
        vals = G.values()
        if ref is None:
            ref = vals
        edges = st["edges_gathered"] + st["edges_scattered"] if algo != "cc" else g.m
        print(json.dumps({"config": cfg, "program": f"{algo} {label}", "ms_per_run": round(float(np.median(ms)), 3),
                          "GTEPS": round(edges / (np.median(ms) * 1e-3) / 1e9, 3), "iterations": st["iterations"],
                          "identical_to_builtin": bool(np.array_equal(vals, ref)),
                          "compile_s": round(t_compile, 2) if "NVRTC" in label else None}), flush=True)
