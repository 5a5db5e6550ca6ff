"""Frontier programs under compute-sanitizer: BFS / SSSP / CC / tolerance PageRank on a
small R-MAT (and CC on its symmetrisation) through every loop driver and direction,
each result compared with the oracle."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import grgen
import oracle
import paper_conf_sc_senguptasas15_b200 as gr

g = grgen.rmat(12, 16, seed=7)
w = grgen.weights(g.m, 1, 64, seed=7)
sym_src = np.concatenate([g.src, g.dst]); sym_dst = np.concatenate([g.dst, g.src])
bad = 0
for algo, (s, d, ww) in (("bfs", (g.src, g.dst, None)), ("sssp", (g.src, g.dst, w)), ("cc", (sym_src, sym_dst, None))):
    og = oracle.OracleGraph(g.n, s, d, ww)
    ref, _, _ = og.run(algo, source=0)
    og.close()
    with gr.GraphReduce(g.n, s, d, ww) as G:
        for loop in ("auto", "device", "host"):
            for direction in ("auto", "push", "pull"):
                G.run(algo, source=0, loop=loop, direction=direction)
                ok = np.array_equal(G.values(algo), ref)
                bad += not ok
                print(algo, loop, direction, "ok" if ok else "MISMATCH", flush=True)
print("mismatches", bad)
