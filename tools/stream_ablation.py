"""Streamed-mode ablations on B200 (Fig. 15 frontier skipping, SURVEY
§8(f) f1 in-place reads): R-MAT ef16 forced-streamed, BFS from 0 and PageRank
(3 iterations), under whole-shard DMA with/without frontier skipping and the
zero-copy policies."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import grgen
import paper_conf_sc_senguptasas15_b200 as gr

scale = int(sys.argv[1]) if len(sys.argv) > 1 else 24
g = grgen.rmat(scale, 16, seed=5)
print(f"# R-MAT s{scale} ef16: n={g.n} m={g.m}, streamed, shard_edges=2^24", flush=True)
cases = [("dma, no skipping", -1, "1"), ("dma + skipping", -1, "0"), ("auto (f1) + skipping", 0, "0"),
         ("zero-copy always", 1, "0")]
if os.environ.get("ZC_SWEEP"):
    cases = [(f"auto, GR_ZC_DIV={d}", 0, "0", d) for d in (4, 8, 16, 32, 64, 128)]
with gr.GraphReduce(g.n, g.src, g.dst, mode="streamed", shard_edges=1 << 24) as G:
    print(f"# shards {G.info()['num_shards']}", flush=True)
    ref = {}
    for algo, kw in (("bfs", {}), ("pagerank", {"max_iters": 3})):
        for name, zc, noskip, *div in cases:
            os.environ["GR_STREAM_NO_SKIP"] = noskip
            if div:
                os.environ["GR_ZC_DIV"] = str(div[0])
            best, st = 1e9, None
            for _ in range(2):
                st = G.run(algo, zero_copy=zc, **kw)
                best = min(best, st["seconds"])
            v = G.values(algo)
            if algo not in ref:
                ref[algo] = v
            same = np.array_equal(v, ref[algo]) if algo == "bfs" else float(np.abs(v - ref[algo]).max())
            print(f"{algo:8s} {name:24s} {best * 1e3:9.1f} ms  h2d {st['bytes_h2d'] / 1e9:7.2f} GB "
                  f"(in place {st['bytes_h2d_zero_copy'] / 1e9:6.2f} GB, {st['zero_copy_phases']} phases)  "
                  f"iters {st['iterations']}  same={same}", flush=True)
