"""Experiment: PageRank iteration time on cfg2 with the generator's ids vs
degree-sorted ids (descending out-degree), and a random permutation."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import grgen
import paper_conf_sc_senguptasas15_b200 as gr

g = grgen.rmat(22, 16, seed=2)
n = g.n
outdeg = np.bincount(g.src, minlength=n)
indeg = np.bincount(g.dst, minlength=n)
rng = np.random.default_rng(0)
perms = {
    "identity": np.arange(n, dtype=np.uint32),
    "by_outdeg": np.argsort(-outdeg, kind="stable").astype(np.uint32),
    "by_in+out": np.argsort(-(outdeg + indeg), kind="stable").astype(np.uint32),
    "random": rng.permutation(n).astype(np.uint32),
}
for name, order in perms.items():
    newid = np.empty(n, np.uint32)
    newid[order] = np.arange(n, dtype=np.uint32)
    src, dst = newid[g.src], newid[g.dst]
    for kern in ("seg", "warphot"):
        os.environ["GR_PR_KERNEL"] = kern
        with gr.GraphReduce(n, src, dst) as G:
            s = torch.cuda.current_stream()
            for _ in range(3):
                G.run("pagerank", stream=s.cuda_stream)
            best = 1e9
            for _ in range(5):
                st = G.run("pagerank", stream=s.cuda_stream, profile=True)
                best = min(best, st["kernel_ms"][0] / 30)
            print(f"{name:10s} {kern:8s} gather {1e3 * best:7.1f} us/iter", flush=True)
