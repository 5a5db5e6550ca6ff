"""Pins for the oracle (SURVEY.md §8(c) "Pins").

Each check compares the oracle with something other than itself: textbook
algorithms from scipy / networkx, closed forms, a dense linear solve, and a
pure-Python set-based brute force of the BSP frontier semantics on tiny
graphs. A plausible mistake in the oracle (dropped term, wrong sign or index,
transposed operand, off-by-one iteration, non-BSP update) fails at least one.
"""
from __future__ import annotations

import collections
import heapq
import os

import networkx as nx
import numpy as np
import pytest
import scipy.sparse as sp
import scipy.sparse.csgraph as csg

import oracle
from oracle import INF

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ----------------------------------------------------------------- helpers
def rand_graph(rng, n, m, sym=False, wmax=None):
    src = rng.integers(0, n, m).astype(np.uint32)
    dst = rng.integers(0, n, m).astype(np.uint32)
    w = rng.integers(1, wmax + 1, m).astype(np.uint32) if wmax else None
    if sym:
        src, dst = np.concatenate([src, dst]), np.concatenate([dst, src])
        if w is not None:
            w = np.concatenate([w, w])
    return src, dst, w


def queue_bfs(n, src, dst, s):
    adj = collections.defaultdict(list)
    for a, b in zip(src.tolist(), dst.tolist()):
        adj[a].append(b)
    d = [INF] * n
    d[s] = 0
    q = collections.deque([s])
    while q:
        u = q.popleft()
        for x in adj[u]:
            if d[x] == INF:
                d[x] = d[u] + 1
                q.append(x)
    return np.array(d, np.uint32)


def heap_dijkstra(n, src, dst, w, s):
    adj = collections.defaultdict(list)
    for a, b, c in zip(src.tolist(), dst.tolist(), w.tolist()):
        adj[a].append((b, c))
    d = [INF] * n
    d[s] = 0
    h = [(0, s)]
    while h:
        du, u = heapq.heappop(h)
        if du > d[u]:
            continue
        for x, c in adj[u]:
            if du + c < d[x]:
                d[x] = du + c
                heapq.heappush(h, (d[x], x))
    return np.array(d, np.uint32)


def union_find_min_label(n, src, dst):
    p = list(range(n))

    def f(x):
        while p[x] != x:
            p[x] = p[p[x]]
            x = p[x]
        return x

    for a, b in zip(src.tolist(), dst.tolist()):
        ra, rb = f(a), f(b)
        if ra != rb:
            p[max(ra, rb)] = min(ra, rb)
    mn = {}
    for v in range(n):
        r = f(v)
        mn[r] = min(mn.get(r, v), v)
    return np.array([mn[f(v)] for v in range(n)], np.uint32)


def dense_pagerank_fixed_point(n, src, dst, d=0.85):
    """R* = (1-d)/n (I - d M^T)^-1 1 with M[u,v] = mult(u->v)/outdeg(u); dangling dropped."""
    M = np.zeros((n, n))
    for a, b in zip(src.tolist(), dst.tolist()):
        M[a, b] += 1.0
    out = M.sum(1)
    nz = out > 0
    M[nz] /= out[nz, None]
    return np.linalg.solve(np.eye(n) - d * M.T, np.full(n, (1 - d) / n))


def brute_trace(n, src, dst, w, algo, source=0, max_iters=0, d=0.85):
    """Pure-Python set-based BSP GAS."""
    ins = collections.defaultdict(list)
    outs = collections.defaultdict(list)
    for i, (a, b) in enumerate(zip(src.tolist(), dst.tolist())):
        c = int(w[i]) if w is not None else 1
        ins[b].append((a, c))
        outs[a].append(b)
    if algo == "pagerank":
        val = {v: 1.0 / n for v in range(n)}
        A = set(range(n))
    elif algo == "cc":
        val = {v: v for v in range(n)}
        A = set(range(n))
    else:
        val = {v: INF for v in range(n)}
        if algo == "bfs":
            A = {source}
        else:
            val[source] = 0
            A = set(outs[source])
    rows, t = [], 0
    while A and (max_iters == 0 or t < max_iters):
        new = {}
        gathered = 0
        for v in A:
            if algo == "bfs":
                new[v] = t if val[v] == INF else val[v]
                continue
            gathered += len(ins[v])
            if algo == "pagerank":
                acc = sum(val[u] / len(outs[u]) for u, _ in ins[v])
                new[v] = (1 - d) / n + d * acc
            elif algo == "cc":
                acc = min([val[u] for u, _ in ins[v]], default=INF)
                new[v] = min(acc, val[v])
            else:
                acc = min([min(val[u] + c, INF) if val[u] != INF else INF for u, c in ins[v]],
                          default=INF)
                new[v] = min(acc, val[v])
        C = set(A) if algo == "pagerank" else {v for v in A if new[v] != val[v]}
        val.update(new)
        if algo == "pagerank":
            rows.append((len(A), len(C), gathered, 0))
            A = set(range(n))
        else:
            rows.append((len(A), len(C), gathered, sum(len(outs[u]) for u in C)))
            A = {x for u in C for x in outs[u]}
        t += 1
    return val, np.array(rows, np.uint64).reshape(-1, 4), t


# ------------------------------------------------------------------- BFS
@pytest.mark.parametrize("seed", range(12))
def test_bfs_vs_queue_bfs_and_scipy(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(2, 80))
    src, dst, _ = rand_graph(rng, n, int(rng.integers(0, 4 * n)))
    s = int(rng.integers(0, n))
    vals, tr, it = oracle.run(n, src, dst, "bfs", source=s)
    np.testing.assert_array_equal(vals, queue_bfs(n, src, dst, s))
    A = sp.csr_matrix((np.ones(len(src)), (src, dst)), shape=(n, n))
    ref = csg.shortest_path(A, directed=True, unweighted=True, indices=s)
    ref = np.where(np.isinf(ref), INF, ref).astype(np.uint32)
    np.testing.assert_array_equal(vals, ref)


def test_bfs_lattice_closed_form():
    W, H = 13, 9
    e = []
    for r in range(H):
        for c in range(W):
            v = r * W + c
            if c + 1 < W:
                e += [(v, v + 1), (v + 1, v)]
            if r + 1 < H:
                e += [(v, v + W), (v + W, v)]
    src, dst = np.array(e, np.uint32).T
    vals, _, _ = oracle.run(W * H, src, dst, "bfs", source=0)
    rr, cc = np.divmod(np.arange(W * H), W)
    np.testing.assert_array_equal(vals, (rr + cc).astype(np.uint32))


def test_bfs_directed_cycle_trace_closed_form():
    n = 17
    src = np.arange(n, dtype=np.uint32)
    dst = ((src + 1) % n).astype(np.uint32)
    vals, tr, it = oracle.run(n, src, dst, "bfs", source=0)
    np.testing.assert_array_equal(vals, np.arange(n, dtype=np.uint32))
    # t < n: one vertex active and changed, one out-edge activated; t = n: vertex 0 re-activated, unchanged
    exp = [(1, 1, 0, 1)] * n + [(1, 0, 0, 0)]
    np.testing.assert_array_equal(tr, np.array(exp, np.uint64))
    assert it == n + 1


def test_bfs_vs_networkx_rmat():
    import grgen

    g = grgen.rmat(10, 8, seed=11)
    vals, _, _ = oracle.run(g.n, g.src, g.dst, "bfs", source=0)
    G = nx.DiGraph()
    G.add_nodes_from(range(g.n))
    G.add_edges_from(zip(g.src.tolist(), g.dst.tolist()))
    ref = np.full(g.n, INF, np.uint32)
    for v, dd in nx.single_source_shortest_path_length(G, 0).items():
        ref[v] = dd
    np.testing.assert_array_equal(vals, ref)


# ------------------------------------------------------------------ SSSP
@pytest.mark.parametrize("seed", range(12))
def test_sssp_vs_dijkstra_and_scipy(seed):
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(2, 70))
    src, dst, w = rand_graph(rng, n, int(rng.integers(0, 4 * n)), wmax=64)
    s = int(rng.integers(0, n))
    vals, _, _ = oracle.run(n, src, dst, "sssp", w=w, source=s)
    np.testing.assert_array_equal(vals, heap_dijkstra(n, src, dst, w, s))
    # scipy sums duplicate entries: reduce multi-edges to their minimum weight first
    best = {}
    for a, b, c in zip(src.tolist(), dst.tolist(), w.tolist()):
        if a != b:
            best[(a, b)] = min(best.get((a, b), c), c)
    if best:
        (ij, cw) = zip(*best.items())
        ii, jj = zip(*ij)
        A = sp.csr_matrix((np.array(cw, float), (ii, jj)), shape=(n, n))
    else:
        A = sp.csr_matrix((n, n))
    ref = csg.dijkstra(A, directed=True, indices=s)
    ref = np.where(np.isinf(ref), INF, ref).astype(np.uint32)
    np.testing.assert_array_equal(vals, ref)


def test_sssp_unit_weights_equals_bfs():
    # "BFS is essentially SSSP with equal edge weights"
    import grgen

    g = grgen.rmat(11, 8, seed=5)
    w = np.ones(g.m, np.uint32)
    b, _, _ = oracle.run(g.n, g.src, g.dst, "bfs", source=3)
    s, _, _ = oracle.run(g.n, g.src, g.dst, "sssp", w=w, source=3)
    np.testing.assert_array_equal(b, s)


def test_sssp_path_prefix_sums_and_lattice_manhattan():
    rng = np.random.default_rng(7)
    n = 40
    w = rng.integers(1, 65, n - 1).astype(np.uint32)
    src = np.arange(n - 1, dtype=np.uint32)
    dst = src + 1
    vals, tr, it = oracle.run(n, src, dst, "sssp", w=w, source=0)
    np.testing.assert_array_equal(vals, np.concatenate([[0], np.cumsum(w)]).astype(np.uint32))
    # path: exactly one vertex active and changed per superstep; A_0 = {1}
    assert it == n - 1
    np.testing.assert_array_equal(tr[:, :2], np.ones((n - 1, 2), np.uint64))
    import grgen

    g = grgen.grid_road(9, 7, p=1.0, wmax=1, seed=1)  # full lattice, unit weights
    vals, _, _ = oracle.run(g.n, g.src, g.dst, "sssp", w=g.w, source=0)
    rr, cc = np.divmod(np.arange(g.n), 9)
    np.testing.assert_array_equal(vals, (rr + cc).astype(np.uint32))


# -------------------------------------------------------------------- CC
@pytest.mark.parametrize("seed", range(12))
def test_cc_vs_union_find_and_scipy(seed):
    rng = np.random.default_rng(200 + seed)
    n = int(rng.integers(1, 90))
    src, dst, _ = rand_graph(rng, n, int(rng.integers(0, 2 * n)), sym=True)
    vals, _, _ = oracle.run(n, src, dst, "cc")
    np.testing.assert_array_equal(vals, union_find_min_label(n, src, dst))
    A = sp.csr_matrix((np.ones(len(src)), (src, dst)), shape=(n, n))
    k, lab = csg.connected_components(A, directed=False)
    assert len(np.unique(vals)) == k
    for c in range(k):
        members = np.nonzero(lab == c)[0]
        assert np.all(vals[members] == members.min())


def test_cc_disjoint_cycles_and_cliques():
    edges, expect, base = [], [], 0
    for kind, size in [("cycle", 5), ("clique", 4), ("cycle", 9), ("clique", 1), ("clique", 6)]:
        vs = list(range(base, base + size))
        if kind == "cycle" and size > 1:
            for i in range(size):
                a, b = vs[i], vs[(i + 1) % size]
                edges += [(a, b), (b, a)]
        else:
            for a in vs:
                for b in vs:
                    if a != b:
                        edges.append((a, b))
        expect += [base] * size
        base += size
    # relabel by a permutation so the min id is not always the first vertex
    perm = np.random.default_rng(3).permutation(base).astype(np.uint32)
    src, dst = (perm[np.array(edges, np.int64).T] if edges else np.zeros((2, 0), np.uint32))
    vals, _, _ = oracle.run(base, src, dst, "cc")
    exp = np.empty(base, np.uint32)
    blocks = np.array(expect)
    for b in np.unique(blocks):
        members = perm[blocks == b]
        exp[members] = members.min()
    np.testing.assert_array_equal(vals, exp)


# -------------------------------------------------------------------- PR
def test_pr_directed_cycle_uniform():
    n = 23
    src = np.arange(n, dtype=np.uint32)
    dst = ((src + 1) % n).astype(np.uint32)
    for iters in (1, 2, 30):
        vals, tr, it = oracle.run(n, src, dst, "pagerank", max_iters=iters)
        assert it == iters
        np.testing.assert_allclose(vals, 1.0 / n, rtol=0, atol=1e-15)
    np.testing.assert_array_equal(tr, np.tile(np.array([n, n, n, 0], np.uint64), (30, 1)))


def test_pr_symmetric_star_closed_form():
    k, d = 3, 0.85
    n = k + 1
    src = np.array([0] * k + list(range(1, n)), np.uint32)
    dst = np.array(list(range(1, n)) + [0] * k, np.uint32)
    vals, _, _ = oracle.run(n, src, dst, "pagerank", max_iters=200)
    leaf = (1 + d / k) / (n * (1 + d))
    hub = (1 - d) / n + d * k * leaf
    np.testing.assert_allclose(vals[1:], leaf, atol=1e-13)
    np.testing.assert_allclose(vals[0], hub, atol=1e-13)
    np.testing.assert_allclose([leaf, hub], [0.1734234234, 0.4797297297], atol=1e-10)


def test_pr_golden_example_dense_solve():
    # tests/golden/pr_example.txt: edges {0->1,0->2,1->2,2->0,2->3}, vertex 3 dangling
    path = os.path.join(GOLDEN, "pr_example.txt")
    rows = [ln.split() for ln in open(path) if ln.strip() and not ln.startswith("#")]
    edges = [(int(r[1]), int(r[2])) for r in rows if r[0] == "e"]
    golden = np.array([float(r[2]) for r in rows if r[0] == "r"])
    src, dst = np.array(edges, np.uint32).T
    vals, _, _ = oracle.run(4, src, dst, "pagerank", max_iters=200)
    np.testing.assert_allclose(vals, golden, atol=1e-8)
    np.testing.assert_allclose(vals, dense_pagerank_fixed_point(4, src, dst), atol=1e-12)
    v30, _, _ = oracle.run(4, src, dst, "pagerank", max_iters=30)
    np.testing.assert_allclose(v30, golden, atol=2e-6)


@pytest.mark.parametrize("seed", range(10))
def test_pr_fixed_point_dense_solve(seed):
    rng = np.random.default_rng(300 + seed)
    n = int(rng.integers(4, 9))
    src, dst, _ = rand_graph(rng, n, int(rng.integers(n, 4 * n)))
    vals, _, _ = oracle.run(n, src, dst, "pagerank", max_iters=200)
    np.testing.assert_allclose(vals, dense_pagerank_fixed_point(n, src, dst), atol=1e-12)


@pytest.mark.parametrize("seed", range(6))
def test_pr_30_iterations_matrix_power(seed):
    rng = np.random.default_rng(400 + seed)
    n = int(rng.integers(4, 30))
    src, dst, _ = rand_graph(rng, n, 3 * n)
    M = np.zeros((n, n))
    np.add.at(M, (src, dst), 1.0)
    out = M.sum(1)
    M[out > 0] /= out[out > 0, None]
    R = np.full(n, 1.0 / n)
    for _ in range(30):
        R = 0.15 / n + 0.85 * (M.T @ R)
    vals, _, _ = oracle.run(n, src, dst, "pagerank", max_iters=30)
    np.testing.assert_allclose(vals, R, atol=1e-15, rtol=1e-12)


@pytest.mark.parametrize("seed", range(5))
def test_pr_networkx_no_dangling(seed):
    rng = np.random.default_rng(500 + seed)
    n = 25
    src, dst, _ = rand_graph(rng, n, 4 * n)
    # give every vertex an out-edge (no dangling) — networkx then agrees exactly
    src = np.concatenate([src, np.arange(n, dtype=np.uint32)])
    dst = np.concatenate([dst, rng.integers(0, n, n).astype(np.uint32)])
    vals, _, _ = oracle.run(n, src, dst, "pagerank", max_iters=200)
    G = nx.MultiDiGraph()
    G.add_nodes_from(range(n))
    G.add_edges_from(zip(src.tolist(), dst.tolist()))
    ref = nx.pagerank(G, alpha=0.85, tol=1e-15, max_iter=1000)
    np.testing.assert_allclose(vals, [ref[v] for v in range(n)], atol=1e-12)
    # invariant: no dangling vertex => sum_v R_t = 1 at every t
    for iters in (1, 2, 7, 30):
        v, _, _ = oracle.run(n, src, dst, "pagerank", max_iters=iters)
        assert abs(v.sum() - 1.0) < 1e-12


# -------------------------------------------------- frontier-trace pins
@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc", "pagerank"])
@pytest.mark.parametrize("seed", range(8))
def test_trace_vs_bruteforce(algo, seed):
    rng = np.random.default_rng(600 + seed)
    n = int(rng.integers(2, 40))
    src, dst, w = rand_graph(rng, n, int(rng.integers(0, 3 * n)), sym=(algo == "cc"), wmax=64)
    s = int(rng.integers(0, n))
    mi = 7 if algo == "pagerank" else 0
    vals, tr, it = oracle.run(n, src, dst, algo, w=w if algo == "sssp" else None, source=s,
                              max_iters=mi)
    bv, btr, bit = brute_trace(n, src, dst, w if algo == "sssp" else None, algo, s, mi)
    assert it == bit
    np.testing.assert_array_equal(tr, btr)
    if algo == "pagerank":
        np.testing.assert_allclose(vals, [bv[v] for v in range(n)], atol=1e-15, rtol=1e-13)
    else:
        np.testing.assert_array_equal(vals, np.array([bv[v] for v in range(n)], np.uint32))


def test_oracle_rejects_bad_input():
    with pytest.raises(ValueError):
        oracle.OracleGraph(4, np.array([0, 5], np.uint32), np.array([1, 2], np.uint32))


# ------------------------------------------------- widest path (user program)
def maxmin_dijkstra(n, src, dst, w, s):
    """Textbook widest path: Dijkstra on the (max, min) semiring."""
    adj = collections.defaultdict(list)
    for a, b, c in zip(src.tolist(), dst.tolist(), w.tolist()):
        adj[a].append((b, c))
    width = [0] * n
    width[s] = INF
    h = [(-INF, s)]
    while h:
        negw, u = heapq.heappop(h)
        if -negw < width[u]:
            continue
        for x, c in adj[u]:
            cand = min(width[u], c)
            if cand > width[x]:
                width[x] = cand
                heapq.heappush(h, (-cand, x))
    return np.array(width, np.uint32)


@pytest.mark.parametrize("seed", range(10))
def test_widest_vs_maxmin_dijkstra(seed):
    rng = np.random.default_rng(700 + seed)
    n = int(rng.integers(2, 60))
    src, dst, w = rand_graph(rng, n, int(rng.integers(0, 4 * n)), wmax=64)
    s = int(rng.integers(0, n))
    vals, tr, _ = oracle.run(n, src, dst, "widest", w=w, source=s)
    np.testing.assert_array_equal(vals, maxmin_dijkstra(n, src, dst, w, s))


def test_widest_path_prefix_min():
    rng = np.random.default_rng(9)
    n = 30
    w = rng.integers(1, 65, n - 1).astype(np.uint32)
    src = np.arange(n - 1, dtype=np.uint32)
    vals, _, _ = oracle.run(n, src, src + 1, "widest", w=w, source=0)
    exp = np.concatenate([[INF], np.minimum.accumulate(w)]).astype(np.uint32)
    np.testing.assert_array_equal(vals, exp)


# ------------------------------------------- tolerance-driven PageRank (f2)
def _jacobi(n, src, dst, iters, d=0.85):
    M = np.zeros((n, n))
    np.add.at(M, (src, dst), 1.0)
    out = M.sum(1)
    M[out > 0] /= out[out > 0, None]
    R = np.full(n, 1.0 / n)
    for _ in range(iters):
        R = (1 - d) / n + d * (M.T @ R)
    return R


@pytest.mark.parametrize("seed", range(6))
def test_prdelta_tolerance0_is_the_jacobi_iteration(seed):
    """tolerance 0: a vertex is skipped only when none of its sources moved, so
    its recomputation would reproduce its value — 30 supersteps equal 30 Jacobi
    iterations of PageRank (fp64 matrix powers) up to fp32 rounding."""
    rng = np.random.default_rng(700 + seed)
    n = int(rng.integers(4, 40))
    src, dst, _ = rand_graph(rng, n, 3 * n)
    vals, tr, it = oracle.run(n, src, dst, "pagerank_delta", max_iters=30, tolerance=0.0)
    R = _jacobi(n, src, dst, it)
    assert vals.dtype == np.float32
    np.testing.assert_allclose(vals.astype(np.float64), R, atol=2e-7, rtol=2e-6)
    assert tr[0, 0] == n and tr[0, 2] == len(src)  # A_0 = V, every in-edge gathered


def test_prdelta_star_fixed_point_and_cycle():
    d, k = 0.85, 3
    n = k + 1
    src = np.array([0] * k + list(range(1, n)), np.uint32)
    dst = np.array(list(range(1, n)) + [0] * k, np.uint32)
    # tolerance 0 may cycle between neighbouring fp32 values forever (every
    # rounding is a "change"); a tolerance above one ulp terminates
    vals, _, it = oracle.run(n, src, dst, "pagerank_delta", max_iters=500, tolerance=1e-6)
    assert it < 500  # the frontier empties
    leaf = (1 + d / k) / (n * (1 + d))
    np.testing.assert_allclose(vals[1:], leaf, rtol=1e-5)
    np.testing.assert_allclose(vals[0], (1 - d) / n + d * k * leaf, rtol=1e-5)
    # directed cycle: R = 1/n is already the fixed point -> one superstep, nothing changes
    n = 31
    s = np.arange(n, dtype=np.uint32)
    vals, tr, it = oracle.run(n, s, (s + 1) % n, "pagerank_delta", tolerance=1e-3)
    np.testing.assert_allclose(vals, 1.0 / n, rtol=1e-6)
    assert it == 1 and tr[0, 1] == 0


@pytest.mark.parametrize("seed", range(6))
def test_prdelta_tolerance_bound_vs_dense_solve(seed):
    """With tolerance tau every vertex ends within tau/n (+ fp32 rounding) of its
    own update f_v(R), and f is a d-contraction in the L1 norm (the columns of
    the transition matrix sum to <= 1), so sum_v |R - R*| <= (tau + n*eps)/(1-d)
    with R* from a dense linear solve. Larger tau never needs more supersteps."""
    rng = np.random.default_rng(800 + seed)
    n = int(rng.integers(6, 60))
    src, dst, _ = rand_graph(rng, n, 4 * n)
    Rstar = dense_pagerank_fixed_point(n, src, dst)
    prev = None
    for tau in (0.0, 1e-6, 1e-4, 1e-2):
        vals, tr, it = oracle.run(n, src, dst, "pagerank_delta", max_iters=10000, tolerance=tau)
        assert it < 10000
        err = np.abs(vals.astype(np.float64) - Rstar).sum()
        assert err <= (tau + n * 2e-7) / (1 - 0.85), (tau, err)
        if prev is not None:
            assert it <= prev + 1
        prev = it
        # |C_t| <= |A_t|, and A_{t+1} is exactly the out-neighbourhood of C_t (brute force)
        assert np.all(tr[:, 1] <= tr[:, 0])
        assert tr[0, 0] == n


def test_prdelta_rejects_bad_parameters():
    src = np.array([0, 1], np.uint32)
    dst = np.array([1, 0], np.uint32)
    for kw in ({"damping": 0.0}, {"damping": 1.0}, {"tolerance": -1.0}):
        with pytest.raises(ValueError):
            oracle.run(2, src, dst, "pagerank_delta", **kw)


# ------------------------------------------------- scatter: SSSP by edge messages
# OR_SSSPMSG (oracle.h): mutable edge state (§2.1, §4.4).
# Pinned to the textbook heap Dijkstra (values) and, by the invariance argument
# of oracle.h (an unsent message could never lower its target), to the frontier
# trace of the plain SSSP program.
@pytest.mark.parametrize("seed", range(10))
def test_sssp_messages_vs_dijkstra(seed):
    rng = np.random.default_rng(700 + seed)
    n = int(rng.integers(2, 70))
    src, dst, w = rand_graph(rng, n, int(rng.integers(0, 4 * n)), wmax=64)
    s = int(rng.integers(0, n))
    vals, tr, it = oracle.run(n, src, dst, "sssp_msg", w=w, source=s)
    np.testing.assert_array_equal(vals, heap_dijkstra(n, src, dst, w, s))
    v2, tr2, it2 = oracle.run(n, src, dst, "sssp", w=w, source=s)
    np.testing.assert_array_equal(tr, tr2)
    assert it == it2


def test_sssp_messages_path_and_lattice():
    # a directed path 0 -> 1 -> ... -> k: prefix sums of the weights, one superstep per hop
    k = 40
    src = np.arange(k, dtype=np.uint32)
    dst = src + 1
    w = (np.arange(k, dtype=np.uint32) % 7) + 1
    vals, tr, it = oracle.run(k + 1, src, dst, "sssp_msg", w=w, source=0)
    np.testing.assert_array_equal(vals, np.concatenate([[0], np.cumsum(w)]).astype(np.uint32))
    assert it == k and np.all(tr[:, 1] == 1) and tr[-1, 3] == 0  # A_0 = {1}, ..., A_{k-1} = {k}


# ------------------- tolerance-driven PageRank: exact brute force of the rule
# DESIGN.md §2 / reading R17-R18 (Figs. 16-17): the
# specification restated with Python's unbounded integers and Fractions (no
# 64/128-bit arithmetic, no ldexp), as a set-based BSP superstep. The oracle's
# values AND its whole frontier trace — so prd_apply's change rule
# |R_new - R_old| > tolerance/n — must equal it exactly.
def _prd_brute(n, src, dst, tau, max_iters, d=0.85):
    from fractions import Fraction
    import math

    ins = collections.defaultdict(list)
    outs = collections.defaultdict(list)
    for a, b in zip(src.tolist(), dst.tolist()):
        ins[b].append(a)
        outs[a].append(b)
    f32 = lambda x: float(np.float32(x))  # round to nearest fp32
    q = math.floor(f32(d) * 2**20 + 0.5)  # round(d * 2^20) of the fp32 damping
    base = ((2**20 - q) * 2**42) // n  # fixed-point (1 - d)/n
    thr = f32(tau) / n

    def fix(r):  # floor(R * 2^62), exact
        return math.floor(Fraction(r) * 2**62)

    def to_f32(rfix):  # fp32(double(R_fix) * 2^-62): nearest double, then nearest fp32
        return f32(float(rfix) * 2.0**-62)

    val = {v: to_f32(2**62 // n) for v in range(n)}
    A, rows, t = set(range(n)), [], 0
    while A and t < max_iters:
        new, gathered = {}, 0
        for v in A:
            S = sum(fix(val[u]) // len(outs[u]) for u in ins[v])
            gathered += len(ins[v])
            new[v] = to_f32(base + (S * q) // 2**20)
        C = {v for v in A if abs(new[v] - val[v]) > thr}
        for v in C:
            val[v] = new[v]
        rows.append((len(A), len(C), gathered, sum(len(outs[u]) for u in C)))
        A = {x for u in C for x in outs[u]}
        t += 1
    return np.array([val[v] for v in range(n)], np.float32), np.array(rows, np.uint64).reshape(-1, 4), t


@pytest.mark.parametrize("tau", [0.0, 1e-6, 1e-3])
@pytest.mark.parametrize("seed", range(8))
def test_prdelta_values_and_trace_vs_exact_bruteforce(seed, tau):
    rng = np.random.default_rng(900 + seed)
    n = int(rng.integers(2, 48))
    src, dst, _ = rand_graph(rng, n, int(rng.integers(0, 4 * n)))
    if seed % 2:  # a hub with many in- and out-edges: large sums, many distinct n_u
        hub = rng.integers(0, n, 3 * n).astype(np.uint32)
        src = np.concatenate([src, hub, np.zeros(n, np.uint32)])
        dst = np.concatenate([dst, np.zeros(3 * n, np.uint32), np.arange(n, dtype=np.uint32)])
    mi = 60
    vals, tr, it = oracle.run(n, src, dst, "pagerank_delta", max_iters=mi, tolerance=tau)
    bv, btr, bit = _prd_brute(n, src, dst, tau, mi)
    assert it == bit
    np.testing.assert_array_equal(tr, btr)
    np.testing.assert_array_equal(vals.view(np.uint32), bv.view(np.uint32))
    if tau == 1e-3:  # the rule really skips: some superstep leaves an active vertex unchanged
        assert it < mi and np.any(tr[:, 1] < tr[:, 0]) or len(src) == 0


# --------------------------- heat diffusion with mutable edge state (OR_HEAT)
# PAPER.md §2.1 L68 ("Heat Simulation"), Scatter L66. Pinned to (a) the plain
# definition — the full fixed-point heat step T_{k+1}[x] = sum_{(u->x)}
# floor(T_k[u] (w+1) / 256) applied to EVERY vertex, no frontier, no edge
# state — so the frontier + scatter + edge-state machinery must reproduce it
# exactly; (b) the fp64 matrix power (W^T)^k T_0 within the floor-loss bound
# k*m in L1 (W^T has unit column sums, so it does not expand L1 errors);
# (c) heat conservation up to that loss.
def _heat_full(n, src, dst, w, s, iters):
    T = [0] * n
    T[s] = oracle.HEAT_H0
    seq = [list(T)]
    for _ in range(iters):
        N = [0] * n
        for a, b, c in zip(src.tolist(), dst.tolist(), w.tolist()):
            N[b] += T[a] * (c + 1) // 256
        T = N
        seq.append(list(T))
    return seq


def _heat_graph(rng, W, H):
    import grgen

    g = grgen.heat_grid(W, H, seed=int(rng.integers(1, 1000)))
    return g.n, g.src, g.dst, g.w


@pytest.mark.parametrize("seed", range(6))
def test_heat_vs_full_iteration_and_matrix_power(seed):
    rng = np.random.default_rng(1000 + seed)
    W, H = int(rng.integers(2, 9)), int(rng.integers(2, 9))
    n, src, dst, w = _heat_graph(rng, W, H)
    s = int(rng.integers(0, n))
    mi = int(rng.integers(1, 40))
    vals, tr, it = oracle.run(n, src, dst, "heat", w=w, source=s, max_iters=mi)
    seq = _heat_full(n, src, dst, w, s, it + 1)
    np.testing.assert_array_equal(vals, np.array(seq[it], np.uint32))
    if it < mi:  # the frontier emptied: a fixed point of the full step
        assert seq[it + 1] == seq[it]
    # (b) fp64 matrix power, (c) conservation
    Wm = np.zeros((n, n))
    np.add.at(Wm, (src, dst), (w.astype(np.float64) + 1) / 256)
    np.testing.assert_allclose(Wm.sum(1), 1.0)  # every vertex keeps or sends all its heat
    T0 = np.zeros(n)
    T0[s] = oracle.HEAT_H0
    exact = np.linalg.matrix_power(Wm.T, it) @ T0
    err = np.abs(vals.astype(np.float64) - exact).sum()
    assert err <= it * len(src) + 1e-3, (err, it * len(src))  # + fp64 rounding of the power
    assert oracle.HEAT_H0 - it * len(src) <= int(vals.astype(np.int64).sum()) <= oracle.HEAT_H0
    assert tr[0, 0] == len(set(dst[src == s].tolist()))  # A_0 = out-neighbours of the source


def test_heat_two_vertices_closed_form():
    # 0 <-> 1 with conductance w: each keeps (255 - (w+1) + 1)/256 and sends (w+1)/256
    w1 = 63  # (w+1)/256 = 1/4
    src = np.array([0, 1, 0, 1], np.uint32)
    dst = np.array([1, 0, 0, 1], np.uint32)
    w = np.array([w1, w1, 255 - (w1 + 1), 255 - (w1 + 1)], np.uint32)
    vals, tr, it = oracle.run(2, src, dst, "heat", w=w, source=0, max_iters=1)
    H0 = oracle.HEAT_H0
    np.testing.assert_array_equal(vals, [H0 * 3 // 4, H0 // 4])
    # T_k = H0/2 (1 +- (1/2)^k) exactly while the shares divide evenly
    vals, tr, it = oracle.run(2, src, dst, "heat", w=w, source=0, max_iters=10)
    np.testing.assert_array_equal(vals, [H0 // 2 + (H0 >> 11), H0 // 2 - (H0 >> 11)])
    assert it == 10 and np.all(tr[:, 1] == 2)


# ------------------------- detail columns of the trace: active shards and S_t
# per superstep, the number of shards holding an active
# vertex (what frontier skipping moves, §5.2) and the number of
# distinct sources the gather reads. Brute force: sets over the same BSP run.
@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc", "pagerank", "pagerank_delta"])
@pytest.mark.parametrize("seed", range(5))
def test_trace_detail_vs_bruteforce(algo, seed):
    rng = np.random.default_rng(1100 + seed)
    n = int(rng.integers(2, 60))
    src, dst, w = rand_graph(rng, n, int(rng.integers(0, 4 * n)), sym=(algo == "cc"), wmax=64)
    P = int(rng.integers(1, 6))
    bounds = np.unique(np.concatenate([[0, n], rng.integers(0, n, P - 1)])).astype(np.uint64)
    mi = 7 if algo.startswith("pagerank") else 0
    ww = w if algo == "sssp" else None
    g = oracle.OracleGraph(n, src, dst, ww)
    vals, tr, det, it = g.run_detail(algo, shard_bounds=bounds, source=0, max_iters=mi)
    v2, tr2, it2 = g.run(algo, source=0, max_iters=mi)
    g.close()
    np.testing.assert_array_equal(tr, tr2)  # the detail run is the same run
    ins = collections.defaultdict(list)
    outs = collections.defaultdict(list)
    for a, b in zip(src.tolist(), dst.tolist()):
        ins[b].append(a)
        outs[a].append(b)
    # replay the frontier from the trace's own activation rule (brute force of A_t)
    if algo == "bfs":
        A = {0}
    elif algo in ("sssp",):
        A = set(outs[0])
    else:
        A = set(range(n))
    shard = lambda v: int(np.searchsorted(bounds, v, side="right")) - 1
    for t in range(it):
        exp_shards = len({shard(v) for v in A})
        exp_src = 0 if algo == "bfs" else len({u for v in A for u in ins[v]})
        assert det[t, 0] == exp_shards, (t, det[t], exp_shards)
        assert det[t, 1] == exp_src, (t, det[t], exp_src)
        assert tr[t, 0] == len(A)
        if t + 1 < it:
            if algo == "pagerank":
                A = set(range(n))
            else:  # A_{t+1} from the changed set of t: recover C_t by re-running t+1 supersteps
                vv, trk, _ = oracle.run(n, src, dst, algo, w=ww, source=0, max_iters=t + 1)
                vp, _, _ = oracle.run(n, src, dst, algo, w=ww, source=0, max_iters=t) if t > 0 else (None, None, None)
                if t == 0:
                    if algo == "bfs":
                        prev = np.full(n, INF, np.uint32)
                    elif algo == "sssp":
                        prev = np.full(n, INF, np.uint32)
                        prev[0] = 0
                    elif algo == "cc":
                        prev = np.arange(n, dtype=np.uint32)
                    else:
                        prev = None
                else:
                    prev = vp
                if prev is None:  # pagerank_delta at t = 0: R_0 = fp32(floor(2^62/n) 2^-62)
                    r0 = np.float32(float((1 << 62) // n) * 2.0 ** -62)
                    prev = np.full(n, r0, np.float32)
                C = set(np.nonzero(vv != prev)[0].tolist())
                A = {x for u in C for x in outs[u]}
