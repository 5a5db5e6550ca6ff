"""T0: generator sanity — exact sizes, determinism across thread
counts (counter-based RNG), shape statistics, grid connectivity."""
import numpy as np
import scipy.sparse as sp
import scipy.sparse.csgraph as csg

import grgen


def test_rmat_exact_size_and_thread_independence():
    g1 = grgen.rmat(12, 16, seed=9)
    assert g1.m == 16 << 12 and g1.n == 4096
    old = grgen.THREADS
    try:
        grgen.THREADS = 1
        g2 = grgen.rmat(12, 16, seed=9)
    finally:
        grgen.THREADS = old
    np.testing.assert_array_equal(g1.src, g2.src)
    np.testing.assert_array_equal(g1.dst, g2.dst)
    assert g1.src.max() < 4096 and g1.dst.max() < 4096
    # R-MAT skew: vertex 0 is the hub (no permutation)
    assert np.bincount(g1.dst, minlength=4096).argmax() == 0
    g3 = grgen.rmat(12, 16, seed=10)
    assert not np.array_equal(g1.src, g3.src)


def test_grid_connected_symmetric_weighted():
    g = grgen.grid_road(64, 48, p=0.58, wmax=64, seed=3)
    assert g.m % 2 == 0
    # both directions present with equal weights
    np.testing.assert_array_equal(g.src[0::2], g.dst[1::2])
    np.testing.assert_array_equal(g.w[0::2], g.w[1::2])
    assert g.w.min() >= 1 and g.w.max() <= 64
    A = sp.csr_matrix((np.ones(g.m), (g.src, g.dst)), shape=(g.n, g.n))
    k, _ = csg.connected_components(A, directed=False)
    assert k == 1
    assert 2.0 < g.m / g.n < 3.0  # road-like average degree (2.41)
    # lattice edges only: |dx| + |dy| == 1
    r1, c1 = np.divmod(g.src.astype(np.int64), 64)
    r2, c2 = np.divmod(g.dst.astype(np.int64), 64)
    assert np.all(np.abs(r1 - r2) + np.abs(c1 - c2) == 1)


def test_web_symmetric_powerlaw():
    g = grgen.web(50_000, seed=4)
    assert np.all(g.src != g.dst)
    np.testing.assert_array_equal(g.src[0::2], g.dst[1::2])
    mean = g.m / g.n
    assert 13.0 < mean < 19.0  # ~16 after symmetrization (2 x 8)
    deg = np.bincount(g.dst, minlength=g.n)
    assert deg.max() > 50 * mean  # heavy tail
