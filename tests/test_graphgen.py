"""Input generators (shared by oracle and CUDA tests): structure checks, CPU only."""
import numpy as np
import pytest

import graphgen


def _check_csr(g, allow_loops=False):
    o, c, w = g.offsets, g.col, g.w
    assert o[0] == 0 and (np.diff(o) >= 0).all() and o[-1] == c.shape[0] == w.shape[0]
    assert c.size == 0 or (c.min() >= 0 and c.max() < g.n)
    u = np.repeat(np.arange(g.n, dtype=np.int64), np.diff(o))
    if not allow_loops:
        assert not (u == c).any()
    # rows strictly increasing (sorted, deduplicated)
    same_row = u[1:] == u[:-1]
    assert (c[1:][same_row] > c[:-1][same_row]).all()
    # symmetric with equal weights
    a = np.lexsort((c, u)); b = np.lexsort((u, c))
    assert (u[a] == c[b]).all() and (c[a] == u[b]).all() and (w[a] == w[b]).all()
    assert np.isfinite(w).all() and (w > 0).all() and (w <= 1).all()


@pytest.mark.parametrize("maker", [
    lambda: graphgen.er(4096, 16.0, seed=2),
    lambda: graphgen.rmat(12, 16, seed=2),
    lambda: graphgen.mesh(37, seed=2),
    lambda: graphgen.mesh(40, keep=0.6, seed=2),
    lambda: graphgen.mesh(33, seed=2, weights="gradient"),
    lambda: graphgen.rmat(10, 8, seed=2, weights="paper"),
])
def test_generators_symmetric_simple(maker):
    _check_csr(maker())


def test_mesh_closed_form():
    side = 50
    g = graphgen.mesh(side)
    assert g.m_u == 2 * side * (side - 1)
    d = g.degrees().reshape(side, side)
    assert d[0, 0] == 2 and d[0, 5] == 3 and d[5, 5] == 4


def test_deterministic_across_threads():
    t0 = graphgen.set_threads(1)
    a = graphgen.rmat(13, 16, seed=9)
    graphgen.set_threads(max(t0, 4))
    b = graphgen.rmat(13, 16, seed=9)
    graphgen.set_threads(t0)
    assert np.array_equal(a.offsets, b.offsets) and np.array_equal(a.col, b.col)
    assert np.array_equal(a.w, b.w)


def test_weight_modes():
    g = graphgen.er(2000, 8.0, seed=1, weights="paper")
    q = np.round(g.w.astype(np.float64) * 1000)
    assert np.allclose(q / 1000, g.w, atol=1e-7) and q.min() >= 1 and q.max() <= 1000
    g = graphgen.er(2000, 8.0, seed=1, weights="ones")
    assert (g.w == 1).all()
    g = graphgen.er(2000, 8.0, seed=1)
    k = g.w.astype(np.float64) * 2 ** 24
    assert (k == np.round(k)).all() and k.min() >= 1 and k.max() <= 2 ** 24


def test_rmat_power_law_shape():
    g = graphgen.rmat(16, 16, seed=1)
    d = g.degrees()
    assert 0.85 * 16 * 2 * 2 ** 16 < g.m <= 16 * 2 * 2 ** 16   # dedup keeps most edges
    assert d.max() > 50 * d.mean()                           # hubs
    assert (d == 0).mean() > 0.1                             # many isolated vertices
