"""Pins for the SSSP oracle (oracle/oracle.c 4b; NEXT row 4): weighted
Floyd-Warshall brute force, scipy.sparse.csgraph.dijkstra, and unit weights,
where distances are BFS levels (closed form on grids and trees)."""
import numpy as np
import pytest

import oracle
from inputs import csr_from_adjacency, edge_weights, grid_csr, kronecker_csr, tree4_csr


def weighted_fw(n, row_ptr, col, w):
    inf = np.iinfo(np.int64).max // 4
    d = np.full((n, n), inf, dtype=np.int64)
    for u in range(n):
        for e in range(row_ptr[u], row_ptr[u + 1]):
            d[u, col[e]] = min(d[u, col[e]], int(w[e]))
    np.fill_diagonal(d, 0)
    for k in range(n):
        d = np.minimum(d, d[:, k:k + 1] + d[k:k + 1, :])
    return d, inf


def brute_parent(n, row_ptr, col, w, dist, src):
    par = np.full(n, -1, dtype=np.int32)
    par[src] = src
    for u in range(n):
        if dist[u] == oracle.UNREACHED_DIST:
            continue
        for e in range(row_ptr[u], row_ptr[u + 1]):
            v = col[e]
            if v != src and int(dist[u]) + int(w[e]) == int(dist[v]):
                par[v] = u if par[v] < 0 else min(par[v], u)
    return par


@pytest.mark.parametrize("n,p,wmax,seed", [(12, 0.3, 5, 0), (30, 0.15, 20, 1), (48, 0.08, 255, 2),
                                           (40, 0.3, 1, 3)])
def test_sssp_vs_weighted_floyd_warshall(n, p, wmax, seed):
    rng = np.random.default_rng(seed)
    a = (rng.random((n, n)) < p).astype(np.int8)
    a = np.triu(a, 1)
    g = csr_from_adjacency(a + a.T)
    w = edge_weights(g.row_ptr, g.col, seed, wmax)
    d, inf = weighted_fw(n, g.row_ptr, g.col, w)
    for src in range(n):
        dist, parent, reached = oracle.sssp(g.row_ptr, g.col, w, src)
        exp = np.where(d[src] >= inf, oracle.UNREACHED_DIST, d[src]).astype(np.uint32)
        np.testing.assert_array_equal(dist, exp)
        np.testing.assert_array_equal(parent, brute_parent(n, g.row_ptr, g.col, w, dist, src))
        assert reached == int((d[src] < inf).sum())


def test_weights_symmetric_and_in_range():
    g = kronecker_csr(10, 16, 1)
    w = edge_weights(g.row_ptr, g.col, 7, 100)
    assert w.min() >= 1 and w.max() <= 100
    rows = np.repeat(np.arange(g.n_vertices), np.diff(g.row_ptr))
    key = dict(zip(zip(rows.tolist(), g.col.tolist()), w.tolist()))
    assert all(key[(v, u)] == x for (u, v), x in key.items())


def test_scipy_dijkstra_cross_check():
    sp = pytest.importorskip("scipy.sparse")
    csg = pytest.importorskip("scipy.sparse.csgraph")
    g = kronecker_csr(12, 16, 3)
    w = edge_weights(g.row_ptr, g.col, 5, 255)
    m = sp.csr_matrix((w.astype(np.float64), g.col, g.row_ptr), shape=(g.n_vertices,) * 2)
    srcs = [int(np.argmax(g.degrees())), int(np.flatnonzero(g.degrees() > 0)[3])]
    d = csg.dijkstra(m, directed=True, indices=srcs)
    for k, s in enumerate(srcs):
        dist, parent, _ = oracle.sssp(g.row_ptr, g.col, w, s)
        exp = np.where(np.isinf(d[k]), oracle.UNREACHED_DIST, d[k]).astype(np.uint32)
        np.testing.assert_array_equal(dist, exp)
        r = (dist != oracle.UNREACHED_DIST) & (np.arange(g.n_vertices) != s)
        assert np.all(dist[parent[r]] < dist[r])  # weights >= 1: a proper tree


@pytest.mark.parametrize("make", [lambda: grid_csr(40, 23), lambda: tree4_csr(5000)])
def test_unit_weights_are_bfs_levels(make):
    g = make()
    w = np.ones(g.nnz, dtype=np.int32)
    for src in (0, g.n_vertices // 3):
        dist, parent, _ = oracle.sssp(g.row_ptr, g.col, w, src)
        level, lpar, _ = oracle.bfs(g.row_ptr, g.col, src)
        np.testing.assert_array_equal(dist.astype(np.int64), np.where(level < 0, oracle.UNREACHED_DIST, level))
        np.testing.assert_array_equal(parent, lpar)  # same min-id rule
