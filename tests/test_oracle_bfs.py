"""Pins for the BFS oracle (oracle/oracle.c sections 1-4).

Each pin is independent of the oracle's own code: brute-force all-pairs
distances (Floyd-Warshall written here in numpy), exhaustive enumeration of
every labelled graph on 5 vertices, closed forms (path, star, complete graph,
disconnected parts, 4096-style grids, the 4-ary heap tree of PAPER.md:301)
and a library routine (scipy.sparse.csgraph.shortest_path). A dropped term,
wrong sign, off-by-one level or transposed operand in the oracle fails at
least one of these.
"""
import itertools

import numpy as np
import pytest

import oracle
from inputs import csr_from_adjacency, edges_to_csr, grid_csr, kronecker_csr, tree4_csr


def floyd_warshall(adj: np.ndarray) -> np.ndarray:
    n = adj.shape[0]
    inf = np.iinfo(np.int64).max // 4
    d = np.full((n, n), inf, dtype=np.int64)
    d[adj.astype(bool)] = 1
    np.fill_diagonal(d, 0)
    for k in range(n):
        d = np.minimum(d, d[:, k:k + 1] + d[k:k + 1, :])
    d[d >= inf] = -1
    return d


def brute_min_id_parent(adj: np.ndarray, dist_row: np.ndarray, root: int) -> np.ndarray:
    n = adj.shape[0]
    par = np.full(n, -1, dtype=np.int32)
    for v in range(n):
        if dist_row[v] < 0:
            continue
        if v == root:
            par[v] = root
            continue
        cands = [u for u in range(n) if adj[v, u] and u != v and dist_row[u] == dist_row[v] - 1]
        par[v] = min(cands)
    return par


def random_adj(n, p, rng):
    a = (rng.random((n, n)) < p).astype(np.int8)
    a = np.triu(a, 1)
    return a + a.T


@pytest.mark.parametrize("n,p,seed", [(8, 0.3, 0), (17, 0.15, 1), (33, 0.08, 2), (64, 0.05, 3),
                                      (64, 0.02, 4), (40, 0.5, 5)])
def test_levels_and_parents_vs_floyd_warshall(n, p, seed):
    rng = np.random.default_rng(seed)
    adj = random_adj(n, p, rng)
    g = csr_from_adjacency(adj)
    d = floyd_warshall(adj)
    for root in range(n):
        level, parent, info = oracle.bfs(g.row_ptr, g.col, root)
        np.testing.assert_array_equal(level, d[root].astype(np.int32))
        np.testing.assert_array_equal(parent, brute_min_id_parent(adj, d[root], root))
        assert info["reached"] == int((d[root] >= 0).sum())


def test_exhaustive_5_vertex_graphs():
    n = 5
    pairs = list(itertools.combinations(range(n), 2))
    assert len(pairs) == 10
    for mask in range(1 << len(pairs)):
        adj = np.zeros((n, n), dtype=np.int8)
        for k, (i, j) in enumerate(pairs):
            if mask >> k & 1:
                adj[i, j] = adj[j, i] = 1
        g = csr_from_adjacency(adj)
        d = floyd_warshall(adj)
        for root in range(n):
            level, parent, _ = oracle.bfs(g.row_ptr, g.col, root)
            assert np.array_equal(level, d[root]), (mask, root)
            assert np.array_equal(parent, brute_min_id_parent(adj, d[root], root)), (mask, root)


def test_closed_form_path_star_complete_disconnected():
    n = 50
    # path 0-1-...-49, root 17: level = |v - 17|, min-id parent = v-1 (v>17) / v+1 (v<17)
    g = edges_to_csr(np.arange(n - 1), np.arange(1, n), n)
    level, parent, _ = oracle.bfs(g.row_ptr, g.col, 17)
    v = np.arange(n)
    np.testing.assert_array_equal(level, np.abs(v - 17))
    exp_par = np.where(v > 17, v - 1, v + 1)
    exp_par[17] = 17
    np.testing.assert_array_equal(parent, exp_par)
    # star centred at 0, root at leaf 5: levels 1 (centre), 0 (root), 2 (others)
    g = edges_to_csr(np.zeros(n - 1, dtype=np.int64), np.arange(1, n), n)
    level, parent, _ = oracle.bfs(g.row_ptr, g.col, 5)
    exp = np.full(n, 2)
    exp[0], exp[5] = 1, 0
    np.testing.assert_array_equal(level, exp)
    assert parent[0] == 5 and parent[5] == 5 and np.all(np.delete(parent, [0, 5]) == 0)
    # complete graph K_n: all level 1, parent root
    adj = np.ones((n, n), dtype=np.int8) - np.eye(n, dtype=np.int8)
    g = csr_from_adjacency(adj)
    level, parent, _ = oracle.bfs(g.row_ptr, g.col, 9)
    assert level[9] == 0 and np.all(np.delete(level, 9) == 1) and np.all(parent == 9)
    # two components: 0..9 path, 10..19 path -> the other half unreachable
    s = np.concatenate([np.arange(9), np.arange(10, 19)])
    g = edges_to_csr(s, s + 1, 20)
    level, parent, info = oracle.bfs(g.row_ptr, g.col, 3)
    assert np.all(level[10:] == -1) and np.all(parent[10:] == -1) and info["reached"] == 10


@pytest.mark.parametrize("rows,cols", [(1, 1), (1, 7), (5, 1), (37, 53), (256, 256)])
def test_closed_form_grid(rows, cols):
    g = grid_csr(rows, cols)
    level, parent, info = oracle.bfs(g.row_ptr, g.col, 0)
    r, c = np.divmod(np.arange(rows * cols), cols)
    np.testing.assert_array_equal(level, r + c)
    v = np.arange(rows * cols)
    exp = np.where(r > 0, v - cols, v - 1)
    exp[0] = 0
    np.testing.assert_array_equal(parent, exp)
    assert info["traversed_edges"] == rows * (cols - 1) + cols * (rows - 1)


@pytest.mark.parametrize("n", [1, 2, 5, 21, 1000, 1 << 16])
def test_closed_form_4ary_heap_tree(n):
    g = tree4_csr(n)
    level, parent, info = oracle.bfs(g.row_ptr, g.col, 0)
    i = np.arange(n, dtype=np.int64)
    # level(i) = k iff 4**k <= 3i+1 < 4**(k+1)
    exp = np.zeros(n, dtype=np.int64)
    x = 3 * i + 1
    k = 0
    while (4 ** (k + 1)) <= x.max():
        k += 1
        exp[x >= 4 ** k] = k
    np.testing.assert_array_equal(level, exp)
    exp_par = np.where(i > 0, (i - 1) // 4, 0)
    np.testing.assert_array_equal(parent, exp_par)
    assert info["traversed_edges"] == n - 1


@pytest.mark.parametrize("scale,seed", [(10, 1), (12, 7)])
def test_scipy_cross_check_kronecker(scale, seed):
    sp = pytest.importorskip("scipy.sparse")
    csg = pytest.importorskip("scipy.sparse.csgraph")
    g = kronecker_csr(scale, 16, seed)
    n = g.n_vertices
    m = sp.csr_matrix((np.ones(g.nnz), g.col, g.row_ptr), shape=(n, n))
    deg = g.degrees()
    roots = [int(np.argmax(deg)), int(np.flatnonzero(deg > 0)[0]), int(np.flatnonzero(deg == 0)[0])]
    d = csg.shortest_path(m, unweighted=True, directed=False, indices=roots)
    for k, root in enumerate(roots):
        level, parent, info = oracle.bfs(g.row_ptr, g.col, root)
        exp = np.where(np.isinf(d[k]), -1, d[k]).astype(np.int32)
        np.testing.assert_array_equal(level, exp)
        assert oracle.validate_tree(g.row_ptr, g.col, root, level, parent) == (0, -1)
        assert info["traversed_edges"] == int(deg[exp >= 0].sum()) // 2


def test_validator_rejects_mutations():
    g = kronecker_csr(10, 16, 1)
    deg = g.degrees()
    root = int(np.argmax(deg))
    level, parent, _ = oracle.bfs(g.row_ptr, g.col, root)
    assert oracle.validate_tree(g.row_ptr, g.col, root, level, parent)[0] == 0
    reached = np.flatnonzero((level > 1))
    v = int(reached[0])

    p = parent.copy(); p[root] = v
    assert oracle.validate_tree(g.row_ptr, g.col, root, level, p)[0] == 1
    lv = level.copy(); lv[v] = -1
    assert oracle.validate_tree(g.row_ptr, g.col, root, lv, parent)[0] == 2
    # parent that is not a neighbour
    nbrs = set(g.col[g.row_ptr[v]:g.row_ptr[v + 1]].tolist())
    non = next(u for u in range(g.n_vertices) if u not in nbrs and u != v and level[u] == level[v] - 1)
    p = parent.copy(); p[v] = non
    assert oracle.validate_tree(g.row_ptr, g.col, root, level, p)[0] == 3
    # parent a neighbour on the same level (if one exists) -> rule 4
    same = [u for u in nbrs if level[u] == level[v]]
    if same:
        p = parent.copy(); p[v] = same[0]
        assert oracle.validate_tree(g.row_ptr, g.col, root, level, p)[0] == 4
    # level shifted by one for one vertex -> rule 4 or 5
    lv = level.copy(); lv[v] += 1
    assert oracle.validate_tree(g.row_ptr, g.col, root, lv, parent)[0] in (4, 5)
    # extra level-0 vertex
    lv = level.copy(); lv[v] = 0
    assert oracle.validate_tree(g.row_ptr, g.col, root, lv, parent)[0] == 2


def test_validator_rule5_exactly():
    """Rule 5 (every CSR edge spans <= 1 level, and never joins a reached and
    an unreached vertex) must fire on inputs that satisfy rules 1-4."""
    # path 0-1-2-3 plus chord 0-3: the path tree with levels 0,1,2,3 passes
    # rules 1-4 (every tree edge is an edge, levels step by one) but the chord
    # spans 3 levels -- true levels are 0,1,2,1
    g = edges_to_csr(np.array([0, 1, 2, 0]), np.array([1, 2, 3, 3]), 4)
    level = np.array([0, 1, 2, 3], dtype=np.int32)
    parent = np.array([0, 0, 1, 2], dtype=np.int32)
    assert oracle.validate_tree(g.row_ptr, g.col, 0, level, parent)[0] == 5
    level2, parent2, _ = oracle.bfs(g.row_ptr, g.col, 0)
    assert level2.tolist() == [0, 1, 2, 1]
    assert oracle.validate_tree(g.row_ptr, g.col, 0, level2, parent2) == (0, -1)
    # an edge spanning exactly 2 levels: 0-1, 1-2, 0-2 with levels 0,1,2
    g = edges_to_csr(np.array([0, 1, 0]), np.array([1, 2, 2]), 3)
    assert oracle.validate_tree(g.row_ptr, g.col, 0, np.array([0, 1, 2], np.int32),
                                np.array([0, 0, 1], np.int32))[0] == 5
    # a reached vertex with an unreached neighbour whose own fields are
    # consistent (level -1, parent -1): path 0-1-2 cut after 1
    g = edges_to_csr(np.array([0, 1]), np.array([1, 2]), 3)
    rule, bad = oracle.validate_tree(g.row_ptr, g.col, 0, np.array([0, 1, -1], np.int32),
                                     np.array([0, 0, -1], np.int32))
    assert rule == 5 and bad in (1, 2)
    # on a Kronecker graph: drop a whole leaf (a reached vertex whose only
    # reached neighbours are one level up, so nobody names it as a parent)
    gk = kronecker_csr(10, 16, 1)
    root = int(np.argmax(gk.degrees()))
    lv, pa, _ = oracle.bfs(gk.row_ptr, gk.col, root)
    children = np.zeros(gk.n_vertices, dtype=bool)
    children[pa[(pa >= 0) & (np.arange(gk.n_vertices) != root)]] = True
    leaf = int(np.flatnonzero((lv > 0) & ~children)[0])
    lv2, pa2 = lv.copy(), pa.copy()
    lv2[leaf], pa2[leaf] = -1, -1
    assert oracle.validate_tree(gk.row_ptr, gk.col, root, lv2, pa2)[0] == 5


def test_min_id_parent_is_min_over_candidates():
    # a diamond: 0-1, 0-2, 1-3, 2-3 ; root 0 -> parent(3) = 1 (not 2)
    g = edges_to_csr(np.array([0, 0, 1, 2]), np.array([1, 2, 3, 3]), 4)
    level, parent, _ = oracle.bfs(g.row_ptr, g.col, 0)
    assert level.tolist() == [0, 1, 1, 2] and parent.tolist() == [0, 0, 0, 1]
    # relabel so the larger id is the only level-1 neighbour through one side
    g = edges_to_csr(np.array([0, 0, 3, 2]), np.array([3, 2, 1, 1]), 4)
    level, parent, _ = oracle.bfs(g.row_ptr, g.col, 0)
    assert level.tolist() == [0, 2, 1, 1] and parent.tolist() == [0, 2, 0, 0]
