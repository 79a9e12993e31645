"""Input generators (inputs/): determinism, exact counts, CSR invariants and
R-MAT quadrant frequencies. Parity against Graph500's own generator is
unpinned (that generator is not available); see DESIGN.md."""
import hashlib

import numpy as np
import pytest

from inputs import (edges_to_csr, grid_csr, hash2, item_of, kronecker_csr, kronecker_edges,
                    permute_ids, sample_roots, tree4_csr)
from inputs.graphs import T_A, T_AB, T_ABC


def sha(csr):
    h = hashlib.sha256()
    h.update(csr.row_ptr.tobytes())
    h.update(csr.col.tobytes())
    return h.hexdigest()


def check_csr(g):
    rp, col = g.row_ptr, g.col
    assert rp[0] == 0 and np.all(np.diff(rp) >= 0) and rp[-1] == col.size
    rows = np.repeat(np.arange(g.n_vertices), np.diff(rp))
    assert np.all(col != rows)  # no self loops
    keys = rows.astype(np.int64) * g.n_vertices + col
    assert np.all(np.diff(keys) > 0)  # rows sorted, no duplicates
    rev = np.sort(col.astype(np.int64) * g.n_vertices + rows)
    np.testing.assert_array_equal(rev, keys)  # symmetric


def test_kronecker_deterministic_and_valid():
    a = kronecker_csr(10, 16, 1)
    b = kronecker_csr(10, 16, 1)
    c = kronecker_csr(10, 16, 2)
    assert sha(a) == sha(b) and sha(a) != sha(c)
    check_csr(a)
    s, d = kronecker_edges(10, 16, 1)
    assert s.size == 16 * 1024 and s.max() < 1024 and d.max() < 1024


def test_rmat_quadrant_frequencies():
    # first-level quadrant frequencies before the permutation ~ (.57, .19, .19, .05) within 4 sigma
    m = 1 << 18
    r = hash2(5, np.arange(m, dtype=np.uint64) * np.uint64(64)) >> np.uint64(32)
    counts = np.array([(r < T_A).sum(), ((r >= T_A) & (r < T_AB)).sum(),
                       ((r >= T_AB) & (r < T_ABC)).sum(), (r >= T_ABC).sum()])
    p = np.array([.57, .19, .19, .05])
    sigma = np.sqrt(m * p * (1 - p))
    assert np.all(np.abs(counts - m * p) < 4 * sigma)


@pytest.mark.parametrize("scale", [1, 5, 10, 17])
def test_permutation_is_bijective(scale):
    x = np.arange(1 << scale, dtype=np.uint64)
    y = permute_ids(x, scale, 123)
    assert np.unique(y).size == x.size and y.max() < x.size


def test_grid_and_tree_counts():
    g = grid_csr(64, 32)
    check_csr(g)
    assert g.nnz == 2 * (64 * 31 + 32 * 63)
    t = tree4_csr(1000)
    check_csr(t)
    assert t.nnz == 2 * 999


def test_edges_to_csr_drops_loops_and_dups():
    g = edges_to_csr(np.array([0, 1, 1, 2, 2]), np.array([0, 2, 2, 1, 3]), 4)
    assert g.row_ptr.tolist() == [0, 0, 1, 3, 4] and g.col.tolist() == [2, 1, 3, 2]


def test_roots_have_degree_and_are_deterministic():
    g = kronecker_csr(10, 16, 1)
    r1 = sample_roots(g.row_ptr, 64, 2)
    r2 = sample_roots(g.row_ptr, 64, 2)
    assert np.array_equal(r1, r2) and np.unique(r1).size == 64
    assert np.all(np.diff(g.row_ptr)[r1] > 0)


def test_items_unique():
    x = item_of(9, np.arange(1 << 20))
    assert np.unique(x).size == 1 << 20
