"""GPU parity of the queue as a generic scheduler (NEXT row 4): label-
correcting SSSP on the same persistent kernel vs the Dijkstra oracle.
Distances and (min-id) parents must be identical element by element."""
import numpy as np
import pytest

import oracle
from inputs import edge_weights, edges_to_csr, grid_csr, kronecker_csr, sample_roots, tree4_csr

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def tq():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_icpp_troendletj19_b200 as m
    return m


def check(g, w, src, dist, parent):
    d_o, p_o, _ = oracle.sssp(g.row_ptr, g.col, w, src)
    d = (dist.cpu().numpy() if hasattr(dist, "cpu") else dist).view(np.uint32)
    p = parent.cpu().numpy() if hasattr(parent, "cpu") else parent
    bad = np.flatnonzero(d != d_o)
    assert bad.size == 0, f"{bad.size} distance mismatches, first v={bad[0]}: {d[bad[0]]} vs {d_o[bad[0]]}"
    bad = np.flatnonzero(p != p_o)
    assert bad.size == 0, f"{bad.size} parent mismatches, first v={bad[0]}: {p[bad[0]]} vs {p_o[bad[0]]}"


def dev(a):
    import torch
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


@pytest.mark.parametrize("wmax", [1, 16, 255, 100000])
def test_sssp_kronecker(tq, wmax):
    g = kronecker_csr(12, 16, 2)
    w = edge_weights(g.row_ptr, g.col, 3, wmax)
    rp, col, wd = dev(g.row_ptr), dev(g.col), dev(w)
    import torch
    dist = torch.empty(g.n_vertices, dtype=torch.int32, device="cuda")
    parent = torch.empty_like(dist)
    with tq.SsspPlan(rp, col, wd, timeout_s=30) as plan:
        for src in sample_roots(g.row_ptr, 4, 5):
            plan.run(int(src), dist, parent)
            check(g, w, int(src), dist, parent)


@pytest.mark.parametrize("chunk", [32, 512])
def test_sssp_hubs_and_small_graphs(tq, chunk):
    for g in (kronecker_csr(14, 16, 6), grid_csr(50, 37), tree4_csr(3000),
              edges_to_csr(np.array([0, 0, 1, 2]), np.array([1, 2, 3, 3]), 6, "diamond+isolated")):
        w = edge_weights(g.row_ptr, g.col, 11, 50)
        rp, col, wd = dev(g.row_ptr), dev(g.col), dev(w)
        src = int(np.argmax(g.degrees()))
        dist, parent, st = tq.sssp(rp, col, wd, src, chunk=chunk, timeout_s=30)
        check(g, w, src, dist, parent)


def test_sssp_host_arrays_and_unit_weights_equal_bfs(tq):
    g = grid_csr(64, 64)
    w = np.ones(g.nnz, dtype=np.int32)
    dist, parent, _ = tq.sssp(g.row_ptr, g.col, w, 0)  # numpy in/out (staged by the library)
    lv, pa, _ = oracle.bfs(g.row_ptr, g.col, 0)
    assert np.array_equal(dist.view(np.uint32).astype(np.int64), lv) and np.array_equal(parent, pa)


def test_sssp_rejects_other_variants(tq):
    g = kronecker_csr(8, 16, 1)
    w = edge_weights(g.row_ptr, g.col, 1, 9)
    with pytest.raises(tq.TQError):
        from paper_conf_icpp_troendletj19_b200 import _lib, api
        import ctypes
        o = api._opts(variant="cas_retry")
        h = ctypes.c_void_p()
        _lib.check(_lib.lib().sssp_plan_create(ctypes.byref(api._csr(g.row_ptr, g.col)), w.ctypes.data,
                                               ctypes.byref(o), ctypes.byref(h)), "sssp_plan_create")


def test_sssp_schedule_independence_under_delay_injection(tq):
    """Delay injection (bfs_opts.debug_delay_ns): distances and
    min-id parents stay identical to Dijkstra under perturbed schedules."""
    for g in (kronecker_csr(11, 16, 4), grid_csr(40, 33)):
        w = edge_weights(g.row_ptr, g.col, 5, 100)
        rp, col, wd = dev(g.row_ptr), dev(g.col), dev(w)
        src = int(np.argmax(g.degrees()))
        for seed in range(3):
            dist, parent, _ = tq.sssp(rp, col, wd, src, chunk=64, timeout_s=30, debug_delay_ns=20000,
                                      debug_delay_seed=seed)
            check(g, w, src, dist, parent)
