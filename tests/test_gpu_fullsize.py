"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (default options: RF/AN, chunk queue, parents='any', full occupancy).

* config 3, grid 4096 x 4096 from the corner: levels against the closed form
  level(r, c) = r + c (every vertex), parents valid; with the min-id rule the
  parents against the closed form v - 4096 (r > 0) / v - 1.
* config 4, Kronecker scale 24: every level against the oracle for 2 roots.
* config 5, Kronecker scale 26: every level against the oracle for 1 root.
"""
import numpy as np
import pytest

import oracle

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


@pytest.fixture(scope="module")
def tq():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_icpp_troendletj19_b200 as m
    return m


def test_grid4096_closed_form(tq):
    import torch
    import inputs.gpu as gg
    rows = 4096
    rp, col = gg.grid_csr_cuda(rows)
    n = rows * rows
    v = torch.arange(n, device="cuda", dtype=torch.int64)
    r, c = v // rows, v % rows
    for parents in ("any", "min_id"):
        level, parent, st = tq.bfs(rp, col, 0, parents=parents)
        assert torch.equal(level.long(), r + c)
        lp = level.long()[parent.long()]
        assert torch.equal(lp[1:], level.long()[1:] - 1) and int(parent[0]) == 0
        # Graph500 rules (tree edges are CSR edges, no edge spans > 1 level)
        assert oracle.validate_tree(rp.cpu().numpy(), col.cpu().numpy(), 0, level.cpu().numpy(),
                                    parent.cpu().numpy()) == (0, -1)
        if parents == "min_id":
            exp = torch.where(r > 0, v - rows, v - 1)
            exp[0] = 0
            assert torch.equal(parent.long(), exp)
        assert st["traversed_edges"] == 2 * rows * (rows - 1) and st["max_level"] == 2 * rows - 2


def _kron_check(tq, scale, n_roots, t0=None):
    import torch
    import inputs.gpu as gg
    from inputs import sample_roots
    rp, col = gg.kronecker_csr_cuda(scale, 16, 1)
    rp_h, col_h = rp.cpu().numpy(), col.cpu().numpy()
    n = rp.numel() - 1
    level = torch.empty(n, dtype=torch.int32, device="cuda")
    parent = torch.empty_like(level)
    with tq.BfsPlan(rp, col) as plan:
        if t0 is not None:  # start the queues just below a 2^32 wrap of the sequence tags
            plan.set_tickets(*t0)
        for root in sample_roots(rp_h, n_roots, 2):
            st = plan.run(int(root), level, parent)
            lv_o, _, info = oracle.bfs(rp_h, col_h, int(root), parents=False)
            lv = level.cpu().numpy()
            bad = np.flatnonzero(lv != lv_o)
            assert bad.size == 0, f"{bad.size} level mismatches"
            pa = parent.cpu().numpy()
            reached = lv_o > 0
            assert np.all(lv_o[pa[reached]] == lv_o[reached] - 1)
            # the default parent rule ('any') at full size: every Graph500 rule,
            # including that each tree edge (parent[v], v) is a CSR edge
            assert oracle.validate_tree(rp_h, col_h, int(root), lv, pa) == (0, -1)
            assert st["traversed_edges"] == info["traversed_edges"]
            assert st["reached"] == info["reached"]


def test_kron24_levels_identical(tq):
    _kron_check(tq, 24, 2)


def test_kron24_across_the_ticket_wrap(tq):
    # the bench's long-running plan crosses 2^32 tickets many times
    _kron_check(tq, 24, 2, t0=((1 << 32) - 5_000_000, (1 << 32) - 3_000))


def test_kron26_levels_identical(tq):
    _kron_check(tq, 26, 1)


@pytest.mark.parametrize("variant", ["rf_an", "per_thread_afa", "an"])
def test_paper_synthetic_tree_closed_form(tq, variant):
    """P:301 synthetic dataset (reading R13): 10,485,760-vertex heap-ordered
    4-ary tree; level(i) = k iff 4^k <= 3i+1 < 4^(k+1), parent (i-1)/4."""
    import torch
    import inputs.gpu as gg
    n = 10485760
    rp, col = gg.tree4_csr_cuda(n)
    level, parent, st = tq.bfs(rp, col, 0, variant=variant, parents="min_id", timeout_s=60)
    i = torch.arange(n, device="cuda", dtype=torch.int64)
    x = 3 * i + 1
    exp = torch.zeros(n, dtype=torch.int64, device="cuda")
    k, p4 = 0, 1
    while p4 * 4 <= int(x.max()):
        k += 1
        p4 *= 4
        exp[x >= p4] = k
    assert torch.equal(level.long(), exp)
    exp_par = torch.where(i > 0, (i - 1) // 4, torch.zeros_like(i))
    assert torch.equal(parent.long(), exp_par)
    assert st["traversed_edges"] == n - 1


def test_queue_bench_full_size_conserves(tq):
    from inputs import fingerprint, item_of
    for variant in ("rf_an", "per_thread_afa", "cas_retry", "an"):
        r = tq.queue_bench(variant, warps=0, batch=32, items=1 << 24, capacity=1 << 20, seed=3)
        assert (r["deq"], r["sum_deq"], r["xor_deq"]) == fingerprint(item_of(3, np.arange(r["items"])))
