"""GPU parity of the persistent-thread BFS (libtq, through the C ABI) against
the sequential oracle.

Levels must be identical element by element; parents must be identical under
the min-id rule (R5) and validate Graph500-style. Every queue
variant runs the same BFS (RF/AN, per-thread AFA, CAS-retry BASE, AN).
"""
import numpy as np
import pytest

import oracle
from inputs import (edges_to_csr, grid_csr, kronecker_csr, sample_roots, tree4_csr)

pytestmark = pytest.mark.gpu

VARIANTS = ["rf_an", "per_thread_afa", "cas_retry", "an"]
# RF/AN runs of graphs that fit one block's shared memory take the
# shared-memory path by default (bfs_opts.smem_path);
# tests on such graphs run both paths: "grid" forces the persistent grid
# (smem_path = -1), "smem" requires the shared-memory path (smem_path = 1)
PATHS = {"grid": -1, "smem": 1}
VARIANT_PATHS = [("rf_an", "grid"), ("rf_an", "smem"), ("per_thread_afa", "grid"), ("cas_retry", "grid"),
                 ("an", "grid")]


@pytest.fixture(scope="module")
def tq():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_icpp_troendletj19_b200 as m
    return m


def to_dev(g):
    import torch
    return torch.from_numpy(g.row_ptr).cuda(), torch.from_numpy(g.col).cuda()


def check_against_oracle(g, root, level, parent, stats=None, min_id=False):
    """Levels: identical to the oracle. Parents: identical under the min-id
    rule; under the default 'any' rule (several trees are correct) checked
    for validity: Graph500 rules and parent one level up in the oracle's
    levels."""
    lv_o, pa_o, info = oracle.bfs(g.row_ptr, g.col, root)
    lv = level.cpu().numpy() if hasattr(level, "cpu") else level
    pa = parent.cpu().numpy() if hasattr(parent, "cpu") else parent
    bad = np.flatnonzero(lv != lv_o)
    assert bad.size == 0, f"{bad.size} level mismatches, first v={bad[0]} gpu={lv[bad[0]]} oracle={lv_o[bad[0]]}"
    if min_id:
        bad = np.flatnonzero(pa != pa_o)
        assert bad.size == 0, f"{bad.size} parent mismatches, first v={bad[0]} gpu={pa[bad[0]]} oracle={pa_o[bad[0]]}"
    else:
        r = lv_o > 0
        assert np.all(lv_o[pa[r]] == lv_o[r] - 1)
    assert oracle.validate_tree(g.row_ptr, g.col, root, lv, pa) == (0, -1)
    if stats is not None:
        assert stats["traversed_edges"] == info["traversed_edges"]
        assert stats["reached"] == info["reached"]
        assert stats["max_level"] == int(lv_o.max())


@pytest.mark.parametrize("parents", ["any", "min_id"])
@pytest.mark.parametrize("variant,path", VARIANT_PATHS)
def test_rmat10_config1_sample_roots(tq, variant, path, parents):
    g = kronecker_csr(10, 16, 1)
    rp, col = to_dev(g)
    import torch
    level = torch.empty(g.n_vertices, dtype=torch.int32, device="cuda")
    parent = torch.empty_like(level)
    with tq.BfsPlan(rp, col, variant=variant, timeout_s=20, parents=parents, smem_path=PATHS[path]) as plan:
        for root in sample_roots(g.row_ptr, 16, 2):
            st = plan.run(int(root), level, parent)
            check_against_oracle(g, int(root), level, parent, st, min_id=parents == "min_id")
            assert st["smem_path"] == (path == "smem")


@pytest.mark.parametrize("path", ["grid", "smem"])
@pytest.mark.parametrize("parents", ["any", "min_id"])
def test_rmat10_all_roots_rf_an(tq, parents, path):
    """Every vertex of the config-1 graph as the root, isolated ones included."""
    import torch
    g = kronecker_csr(10, 16, 1)
    rp, col = to_dev(g)
    level = torch.empty(g.n_vertices, dtype=torch.int32, device="cuda")
    parent = torch.empty_like(level)
    with tq.BfsPlan(rp, col, timeout_s=20, parents=parents, smem_path=PATHS[path]) as plan:
        for root in range(g.n_vertices):
            st = plan.run(root, level, parent)
            check_against_oracle(g, root, level, parent, st, min_id=parents == "min_id")


def test_smem_path_is_the_default_for_graphs_that_fit(tq):
    """Auto (smem_path = 0): config 1's graph runs on the shared-memory path
    (one 1024-thread block), a graph too large for it on the persistent grid;
    requiring it for a graph that does not fit, or for another variant, is
    TQ_ERR_UNSUPPORTED."""
    g = kronecker_csr(10, 16, 1)
    rp, col = to_dev(g)
    root = int(sample_roots(g.row_ptr, 1, 2)[0])
    level, parent, st = tq.bfs(rp, col, root)
    check_against_oracle(g, root, level, parent, st)
    assert st["smem_path"] == 1 and st["persistent_threads"] == 1024
    big = kronecker_csr(13, 16, 1)
    rpb, colb = to_dev(big)
    _, _, st = tq.bfs(rpb, colb, int(sample_roots(big.row_ptr, 1, 2)[0]))
    assert st["smem_path"] == 0
    for kw in ({}, {"variant": "an"}):
        with pytest.raises(tq.TQError) as ei:
            tq.bfs(rpb if not kw else rp, colb if not kw else col, 0, smem_path=1, **kw)
        assert ei.value.status == -6


@pytest.mark.parametrize("variant,path", VARIANT_PATHS)
def test_small_closed_form_graphs_min_id(tq, variant, path):
    """Closed-form graphs with the min-id rule: parents are unique, so the
    grid / tree / path parents must equal the oracle's (and the formulas)."""
    for g in [edges_to_csr(np.arange(99), np.arange(1, 100), 100, "path100"), grid_csr(48, 31),
              tree4_csr(3000)]:
        rp, col = to_dev(g)
        for root in {0, g.n_vertices // 2}:
            level, parent, st = tq.bfs(rp, col, root, variant=variant, timeout_s=20, parents="min_id",
                                       smem_path=PATHS[path])
            check_against_oracle(g, root, level, parent, st, min_id=True)


@pytest.mark.parametrize("variant,path", VARIANT_PATHS)
def test_small_closed_form_graphs(tq, variant, path):
    graphs = [
        edges_to_csr(np.arange(99), np.arange(1, 100), 100, "path100"),
        edges_to_csr(np.zeros(999, dtype=np.int64), np.arange(1, 1000), 1000, "star1000"),
        grid_csr(64, 33),
        tree4_csr(5000),
        edges_to_csr(np.array([0]), np.array([1]), 2, "edge"),
        edges_to_csr(np.array([0, 0, 1, 2, 3]), np.array([1, 2, 3, 4, 4]), 8, "with_isolated"),
    ]
    for g in graphs:
        rp, col = to_dev(g)
        for root in {0, g.n_vertices // 2, g.n_vertices - 1}:
            level, parent, st = tq.bfs(rp, col, root, variant=variant, timeout_s=20, smem_path=PATHS[path])
            check_against_oracle(g, root, level, parent, st)


def test_single_vertex_and_isolated_root(tq):
    g = edges_to_csr(np.array([], dtype=np.int64), np.array([], dtype=np.int64), 1, "one")
    rp, col = to_dev(g)
    level, parent, st = tq.bfs(rp, col, 0)
    assert level.tolist() == [0] and parent.tolist() == [0] and st["traversed_edges"] == 0
    g = kronecker_csr(10, 16, 1)
    iso = int(np.flatnonzero(g.degrees() == 0)[0])
    rp, col = to_dev(g)
    level, parent, st = tq.bfs(rp, col, iso)
    check_against_oracle(g, iso, level, parent, st)
    assert st["reached"] == 1


@pytest.mark.parametrize("path", ["grid", "smem"])
def test_label_correcting_motif(tq, path):
    """r-a, r-b, a-c, c-x, b-x: x has level 2 via b, not 3 via a-c (R4).
    Repeated many times so that different schedules occur."""
    # plus a long path hanging off a to slow one side down
    n = 6 + 200
    src = [0, 0, 1, 3, 2] + [1] + list(range(6, n - 1))
    dst = [1, 2, 3, 4, 4] + [6] + list(range(7, n))
    g = edges_to_csr(np.array(src), np.array(dst), n)
    rp, col = to_dev(g)
    for _ in range(20):
        level, parent, st = tq.bfs(rp, col, 0, smem_path=PATHS[path])
        check_against_oracle(g, 0, level, parent, st)


@pytest.mark.parametrize("parents", ["any", "min_id"])
@pytest.mark.parametrize("variant,path", [("rf_an", "grid"), ("rf_an", "auto"), ("an", "grid")])
def test_schedule_independence_under_delay_injection(tq, variant, path, parents):
    """SURVEY §8(c) "schedule independence": with the test-only delay
    injection (bfs_opts.debug_delay_ns) 1/8 of the vertices are expanded late
    and another 1/8 with a level read long before their offers land, for
    several seeds: levels stay identical to the oracle, parents identical
    under min-id and valid under 'any' (label correcting, R4)."""
    n = 6 + 200
    src = [0, 0, 1, 3, 2] + [1] + list(range(6, n - 1))
    dst = [1, 2, 3, 4, 4] + [6] + list(range(7, n))
    graphs = [edges_to_csr(np.array(src), np.array(dst), n), kronecker_csr(11, 16, 7), grid_csr(48, 37),
              tree4_csr(3000)]
    for g in graphs:
        rp, col = to_dev(g)
        root = int(sample_roots(g.row_ptr, 1, 3)[0]) if g.n_vertices > 5000 else 0
        for seed in range(4):
            level, parent, st = tq.bfs(rp, col, root, variant=variant, parents=parents, timeout_s=30,
                                       chunk=64, debug_delay_ns=20000, debug_delay_seed=seed,
                                       smem_path=PATHS.get(path, 0))
            check_against_oracle(g, root, level, parent, st, min_id=parents == "min_id")


def test_delay_injection_perturbs_the_schedule(tq):
    """The injection really changes the execution: on the motif graph with a
    slow path the delayed runs re-enqueue (level corrections) or take longer."""
    g = kronecker_csr(12, 16, 3)
    rp, col = to_dev(g)
    root = int(sample_roots(g.row_ptr, 1, 4)[0])
    _, _, st0 = tq.bfs(rp, col, root)
    _, _, st1 = tq.bfs(rp, col, root, debug_delay_ns=50000, debug_delay_seed=1)
    assert st1["ms_kernel"] > st0["ms_kernel"]
    with pytest.raises(tq.TQError):
        tq.bfs(rp, col, root, debug_delay_ns=2_000_000)  # out of range -> TQ_ERR_INVALID


@pytest.mark.parametrize("chunk", [32, 64, 1024])
def test_hub_chunking(tq, chunk):
    """Vertices with more than `chunk` edges are split into chunk tokens."""
    g = kronecker_csr(14, 16, 5)
    rp, col = to_dev(g)
    deg = g.degrees()
    for root in (int(np.argmax(deg)), int(sample_roots(g.row_ptr, 1, 9)[0])):
        level, parent, st = tq.bfs(rp, col, root, chunk=chunk)
        check_against_oracle(g, root, level, parent, st)
        n_hub_reached = int(((deg > chunk) & (level.cpu().numpy() >= 0)).sum())
        if n_hub_reached:
            assert st["chunk_tasks"] > 0


def test_host_pointers_match_device(tq):
    g = kronecker_csr(12, 16, 3)
    root = int(sample_roots(g.row_ptr, 1, 4)[0])
    lh, ph, sth = tq.bfs(g.row_ptr, g.col, root)  # numpy in, numpy out
    assert isinstance(lh, np.ndarray)
    check_against_oracle(g, root, lh, ph, sth)


def test_queue_full_aborts_and_retry_succeeds(tq):
    """queue-full aborts (no retry); the user may retry with a larger queue."""
    g = kronecker_csr(12, 16, 1)
    rp, col = to_dev(g)
    root = int(np.argmax(g.degrees()))
    with pytest.raises(tq.TQError) as ei:
        tq.bfs(rp, col, root, capacity=64)
    assert ei.value.status == -4
    level, parent, st = tq.bfs(rp, col, root, capacity=1 << 14)
    check_against_oracle(g, root, level, parent, st)


def test_smem_queue_full_aborts_and_retry_succeeds(tq):
    """The same queue-full exception on the shared-memory ring (P:268 line 25,
    P:281): a ring of 64 slots overflows from the top hub of config 1's graph;
    with a larger ring the same run is exact; a plan answering the abort with
    grow_on_full moves on to a ring too large for shared memory, i.e. to the
    persistent grid, and is exact too."""
    g = kronecker_csr(10, 16, 1)
    rp, col = to_dev(g)
    root = int(np.argmax(g.degrees()))
    with pytest.raises(tq.TQError) as ei:
        tq.bfs(rp, col, root, capacity=64, smem_path=1)
    assert ei.value.status == -4
    level, parent, st = tq.bfs(rp, col, root, capacity=4096, smem_path=1)
    assert st["smem_path"] == 1
    check_against_oracle(g, root, level, parent, st)
    with tq.BfsPlan(rp, col, capacity=64) as plan:
        st = plan.run(root, level, parent, grow_on_full=True)
        assert plan.regrows >= 1 and st["smem_path"] == 0
        check_against_oracle(g, root, level, parent, st)


def test_concurrent_plans_on_two_streams(tq):
    """bfs_plan_launch / bfs_plan_wait: two BFS in flight at once on two
    streams (half the persistent grid each); both results exact."""
    import torch
    g = kronecker_csr(13, 16, 3)
    rp, col = to_dev(g)
    half = tq.persistent_threads() // 2
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    plans = [tq.BfsPlan(rp, col, stream=s, threads=half, parents=pr) for s, pr in zip(streams, ["any", "min_id"])]
    lv = [torch.empty(g.n_vertices, dtype=torch.int32, device="cuda") for _ in plans]
    pa = [torch.empty_like(lv[0]) for _ in plans]
    roots = [int(r) for r in sample_roots(g.row_ptr, 6, 8)]
    for k in range(0, len(roots), 2):
        for i in range(2):
            plans[i].launch(roots[k + i], lv[i], pa[i])
        for i in range(2):
            st = plans[i].wait()
            check_against_oracle(g, roots[k + i], lv[i], pa[i], st, min_id=(i == 1))
    with pytest.raises(tq.TQError):
        plans[0].wait()  # nothing in flight
    stats = tq.run_concurrent(plans, roots)
    assert [s["reached"] for s in stats] == [oracle.bfs(g.row_ptr, g.col, r, parents=False)[2]["reached"]
                                             for r in roots]
    for p_ in plans:
        p_.close()


@pytest.mark.parametrize("where", ["pinned", "pageable", "device"])
def test_run_batch_overlapped_outputs(tq, where):
    """bfs_plan_run_batch: one output row per root; host rows are filled by
    D2H copies overlapped with the next root's BFS."""
    import torch
    g = kronecker_csr(12, 16, 9)
    rp, col = to_dev(g)
    roots = [int(r) for r in sample_roots(g.row_ptr, 5, 10)]
    n = g.n_vertices
    if where == "device":
        lv = torch.empty(len(roots) * n, dtype=torch.int32, device="cuda")
        pa = torch.empty_like(lv)
    elif where == "pinned":
        lv = torch.empty(len(roots) * n, dtype=torch.int32, pin_memory=True).numpy()
        pa = torch.empty(len(roots) * n, dtype=torch.int32, pin_memory=True).numpy()
    else:
        lv = np.empty(len(roots) * n, dtype=np.int32)
        pa = np.empty_like(lv)
    with tq.BfsPlan(rp, col) as plan:
        stats = plan.run_batch(roots, lv, pa)
        lvh = lv.cpu().numpy() if where == "device" else lv
        pah = pa.cpu().numpy() if where == "device" else pa
        for i, r in enumerate(roots):
            check_against_oracle(g, r, lvh[i * n:(i + 1) * n], pah[i * n:(i + 1) * n], stats[i])
        # stride 0: one reused buffer, last root's result remains
        one = np.empty(n, dtype=np.int32)
        plan.run_batch(roots, one, None, stride=0)
        assert np.array_equal(one, oracle.bfs(g.row_ptr, g.col, roots[-1], parents=False)[0])


def test_grow_on_full_retries_with_larger_queue(tq):
    g = kronecker_csr(12, 16, 1)
    rp, col = to_dev(g)
    root = int(np.argmax(g.degrees()))
    with tq.BfsPlan(rp, col, capacity=64) as plan:
        import torch
        level = torch.empty(g.n_vertices, dtype=torch.int32, device="cuda")
        parent = torch.empty_like(level)
        st = plan.run(root, level, parent, grow_on_full=True)
        assert plan.regrows >= 1
        check_against_oracle(g, root, level, parent, st)


def test_plan_reuse_after_abort_and_many_runs(tq):
    import torch
    from inputs import kronecker_edges
    s, d = kronecker_edges(11, 16, 2)
    # the Kronecker graph plus a separate 300-vertex path component
    n0 = 1 << 11
    ps = np.arange(n0, n0 + 299, dtype=np.uint64)
    g = edges_to_csr(np.concatenate([s, ps]), np.concatenate([d, ps + np.uint64(1)]), n0 + 300)
    rp, col = to_dev(g)
    level = torch.empty(g.n_vertices, dtype=torch.int32, device="cuda")
    parent = torch.empty_like(level)
    roots = sample_roots(g.row_ptr[: n0 + 1], 8, 1)
    with tq.BfsPlan(rp, col, capacity=128) as small:
        with pytest.raises(tq.TQError) as ei:
            small.run(int(np.argmax(g.degrees())), level, parent)
        assert ei.value.status == -4
        # the dirty plan resets its queue; the small component still fits
        for _ in range(3):
            small.run(n0 + 150, level, parent)
            check_against_oracle(g, n0 + 150, level, parent)
    with tq.BfsPlan(rp, col) as plan:
        for _ in range(3):
            for r in roots:  # tickets continue across runs without an O(C) reset
                plan.run(int(r), level, parent)
                check_against_oracle(g, int(r), level, parent)


@pytest.mark.parametrize("threads", [256, 2048, 32768])
def test_thread_counts(tq, threads):
    g = kronecker_csr(12, 16, 7)
    rp, col = to_dev(g)
    root = int(sample_roots(g.row_ptr, 1, 3)[0])
    level, parent, st = tq.bfs(rp, col, root, threads=threads)
    check_against_oracle(g, root, level, parent, st)
    assert st["persistent_threads"] == threads


def test_no_backoff_and_large_backoff(tq):
    g = grid_csr(128, 128)
    rp, col = to_dev(g)
    for b in (-1, 4096):
        level, parent, st = tq.bfs(rp, col, 0, backoff_ns=b)
        check_against_oracle(g, 0, level, parent, st)


@pytest.mark.parametrize("variant", VARIANTS)
def test_any_parent_rule_levels_exact_tree_valid(tq, variant):
    """parents='any': levels still bit-exact; the parent tree is checked for
    validity (Graph500 rules + parent one level up in the oracle's levels)."""
    g = kronecker_csr(13, 16, 4)
    rp, col = to_dev(g)
    for root in sample_roots(g.row_ptr, 4, 6):
        level, parent, st = tq.bfs(rp, col, int(root), variant=variant)  # default rule: any
        lv_o, _, info = oracle.bfs(g.row_ptr, g.col, int(root), parents=False)
        lv, pa = level.cpu().numpy(), parent.cpu().numpy()
        assert np.array_equal(lv, lv_o)
        assert oracle.validate_tree(g.row_ptr, g.col, int(root), lv, pa) == (0, -1)
        reached = lv_o > 0
        assert np.all(lv_o[pa[reached]] == lv_o[reached] - 1)
        assert st["traversed_edges"] == info["traversed_edges"]


@pytest.mark.parametrize("path,cap", [("grid", 1024), ("smem", 256)])
def test_ring_wraps_within_runs(tq, path, cap):
    """A queue smaller than one run's ticket count: every run crosses the
    first-lap boundary t0 + C (R18) and the ring wraps many times
    across consecutive runs on one plan (the shared-memory ring restarts at
    ticket 0 each run and wraps within it: on a 48 x 31 grid, whose frontier
    stays small, ~1,500 tickets per run through 256 slots); results stay
    exact."""
    import torch
    g = kronecker_csr(10, 16, 1) if path == "grid" else grid_csr(48, 31)
    rp, col = to_dev(g)
    level = torch.empty(g.n_vertices, dtype=torch.int32, device="cuda")
    parent = torch.empty_like(level)
    with tq.BfsPlan(rp, col, capacity=cap, parents="min_id", smem_path=PATHS[path]) as plan:
        tickets, wrapped = 0, 0
        for r in sample_roots(g.row_ptr, 12, 5):
            st = plan.run(int(r), level, parent, grow_on_full=path == "grid")
            tickets += st["tickets"]
            wrapped += st["tickets"] > 4 * cap
            check_against_oracle(g, int(r), level, parent, st, min_id=True)
    assert tickets > 8 * cap
    if path == "smem":  # its ring restarts each run: the wrap is within the runs
        assert wrapped == 12


def test_probe_ceiling_measures(tq):
    g = tq.probe_ceiling(1 << 24, 1 << 22)
    assert 1.0 < g < 10000.0


def test_plans_recycled_through_the_memory_pool(tq):
    """Plans built from host CSRs of different sizes, destroyed and rebuilt
    (their device memory recycled by the library's stream-ordered pool), and
    the pool trimmed in between: every run stays identical to the oracle."""
    graphs = [kronecker_csr(12, 16, 3), grid_csr(64, 64), kronecker_csr(12, 16, 3), kronecker_csr(11, 8, 4)]
    for i, g in enumerate(graphs):
        root = int(sample_roots(g.row_ptr, 1, seed=i)[0])
        lv = np.empty(g.n_vertices, dtype=np.int32)
        pa = np.empty(g.n_vertices, dtype=np.int32)
        with tq.BfsPlan(g.row_ptr, g.col, parents="min_id") as plan:
            st = plan.run(root, lv, pa)
        check_against_oracle(g, root, lv, pa, st, min_id=True)
        if i == 1:
            tq.memory_trim(0)
    tq.memory_trim(0)


@pytest.mark.parametrize("bits", [4, 8])
@pytest.mark.parametrize("parents", ["any", "min_id"])
def test_level_mirror_widths(tq, bits, parents):
    """Both level-mirror widths (R8; the plan picks nibbles above
    2^25 vertices, bfs_opts.mirror_bits forces one): identical levels on graphs
    whose depth stays below, crosses and far exceeds the nibble's saturation
    (14) and the byte's (254), with delay injection perturbing the schedule."""
    graphs = [kronecker_csr(12, 16, 5), grid_csr(40, 23),
              edges_to_csr(np.arange(599), np.arange(1, 600), 600, "path600"), tree4_csr(20000)]
    for g in graphs:
        rp, col = to_dev(g)
        roots = [0, int(sample_roots(g.row_ptr, 1, seed=9)[0])]
        with tq.BfsPlan(rp, col, parents=parents, timeout_s=20, mirror_bits=bits, smem_path=-1) as plan:
            import torch
            lv = torch.empty(g.n_vertices, dtype=torch.int32, device="cuda")
            pa = torch.empty(g.n_vertices, dtype=torch.int32, device="cuda")
            for root in roots:
                st = plan.run(root, lv, pa)
                check_against_oracle(g, root, lv, pa, st, min_id=parents == "min_id")
        with tq.BfsPlan(rp, col, parents=parents, timeout_s=20, debug_delay_ns=2000,
                        debug_delay_seed=3, mirror_bits=bits, smem_path=-1) as plan:
            st = plan.run(roots[1], lv, pa)
            check_against_oracle(g, roots[1], lv, pa, st, min_id=parents == "min_id")


def test_deep_graph_plans_shrink_the_grid(tq):
    """threads == 0: a plan over >= 2^20 CSR entries starts at the full grid
    and, after a run of >= 1,024 levels, launches one block per SM (DESIGN.md
    7a); shallow graphs keep the full grid; graphs below 2^20 entries use one
    block per SM from the start; an explicit thread count is never changed.
    Results stay exact."""
    import torch
    full = tq.persistent_threads()
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    deep = grid_csr(1100, 512)  # 2.25M CSR entries, 1,610 levels from the corner
    rp, col = to_dev(deep)
    lv = torch.empty(deep.n_vertices, dtype=torch.int32, device="cuda")
    pa = torch.empty_like(lv)
    with tq.BfsPlan(rp, col, timeout_s=30) as plan:
        st1 = plan.run(0, lv, pa)
        check_against_oracle(deep, 0, lv, pa, st1)
        st2 = plan.run(1500, lv, pa)
        check_against_oracle(deep, 1500, lv, pa, st2)
    assert st1["persistent_threads"] == full and st2["persistent_threads"] == sms * 256
    with tq.BfsPlan(rp, col, threads=4096, timeout_s=30) as plan:
        plan.run(0, lv, pa)
        assert plan.run(7, lv, pa)["persistent_threads"] == 4096
    g = kronecker_csr(16, 16, 5)  # shallow, > 2^20 entries: the full grid stays
    rp, col = to_dev(g)
    lv = torch.empty(g.n_vertices, dtype=torch.int32, device="cuda")
    with tq.BfsPlan(rp, col) as plan:
        plan.run(int(sample_roots(g.row_ptr, 1, 1)[0]), lv, None)
        assert plan.run(int(sample_roots(g.row_ptr, 1, 2)[0]), lv, None)["persistent_threads"] == full
    small = edges_to_csr(np.arange(2999), np.arange(1, 3000), 3000, "path3000")
    rp, col = to_dev(small)
    lv = torch.empty(small.n_vertices, dtype=torch.int32, device="cuda")
    with tq.BfsPlan(rp, col, timeout_s=30, smem_path=-1) as plan:
        st = plan.run(0, lv, pa[:small.n_vertices])
        check_against_oracle(small, 0, lv, pa[:small.n_vertices], st)
        assert st["persistent_threads"] == sms * 256


@pytest.mark.parametrize("t_main,t_chunk", [((1 << 32) - 3000, (1 << 32) - 40),
                                            (5 * (1 << 32) - 1, (1 << 33) - 1),
                                            ((1 << 61) + (1 << 32) - 2000, (1 << 32) - 7)])
@pytest.mark.parametrize("parents", ["any", "min_id"])
def test_runs_across_the_32bit_ticket_wrap(tq, t_main, t_chunk, parents):
    """The kernel keeps the low 32 bits of a ticket (slot and sequence tag,
    DESIGN.md R1); a plan that has run many BFS carries its tickets on across
    runs (bench.py: ~1,600 scale-26 runs reach ~5e10 tickets, crossing 2^32
    about ten times).  Start both queues just below a 2^32 multiple
    (bfs_plan_set_tickets) and check levels and parents of consecutive runs on
    both sides of the wrap, with hub chunks (chunk = 32) in the chunk queue."""
    import torch
    g = kronecker_csr(12, 16, 3)
    rp, col = to_dev(g)
    lv = torch.empty(g.n_vertices, dtype=torch.int32, device="cuda")
    pa = torch.empty_like(lv)
    roots = [int(r) for r in sample_roots(g.row_ptr, 4, 21)]
    with tq.BfsPlan(rp, col, chunk=32, parents=parents, timeout_s=20) as plan:
        plan.set_tickets(t_main, t_chunk)
        assert plan.tickets() == (t_main, t_chunk)
        for r in roots:
            st = plan.run(r, lv, pa)
            check_against_oracle(g, r, lv, pa, st, min_id=parents == "min_id")
        m, c = plan.tickets()
        assert m > t_main and c > t_chunk
        assert (m >> 32) > (t_main >> 32) and (c >> 32) > (t_chunk >> 32)  # both crossed a 2^32 multiple


def test_set_tickets_argument_checks(tq):
    g = kronecker_csr(8, 16, 1)
    rp, col = to_dev(g)
    with tq.BfsPlan(rp, col) as plan:
        with pytest.raises(tq.TQError):
            plan.set_tickets(1 << 62, 0)
        with pytest.raises(tq.TQError):
            plan.set_tickets(0, 1 << 63)


@pytest.mark.parametrize("path", ["grid", "auto"])
@pytest.mark.parametrize("lanes", [1, 3, 17, 32])
@pytest.mark.parametrize("parents", ["any", "min_id"])
def test_ticket_lanes(tq, lanes, parents, path):
    """bfs_opts.ticket_lanes: only the first `lanes` lanes of a warp hold
    main-queue tickets (the default picks fewer on small graphs); results stay
    exact for any count, also with delay injection."""
    import torch
    graphs = [kronecker_csr(12, 16, 2), grid_csr(50, 31), tree4_csr(3000)]
    for g in graphs:
        rp, col = to_dev(g)
        lv = torch.empty(g.n_vertices, dtype=torch.int32, device="cuda")
        pa = torch.empty_like(lv)
        root = int(sample_roots(g.row_ptr, 1, 5)[0])
        sp = PATHS.get(path, 0)
        with tq.BfsPlan(rp, col, parents=parents, ticket_lanes=lanes, timeout_s=20, smem_path=sp) as plan:
            st = plan.run(root, lv, pa)
            check_against_oracle(g, root, lv, pa, st, min_id=parents == "min_id")
        with tq.BfsPlan(rp, col, parents=parents, ticket_lanes=lanes, timeout_s=20, debug_delay_ns=2000,
                        debug_delay_seed=lanes, smem_path=sp) as plan:
            st = plan.run(root, lv, pa)
            check_against_oracle(g, root, lv, pa, st, min_id=parents == "min_id")
    with pytest.raises(tq.TQError):
        tq.bfs(rp, col, 0, ticket_lanes=33)


def test_persisting_l2_limit_is_reference_counted(tq):
    """The device-wide persisting-L2 limit is raised by the first plan whose
    mirror gets an access-policy window and restored only when the last such
    plan is destroyed (destroying one plan must not reset another's lines)."""
    import torch
    from cuda.bindings import runtime as cudart
    import inputs.gpu as gg

    def limit():
        err, v = cudart.cudaDeviceGetLimit(cudart.cudaLimit.cudaLimitPersistingL2CacheSize)
        assert err == cudart.cudaError_t.cudaSuccess
        return v

    torch.cuda.synchronize()
    rp, col = gg.kronecker_csr_cuda(23, 8, 1)  # 8M vertices: an 8 MB byte mirror gets a window
    before = limit()
    a = tq.BfsPlan(rp, col)
    raised = limit()
    assert raised >= 8 << 20 or raised > before
    b = tq.BfsPlan(rp, col)
    assert limit() == raised
    a.close()
    assert limit() == raised  # b still holds it
    lv = torch.empty(rp.numel() - 1, dtype=torch.int32, device="cuda")
    from inputs import sample_roots
    r = int(sample_roots(rp.cpu().numpy(), 1, 3)[0])
    b.run(r, lv, None)
    b.close()
    assert limit() == before


@pytest.mark.parametrize("parents", ["any", "min_id"])
@pytest.mark.parametrize("relabel", [-1, 1])
def test_relabelled_plans(tq, relabel, parents):
    """bfs_opts.relabel: the plan runs on a
    degree-sorted copy of the CSR, but roots, outputs and parent ids are in
    the original numbering -- levels identical to the oracle, min-id parents
    identical (the minimum over ORIGINAL ids), 'any' parents Graph500-valid;
    roots include the top hub and an isolated vertex; a uniform grid and a
    tree (relabelled only when forced) too; host-CSR plans as well."""
    import torch
    graphs = [kronecker_csr(13, 16, 3), grid_csr(64, 40), tree4_csr(20000)]
    for g in graphs:
        rp, col = to_dev(g)
        deg = g.degrees()
        roots = [int(np.argmax(deg)), int(sample_roots(g.row_ptr, 1, 4)[0]), g.n_vertices - 1]
        if (deg == 0).any():
            roots.append(int(np.flatnonzero(deg == 0)[0]))
        lv = torch.empty(g.n_vertices, dtype=torch.int32, device="cuda")
        pa = torch.empty_like(lv)
        with tq.BfsPlan(rp, col, parents=parents, relabel=relabel, smem_path=-1, timeout_s=20) as plan:
            for r in roots:
                st = plan.run(r, lv, pa)
                check_against_oracle(g, r, lv, pa, st, min_id=parents == "min_id")
                assert st["relabelled"] == (relabel > 0)
            lvb = np.empty(len(roots) * g.n_vertices, dtype=np.int32)
            pab = np.empty_like(lvb)
            stats = plan.run_batch(roots, lvb, pab)
            for i, r in enumerate(roots):
                n = g.n_vertices
                check_against_oracle(g, r, lvb[i * n:(i + 1) * n], pab[i * n:(i + 1) * n], stats[i],
                                     min_id=parents == "min_id")
    g = kronecker_csr(12, 16, 8)
    r = int(sample_roots(g.row_ptr, 1, 1)[0])
    lh, ph, st = tq.bfs(g.row_ptr, g.col, r, parents=parents, relabel=relabel, smem_path=-1)  # host CSR
    check_against_oracle(g, r, lh, ph, st, min_id=parents == "min_id")
    assert st["relabelled"] == (relabel > 0)


def test_relabel_auto_rule(tq):
    """Auto: a graph with a vertex of more than `chunk` edges (Kronecker) is
    relabelled, a uniform grid is not; delay injection and chunk tokens on a
    relabelled plan stay exact."""
    g = kronecker_csr(14, 16, 2)
    rp, col = to_dev(g)
    r = int(sample_roots(g.row_ptr, 1, 3)[0])
    level, parent, st = tq.bfs(rp, col, r)
    check_against_oracle(g, r, level, parent, st)
    assert st["relabelled"] == 1 and st["chunk_tasks"] > 0
    for seed in range(3):
        level, parent, st = tq.bfs(rp, col, r, parents="min_id", chunk=64, debug_delay_ns=20000,
                                   debug_delay_seed=seed)
        check_against_oracle(g, r, level, parent, st, min_id=True)
    gg = grid_csr(256, 256)
    rp, col = to_dev(gg)
    level, parent, st = tq.bfs(rp, col, 0)
    check_against_oracle(gg, 0, level, parent, st)
    assert st["relabelled"] == 0
    # the relabelling happens at a plan's first run, whichever entry point it is
    roots = [int(x) for x in sample_roots(g.row_ptr, 3, 11)]
    lvb = np.empty(3 * g.n_vertices, dtype=np.int32)
    pab = np.empty_like(lvb)
    with tq.BfsPlan(g.row_ptr, g.col) as plan:  # host CSR: the plan owns its copies
        stats = plan.run_batch(roots, lvb, pab)
    n = g.n_vertices
    for i, r in enumerate(roots):
        check_against_oracle(g, r, lvb[i * n:(i + 1) * n], pab[i * n:(i + 1) * n], stats[i])
        assert stats[i]["relabelled"] == 1


@pytest.mark.parametrize("parents", ["any", "min_id"])
@pytest.mark.parametrize("level_bits", [0, 1, 2, 3])
def test_level_tokens(tq, level_bits, parents):
    """RF/AN BFS tokens carry their level (R22): a consumer then
    needs no acquire and a producer no release fence.  Levels that do not fit
    the field travel the fenced path (producer fence, consumer acquire
    re-read of the slot); a plan whose levels outgrew the field runs its later
    BFS with acquire polls.  bfs_opts.level_bits (test only) narrows the field
    so that both kinds of token mix within one run, also under delay injection
    (stale W reads) and with hub chunk tokens."""
    import torch
    graphs = [kronecker_csr(13, 16, 3), grid_csr(70, 41), tree4_csr(20000)]
    for g in graphs:
        rp, col = to_dev(g)
        lv = torch.empty(g.n_vertices, dtype=torch.int32, device="cuda")
        pa = torch.empty_like(lv)
        roots = [int(r) for r in sample_roots(g.row_ptr, 3, 7)]
        with tq.BfsPlan(rp, col, parents=parents, level_bits=level_bits, chunk=64, smem_path=-1,
                        timeout_s=20) as plan:
            sts = []
            for r in roots:
                st = plan.run(r, lv, pa)
                check_against_oracle(g, r, lv, pa, st, min_id=parents == "min_id")
                sts.append(st)
            field = (1 << level_bits) - 1 if level_bits else None
            assert sts[0]["level_tokens"] == 1
            if field is not None and sts[0]["max_level"] >= field:
                assert sts[1]["level_tokens"] == 0  # outgrown: acquire polls from then on
            if level_bits == 0:
                assert all(s["level_tokens"] == 1 for s in sts)
        with tq.BfsPlan(rp, col, parents=parents, level_bits=level_bits, chunk=64, smem_path=-1, timeout_s=20,
                        debug_delay_ns=20000, debug_delay_seed=level_bits) as plan:
            st = plan.run(roots[0], lv, pa)
            check_against_oracle(g, roots[0], lv, pa, st, min_id=parents == "min_id")
    with pytest.raises(tq.TQError):
        tq.bfs(rp, col, 0, level_bits=31)
