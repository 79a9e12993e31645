"""The public device API (include/tq_device.cuh) driven by a user kernel
(tests/csrc/devapi_test.cu, built against the headers only):
tq_warp_enqueue_n with 0..32 items per lane (Listing 3; arbitrary
n), tq_warp_dequeue_n (Listing 1) and tq_take / tq_poll
(Listing 2), checked against the oracle's sequential ticket model
(oracle.QueueModel): the ticket -> item maps of both sides are the same
bijection (FIFO hand-off), no item is lost or duplicated, and the
queue-full abort fires exactly when the model says the write at ticket t finds
ticket t - C untaken (P:268 line 25) -- including runs whose tickets
cross the 2^32 wrap of the 32-bit sequence tags (tq_reset_at)."""
import ctypes
import os

import numpy as np
import pytest

import oracle

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
STATUS_RUNNING, STATUS_FULL = 0, 2


@pytest.fixture(scope="module")
def tq():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_icpp_troendletj19_b200 as m
    return m


@pytest.fixture(scope="module")
def dev():
    from paper_conf_icpp_troendletj19_b200 import _build
    so = _build.build_user_kernel(os.path.join(ROOT, "tests", "csrc", "devapi_test.cu"),
                                  os.path.join(ROOT, "tests", "libtqdevapi.so"))
    L = ctypes.CDLL(so)
    vp, u64 = ctypes.c_void_p, ctypes.c_uint64
    L.devapi_run.restype = ctypes.c_int
    L.devapi_run.argtypes = [vp, ctypes.c_int, ctypes.c_int, vp, u64, vp, vp, u64, ctypes.c_int,
                             ctypes.c_double, vp, vp]
    return L


def run(tq, dev, capacity, t0, nmine, use_poll):
    """nmine: uint32[warps, rounds, 32]. Returns (counters, enq_log, deq_log, out)."""
    import torch
    warps, rounds, _ = nmine.shape
    q = tq.Queue(capacity)
    q.reset_at(t0)
    torch.cuda.synchronize()
    v = q.view()
    total = int(nmine.sum())
    n_dev = torch.from_numpy(nmine.reshape(-1).astype(np.int32)).cuda()
    enq = torch.full((max(total, 1),), -1, dtype=torch.int32, device="cuda")
    deq = torch.full((max(total, 1),), -1, dtype=torch.int32, device="cuda")
    out = torch.zeros(4, dtype=torch.int64, device="cuda")
    rc = dev.devapi_run(ctypes.byref(v), warps, rounds, n_dev.data_ptr(), t0, enq.data_ptr(), deq.data_ptr(),
                        total, int(use_poll), 20.0, out.data_ptr(), None)
    assert rc == 0
    c = q.counters()
    q.close()
    return (c, enq.cpu().numpy().view(np.uint32), deq.cpu().numpy().view(np.uint32),
            out.cpu().numpy())


def replay(enq, n):
    """The sequential model given the GPU's reservation order (ticket order)."""
    m = oracle.QueueModel(capacity=max(n, 1), max_tickets=max(n, 1))
    m.enqueue_n(enq[:n])
    base = m.dequeue_n(n)
    return np.array([m.take(base + t) for t in range(n)], dtype=np.uint32)


def expected_items(nmine):
    w, r, _ = nmine.shape
    idx = np.arange(w * r * 32).reshape(w, r, 32)
    return np.sort(np.concatenate([idx.reshape(-1)[k] * 32 + np.arange(nmine.reshape(-1)[k])
                                   for k in range(idx.size)]).astype(np.uint32))


@pytest.mark.parametrize("t0", [0, (1 << 32) - 777, 3 * (1 << 32) - 5])
@pytest.mark.parametrize("use_poll", [0, 1])
@pytest.mark.parametrize("warps,rounds", [(1, 6), (16, 4), (296, 3)])
def test_fifo_bijection_against_the_model(tq, dev, t0, use_poll, warps, rounds):
    rng = np.random.default_rng(1000 * warps + rounds + use_poll)
    nmine = rng.integers(0, 33, size=(warps, rounds, 32)).astype(np.uint32)
    nmine[0, 0, :] = 0                      # a round where the whole warp enqueues nothing
    nmine[0, 1 % rounds, :] = 32            # a full warp of full lanes (1,024 items)
    total = int(nmine.sum())
    c, enq, deq, out = run(tq, dev, 1 << 22, t0, nmine, use_poll)
    assert c["status"] == STATUS_RUNNING
    assert c["front"] == c["rear"] == t0 + total
    assert int(out[0]) == total and int(out[1]) == total
    # one AFA per warp operation: enqueue once per round, dequeue once per 32 items
    exp_atomics = sum(1 + (-(-int(nmine[w, r].sum()) // 32)) if nmine[w, r].sum() else 0
                      for w in range(warps) for r in range(rounds))
    assert int(out[2]) == exp_atomics
    assert np.array_equal(np.sort(enq[:total]), expected_items(nmine))
    assert np.array_equal(replay(enq, total), deq[:total])


@pytest.mark.parametrize("t0", [0, (1 << 32) - 40])
def test_queue_full_abort_matches_the_model(tq, dev, t0):
    """One warp, C = 64: a round of 100 items must abort at ticket 64 (slot 0
    still holds ticket 0's untaken item), exactly 64 items fit, and rounds of
    <= 64 that are drained before the next never abort however many tickets
    they use in total (the model decides each case the same way)."""
    cap = 64
    cases = {"over": [100], "exact": [64], "drained": [64, 50, 64, 33, 64]}
    for name, per_round in cases.items():
        nmine = np.zeros((1, len(per_round), 32), dtype=np.uint32)
        for r, k in enumerate(per_round):
            nmine[0, r, :k // 4] = 4
            nmine[0, r, k // 4] = k % 4
        m = oracle.QueueModel(capacity=cap, max_tickets=4096)
        for r in range(len(per_round)):
            items = np.arange(int(nmine[0, r].sum()), dtype=np.uint32)
            m.enqueue_n(items)
            if m.aborted:
                break
            b = m.dequeue_n(items.size)
            for t in range(items.size):
                m.take(b + t)
        c, enq, deq, out = run(tq, dev, cap, t0, nmine, use_poll=0)
        assert (c["status"] == STATUS_FULL) == m.aborted, name
        if not m.aborted:
            total = int(nmine.sum())
            assert c["front"] == c["rear"] == t0 + total
            assert np.array_equal(replay(enq, total), deq[:total])
    assert oracle.QueueModel(capacity=cap, max_tickets=256).enqueue_n(np.arange(100)) == 0
