"""GPU queue micro-benchmark checks (tq_bench through the C ABI): every queue
variant conserves the multiset of items (every enqueued item dequeued exactly
once), and with full logs the ticket -> item maps of enqueue and dequeue are
the same bijection (FIFO hand-off), checked by the sequential model."""
import numpy as np
import pytest

import oracle
from inputs import fingerprint, item_of

pytestmark = pytest.mark.gpu

VARIANTS = ["rf_an", "per_thread_afa", "cas_retry", "an", "rf_an_cta"]


@pytest.fixture(scope="module")
def tq():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_icpp_troendletj19_b200 as m
    return m


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("warps,batch", [(1, 1), (1, 32), (7, 5), (64, 32), (0, 8)])
def test_conservation(tq, variant, warps, batch):
    items = 1 << 16 if warps else 1 << 22  # full occupancy needs >= 1 item per lane
    r = tq.queue_bench(variant, warps=warps, batch=batch, items=items, capacity=1 << 20,
                       seed=11, timeout_s=30)
    exp = fingerprint(item_of(11, np.arange(r["items"])))
    assert (r["enq"], r["sum_enq"], r["xor_enq"]) == exp
    assert (r["deq"], r["sum_deq"], r["xor_deq"]) == exp
    if variant == "rf_an":
        # one atomic per warp operation: 2 per iteration per warp
        per_item = r["atomics"] / r["items"]
        assert per_item == pytest.approx(2.0 / batch)


@pytest.mark.parametrize("variant", VARIANTS)
def test_full_logs_are_a_fifo_bijection(tq, variant):
    r = tq.queue_bench(variant, warps=32, batch=16, items=1 << 15, capacity=1 << 12, seed=5,
                       log=True, timeout_s=30)
    n = r["items"]
    enq = r["enq_log"][:n].cpu().numpy().view(np.uint32)
    deq = r["deq_log"][:n].cpu().numpy().view(np.uint32)
    # the sequential model replays the GPU's reservation order: the item that
    # was enqueued at ticket t must be the one the holder of ticket t took
    q = oracle.QueueModel(capacity=n, max_tickets=n)
    q.enqueue_n(enq)
    base = q.dequeue_n(n)
    expected = np.array([q.take(base + t) for t in range(n)], dtype=np.uint32)
    assert np.array_equal(expected, deq)
    assert np.unique(enq).size == n
    assert set(enq.tolist()) == set(item_of(5, np.arange(n)).tolist())


def test_queue_full_is_reported(tq):
    # capacity smaller than the in-flight items is rejected up front
    with pytest.raises(tq.TQError):
        tq.queue_bench("rf_an", warps=64, batch=32, items=1 << 14, capacity=256)


def test_atomic_ceiling_runs(tq):
    r = tq.queue_bench("atomic_ceiling", warps=0, batch=32, items=1 << 22)
    assert r["atomics"] == r["items"] // 32


def test_queue_object_roundtrip(tq):
    q = tq.Queue(1000)
    assert q.capacity == 1024
    c = q.counters()
    assert (c["front"], c["rear"], c["done"], c["status"]) == (0, 0, 0, 0)
    q.reset()
    q.close()
    with pytest.raises(tq.TQError):
        tq.Queue(1)
