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


# Pipelined groups (tq_bench_cfg.depth = 2): warp, CTA and cluster proxies.
PIPED = [("rf_an_cta", 0), ("rf_an_cluster", 2), ("rf_an_cluster", 4),
         ("rf_an_cluster", 8), ("rf_an_cluster", 16)]


@pytest.mark.parametrize("variant,cluster", PIPED)
@pytest.mark.parametrize("warps,batch", [(128, 1), (128, 32), (0, 8), (0, 32)])
def test_pipelined_conservation(tq, variant, cluster, warps, batch):
    items = 1 << 16 if warps else 1 << 23
    try:
        r = tq.queue_bench(variant, warps=warps, batch=batch, items=items, capacity=1 << 20, seed=13,
                           timeout_s=30, depth=2, cluster=cluster)
    except tq.TQError as e:  # a 16-CTA cluster may not be schedulable on this part
        if cluster == 16 and e.status == -1:
            pytest.skip("16-CTA clusters not co-resident here")
        raise
    exp = fingerprint(item_of(13, np.arange(r["items"])))
    assert (r["enq"], r["sum_enq"], r["xor_enq"]) == exp
    assert (r["deq"], r["sum_deq"], r["xor_deq"]) == exp
    group = {"rf_an_cta": 8, "rf_an_cluster": 8 * cluster}[variant]
    # one atomic on Rear and one on Front per proxy group per iteration
    assert r["atomics"] / r["items"] == pytest.approx(2.0 / (batch * group))


@pytest.mark.parametrize("variant,cluster", PIPED[:4])
def test_pipelined_logs_are_a_fifo_bijection(tq, variant, cluster):
    r = tq.queue_bench(variant, warps=64, batch=16, items=1 << 15, capacity=1 << 12, seed=7,
                       log=True, timeout_s=30, depth=2, cluster=cluster)
    n = r["items"]
    enq = r["enq_log"][:n].cpu().numpy().view(np.uint32)
    deq = r["deq_log"][:n].cpu().numpy().view(np.uint32)
    q = oracle.QueueModel(capacity=n, max_tickets=n)
    q.enqueue_n(enq)
    base = q.dequeue_n(n)
    expected = np.array([q.take(base + t) for t in range(n)], dtype=np.uint32)
    assert np.array_equal(expected, deq)
    assert set(enq.tolist()) == set(item_of(7, np.arange(n)).tolist())


def test_pipelined_argument_checks(tq):
    with pytest.raises(tq.TQError):  # not a multiple of 8 warps per CTA x cluster
        tq.queue_bench("rf_an_cluster", warps=24, batch=4, items=1 << 14, cluster=4)
    with pytest.raises(tq.TQError):  # pipelining is for CTA / cluster proxy groups only
        tq.queue_bench("cas_retry", warps=8, batch=4, items=1 << 14, depth=2)
    with pytest.raises(tq.TQError):
        tq.queue_bench("rf_an", warps=8, batch=4, items=1 << 14, depth=2)
    with pytest.raises(tq.TQError):  # two iterations in flight must fit the ring
        tq.queue_bench("rf_an_cta", warps=64, batch=32, items=1 << 14, capacity=2048, depth=2)


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
