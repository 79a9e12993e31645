"""Pins for the sequential queue model (oracle/oracle.c section 5) and a
brute-force model check of the {seq, item} slot protocol the CUDA queue uses.

Pins come from the paper's text: the worked dequeue example (PAPER.md:167-171,
tests/golden/p167_dequeue_example.json), the queue-full rule (Listing 3
line 25, P:71 fn2), the arrival check (Listing 2) and FIFO
hand-off.
"""
import json
import os

import numpy as np
import pytest

import oracle
from inputs import fingerprint, item_of

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def test_paper_worked_dequeue_example():
    ex = json.load(open(os.path.join(GOLDEN, "p167_dequeue_example.json")))
    q = oracle.QueueModel(capacity=8, max_tickets=16)
    q.start_at(ex["front_before"])  # tickets 0, 1 already consumed
    q.enqueue_n([101, 102])  # data present in slots 2 and 3 (Figure 2)
    assert q.rear == ex["rear_before"]
    base = q.dequeue_n(ex["hungry"])  # the proxy's single atomic_fetch_add(Front, 3)
    assert base == ex["start_slot_index"]
    assert q.front == ex["front_after"]
    slots = [base + i for i in range(ex["hungry"])]
    assert slots == ex["assigned_slots"]
    arrived = [q.take(t) is not None for t in slots[:2]] + [q.take(slots[2]) is not None]
    assert arrived == ex["data_arrived"]
    # the third thread keeps its slot and sees the data when it arrives
    q.enqueue_n([103])
    assert q.take(4) == 103


def test_take_is_once_and_fifo():
    q = oracle.QueueModel(capacity=16, max_tickets=64)
    items = [7, 8, 9, 10, 11]
    base = q.enqueue_n(items)
    t = q.dequeue_n(5)
    assert (base, t) == (0, 0)
    got = [q.take(t + i) for i in range(5)]
    assert got == items  # ticket t receives the item enqueued at ticket t
    assert all(q.take(t + i) is None for i in range(5))  # slot now holds dna again
    assert q.take(5) is None  # beyond Rear: data not arrived


@pytest.mark.parametrize("cap", [1, 2, 4, 8])
def test_queue_full_rule(cap):
    # exactly C outstanding items never abort; the (C+1)-th does
    q = oracle.QueueModel(capacity=cap, max_tickets=64)
    q.enqueue_n(list(range(cap)))
    assert not q.aborted
    q.enqueue_n([999])
    assert q.aborted
    # same, but ticket 0 is taken first: the slot is free again, no abort
    q = oracle.QueueModel(capacity=cap, max_tickets=64)
    q.enqueue_n(list(range(cap)))
    q.dequeue_n(1)
    assert q.take(0) == 0
    q.enqueue_n([999])
    assert not q.aborted
    # reserved-but-untaken (dequeued, not yet arrived-checked) still blocks
    q = oracle.QueueModel(capacity=cap, max_tickets=64)
    q.enqueue_n(list(range(cap)))
    q.dequeue_n(1)
    q.enqueue_n([999])
    assert q.aborted


def test_never_aborts_within_capacity_random():
    rng = np.random.default_rng(0)
    for trial in range(50):
        cap = int(2 ** rng.integers(0, 6))
        q = oracle.QueueModel(capacity=cap, max_tickets=4096)
        live = []
        enq = deq = 0
        for _ in range(200):
            if rng.random() < 0.5 and len(live) < cap:
                k = int(rng.integers(1, cap - len(live) + 1))
                items = list(range(enq, enq + k))
                q.enqueue_n(items)
                live += items
                enq += k
            elif live:
                t = q.dequeue_n(1)
                assert q.take(t) == live.pop(0)
                deq += 1
        assert not q.aborted


def test_replay_conserves_multiset():
    seed, n = 3, 5000
    items = item_of(seed, np.arange(n))
    assert np.unique(items).size == n  # unique by construction
    for b in (1, 7, 32):
        sec, fp = oracle.queue_replay(64, items, b)
        assert fp == fingerprint(items)
        assert sec >= 0


# ---------------------------------------------------------------------------
# Model check of the CUDA slot protocol against the ticket model.
#
# Slot i holds (seq, item); initially seq = i. Ticket t maps to slot t mod C.
#   producer writing ticket t: read slot; seq == t -> store (t+1, item),
#                              else queue full -> abort (Listing 3 line 25)
#   consumer holding ticket t: poll slot; seq == t+1 -> take item and store
#                              seq = t + C (slot empty for the next lap)
# Every interleaving of 2 producers x 2 consumers (each producer enqueues
# 1 or 2 items with one arbitrary-n reservation) is explored; at each
# producer check the protocol's decision must equal the ticket model's
# predicate (t >= C and ticket t-C not taken -> abort), each consumer must
# receive exactly the item enqueued at its ticket, and with no abort every
# reserved ticket is eventually taken.
# ---------------------------------------------------------------------------

def _explore(cap, prod_items, n_cons):
    init_slots = tuple((i, None) for i in range(cap))
    # producer state: ("R",) before reservation; ("C", base, i) check item i;
    # ("W", base, i) write item i; ("D",) done
    # consumer state: ("R",) before reservation; ("P", t) polling; ("S", t, item) reset; ("D", t, item)
    start = (init_slots, 0, 0, tuple(("R",) for _ in prod_items), tuple(("R",) for _ in range(n_cons)),
             frozenset(), frozenset(), False, frozenset())
    seen = set()
    stack = [start]
    terminals = 0
    while stack:
        st = stack.pop()
        if st in seen:
            continue
        seen.add(st)
        slots, front, rear, ps, cs, taken, written, aborted, reserved = st
        succ = []
        if not aborted:
            for k, p in enumerate(ps):
                items = prod_items[k]
                if p[0] == "R":
                    nps = list(ps); nps[k] = ("C", rear, 0)
                    res = reserved | {(rear + j, items[j]) for j in range(len(items))}
                    succ.append((slots, front, rear + len(items), tuple(nps), cs, taken, written, False, res))
                elif p[0] == "C":
                    base, i = p[1], p[2]
                    t = base + i
                    seq, _ = slots[t % cap]
                    model_abort = t >= cap and (t - cap) not in taken
                    proto_abort = seq != t
                    assert model_abort == proto_abort, (cap, st)
                    nps = list(ps)
                    if proto_abort:
                        nps[k] = ("D",)
                        succ.append((slots, front, rear, tuple(nps), cs, taken, written, True, reserved))
                    else:
                        nps[k] = ("W", base, i)
                        succ.append((slots, front, rear, tuple(nps), cs, taken, written, False, reserved))
                elif p[0] == "W":
                    base, i = p[1], p[2]
                    t = base + i
                    ns = list(slots); ns[t % cap] = (t + 1, items[i])
                    nps = list(ps)
                    nps[k] = ("C", base, i + 1) if i + 1 < len(items) else ("D",)
                    succ.append((tuple(ns), front, rear, tuple(nps), cs, taken, written | {t}, False, reserved))
            for k, c in enumerate(cs):
                if c[0] == "R":
                    ncs = list(cs); ncs[k] = ("P", front)
                    succ.append((slots, front + 1, rear, ps, tuple(ncs), taken, written, False, reserved))
                elif c[0] == "P":
                    t = c[1]
                    seq, item = slots[t % cap]
                    if seq == t + 1:
                        ncs = list(cs); ncs[k] = ("S", t, item)
                        succ.append((slots, front, rear, ps, tuple(ncs), taken, written, False, reserved))
                elif c[0] == "S":
                    t, item = c[1], c[2]
                    ns = list(slots); ns[t % cap] = (t + cap, None)
                    ncs = list(cs); ncs[k] = ("D", t, item)
                    succ.append((tuple(ns), front, rear, ps, tuple(ncs), taken | {t}, written, False, reserved))
        if not succ:
            terminals += 1
            res = dict(reserved)
            got = [c for c in cs if c[0] in ("S", "D")]
            for c in got:
                assert res[c[1]] == c[2]  # FIFO: ticket t gets the item enqueued at t
            assert len({c[1] for c in got}) == len(got)
            if not aborted:
                for c in cs:
                    if c[0] == "P":
                        assert c[1] >= rear  # only tickets with no data left pending
        stack.extend(succ)
    return terminals, len(seen)


@pytest.mark.parametrize("cap", [2, 4])
@pytest.mark.parametrize("prod_items", [((1,), (2,)), ((1, 2), (3,)), ((1, 2), (3, 4))])
def test_slot_protocol_model_check(cap, prod_items):
    terminals, states = _explore(cap, prod_items, n_cons=2)
    assert terminals > 0 and states > 10


def test_slot_protocol_needs_capacity_two():
    # With C = 1 "item ready for ticket t" (seq = t+1) is indistinguishable
    # from "empty for ticket t+C" (seq = t+C): the checker must find the
    # disagreement, which is why tq_create rejects capacity < 2.
    with pytest.raises(AssertionError):
        _explore(1, ((1,), (2,)), n_cons=2)
