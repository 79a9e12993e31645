"""oracle/ -- TEST INFRASTRUCTURE, NOT PRODUCT CODE.

Python face of the plain sequential CPU oracle in `oracle/oracle.c` (see its
header for what each function computes and which PAPER.md passage it follows).
Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s `cpu_baseline` /
`--impl reference` legs may import this package. The product path
(`paper_conf_icpp_troendletj19_b200`) never imports it, and this package
never imports the product path: the two share no code. The only common
dependency is `inputs/` (seeded input generators, no method arithmetic).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

OQ_DNA = 0xFFFFFFFFFFFFFFFF

VALIDATE_RULES = {
    0: "ok",
    1: "root: parent[root] != root or level[root] != 0",
    2: "reached-ness / id range / level-0 uniqueness",
    3: "tree edge (parent[v], v) is not a graph edge",
    4: "level[v] != level[parent[v]] + 1",
    5: "graph edge crosses reached/unreached or spans > 1 level",
}


def build(force: bool = False) -> str:
    """Compile liboracle.so with plain gcc (-O2, no OpenMP: single core)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=gnu11", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        i64, i32, u64, dbl = ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64, ctypes.c_double
        vp = ctypes.c_void_p
        L.oracle_bfs_levels.argtypes = [i64, vp, vp, i32, vp]
        L.oracle_bfs_levels.restype = i64
        L.oracle_min_id_parents.argtypes = [i64, vp, vp, vp, i32, vp]
        L.oracle_min_id_parents.restype = ctypes.c_int
        L.oracle_bfs.argtypes = [i64, vp, vp, i32, vp, vp, ctypes.POINTER(dbl), ctypes.POINTER(dbl)]
        L.oracle_bfs.restype = i64
        L.oracle_traversed_edges.argtypes = [i64, vp, vp]
        L.oracle_traversed_edges.restype = i64
        L.oracle_validate_tree.argtypes = [i64, vp, vp, i32, vp, vp, ctypes.POINTER(i64)]
        L.oracle_validate_tree.restype = ctypes.c_int
        L.oracle_sssp.argtypes = [i64, vp, vp, vp, i32, vp, vp]
        L.oracle_sssp.restype = i64
        L.oq_create.argtypes = [u64, u64]
        L.oq_create.restype = vp
        L.oq_destroy.argtypes = [vp]
        L.oq_start_at.argtypes = [vp, u64]
        L.oq_start_at.restype = ctypes.c_int
        L.oq_front.argtypes = [vp]
        L.oq_front.restype = u64
        L.oq_rear.argtypes = [vp]
        L.oq_rear.restype = u64
        L.oq_aborted.argtypes = [vp]
        L.oq_aborted.restype = ctypes.c_int
        L.oq_dequeue_n.argtypes = [vp, u64]
        L.oq_dequeue_n.restype = u64
        L.oq_enqueue_n.argtypes = [vp, vp, u64]
        L.oq_enqueue_n.restype = u64
        L.oq_take.argtypes = [vp, u64]
        L.oq_take.restype = u64
        L.oq_replay.argtypes = [u64, vp, u64, u64, vp]
        L.oq_replay.restype = dbl
        _lib = L
    return _lib


def _arr(a, dtype):
    a = np.ascontiguousarray(a, dtype=dtype)
    return a, a.ctypes.data


def bfs(row_ptr, col, root: int, parents: bool = True):
    """Sequential BFS: returns (level int32[V], parent int32[V] or None, info).

    info = {"reached", "seconds_levels", "seconds_total", "traversed_edges"}.
    """
    rp, rpp = _arr(row_ptr, np.int64)
    c, cp = _arr(col, np.int32)
    n = rp.size - 1
    level = np.empty(n, dtype=np.int32)
    parent = np.empty(n, dtype=np.int32) if parents else None
    sl, st = ctypes.c_double(), ctypes.c_double()
    reached = lib().oracle_bfs(n, rpp, cp, int(root), level.ctypes.data,
                               parent.ctypes.data if parents else None,
                               ctypes.byref(sl), ctypes.byref(st))
    if reached < 0:
        raise ValueError("oracle_bfs: bad arguments")
    te = lib().oracle_traversed_edges(n, rpp, level.ctypes.data)
    return level, parent, {"reached": int(reached), "seconds_levels": sl.value,
                           "seconds_total": st.value, "traversed_edges": int(te)}


def bfs_levels(row_ptr, col, root: int) -> np.ndarray:
    return bfs(row_ptr, col, root, parents=False)[0]


def min_id_parents(row_ptr, col, level, root: int) -> np.ndarray:
    rp, rpp = _arr(row_ptr, np.int64)
    c, cp = _arr(col, np.int32)
    lv, lvp = _arr(level, np.int32)
    parent = np.empty(rp.size - 1, dtype=np.int32)
    if lib().oracle_min_id_parents(rp.size - 1, rpp, cp, lvp, int(root), parent.ctypes.data):
        raise ValueError("oracle_min_id_parents: bad arguments")
    return parent


def traversed_edges(row_ptr, level) -> int:
    rp, rpp = _arr(row_ptr, np.int64)
    lv, lvp = _arr(level, np.int32)
    return int(lib().oracle_traversed_edges(rp.size - 1, rpp, lvp))


def validate_tree(row_ptr, col, root: int, level, parent):
    """Graph500-style validation; returns (rule, bad_vertex), rule 0 = valid."""
    rp, rpp = _arr(row_ptr, np.int64)
    c, cp = _arr(col, np.int32)
    lv, lvp = _arr(level, np.int32)
    pa, pap = _arr(parent, np.int32)
    bad = ctypes.c_int64()
    rule = lib().oracle_validate_tree(rp.size - 1, rpp, cp, int(root), lvp, pap, ctypes.byref(bad))
    return int(rule), int(bad.value)


UNREACHED_DIST = 0xFFFFFFFF


def sssp(row_ptr, col, weights, src: int):
    """Dijkstra (oracle.c 4b): returns (dist uint32[V], parent int32[V], reached)."""
    rp, rpp = _arr(row_ptr, np.int64)
    c, cp = _arr(col, np.int32)
    w, wp = _arr(weights, np.int32)
    if w.size != c.size or (w.size and w.min() < 1):
        raise ValueError("one weight >= 1 per CSR entry")
    n = rp.size - 1
    dist = np.empty(n, dtype=np.uint32)
    parent = np.empty(n, dtype=np.int32)
    reached = lib().oracle_sssp(n, rpp, cp, wp, int(src), dist.ctypes.data, parent.ctypes.data)
    if reached < 0:
        raise ValueError("oracle_sssp: bad arguments")
    return dist, parent, int(reached)


class QueueModel:
    """Sequential ticket model of the RF/AN queue (oracle.c section 5)."""

    def __init__(self, capacity: int, max_tickets: int):
        self._q = lib().oq_create(capacity, max_tickets)
        if not self._q:
            raise MemoryError("oq_create failed")
        self.capacity = capacity

    def __del__(self):
        q = getattr(self, "_q", None)
        if q:
            lib().oq_destroy(q)
            self._q = None

    def start_at(self, ticket: int):
        if lib().oq_start_at(self._q, ticket):
            raise ValueError("start_at beyond max_tickets")

    @property
    def front(self) -> int:
        return int(lib().oq_front(self._q))

    @property
    def rear(self) -> int:
        return int(lib().oq_rear(self._q))

    @property
    def aborted(self) -> bool:
        return bool(lib().oq_aborted(self._q))

    def dequeue_n(self, k: int) -> int:
        return int(lib().oq_dequeue_n(self._q, k))

    def enqueue_n(self, items) -> int:
        a, ap = _arr(items, np.uint32)
        base = int(lib().oq_enqueue_n(self._q, ap, a.size))
        if base == OQ_DNA:
            raise ValueError("model ticket space exhausted")
        return base

    def take(self, ticket: int):
        """Item at `ticket`, or None for the data-not-arrived sentinel."""
        r = int(lib().oq_take(self._q, ticket))
        return None if r == OQ_DNA else r


def queue_replay(capacity: int, items, batch: int):
    """Time the sequential model pushing `items` through in batches of `batch`.

    Returns (seconds, (count, sum, xor) fingerprint of dequeued items).
    """
    a, ap = _arr(items, np.uint32)
    fp = np.zeros(3, dtype=np.uint64)
    sec = lib().oq_replay(capacity, ap, a.size, batch, fp.ctypes.data)
    if sec < 0:
        raise RuntimeError("queue_replay failed (code %s)" % sec)
    return sec, (int(fp[0]), int(fp[1]), int(fp[2]))
