"""Python binding of the tq C ABI (include/tq.h): argument marshalling only.

Every step of the hot path runs in libtq.so's CUDA kernels; this module only
turns torch tensors / numpy arrays into pointers and status codes into
exceptions. PyTorch is used for device memory and streams.
"""
from __future__ import annotations

import ctypes
from typing import Optional

import numpy as np

from . import _lib
from ._lib import TQError, VARIANTS, check, lib

__all__ = ["bfs", "BfsPlan", "Queue", "queue_bench", "persistent_threads", "TQError", "VARIANTS",
           "version"]


def _torch():
    import torch
    return torch


def _is_tensor(x) -> bool:
    try:
        import torch
        return isinstance(x, torch.Tensor)
    except ImportError:  # pragma: no cover
        return False


def _ptr(x) -> Optional[int]:
    if x is None:
        return None
    if _is_tensor(x):
        if not x.is_contiguous():
            raise ValueError("tensor must be contiguous")
        return x.data_ptr()
    if isinstance(x, np.ndarray):
        if not x.flags.c_contiguous:
            raise ValueError("array must be C-contiguous")
        return x.ctypes.data
    raise TypeError(f"expected a torch.Tensor or numpy.ndarray, got {type(x)}")


def _variant(v) -> int:
    if isinstance(v, str):
        return VARIANTS[v]
    return int(v)


def _stream_ptr(stream, like=None) -> Optional[int]:
    if stream is not None:
        return stream if isinstance(stream, int) else stream.cuda_stream
    if like is not None and _is_tensor(like) and like.is_cuda:
        torch = _torch()
        return torch.cuda.current_stream(like.device).cuda_stream
    return None


def _csr(row_ptr, col) -> _lib.tq_csr:
    n = int(row_ptr.shape[0]) - 1
    nnz = int(col.shape[0])
    if _is_tensor(row_ptr):
        torch = _torch()
        if row_ptr.dtype != torch.int64 or col.dtype != torch.int32:
            raise TypeError("row_ptr must be int64 and col int32")
    else:
        if row_ptr.dtype != np.int64 or col.dtype != np.int32:
            raise TypeError("row_ptr must be int64 and col int32")
    return _lib.tq_csr(n, nnz, _ptr(row_ptr), _ptr(col))


def _opts(variant="rf_an", capacity=0, threads=0, block=0, chunk=0, stream=None, timeout_s=0.0,
          backoff_ns=0, device=0, parents="any", hub_queue=True, debug_delay_ns=0,
          debug_delay_seed=0, cas_backoff_ns=0, mirror_bits=0, deep_grid=True, ticket_lanes=0,
          l2_persist=True, smem_path=0, relabel=0, level_bits=0) -> _lib.bfs_opts:
    return _lib.bfs_opts(int(capacity), int(threads), int(block), int(chunk), _variant(variant),
                         stream, float(timeout_s), int(backoff_ns), int(device),
                         _lib.PARENT_RULES[parents] if isinstance(parents, str) else int(parents),
                         0 if hub_queue else -1, int(debug_delay_ns), int(debug_delay_seed) & 0xFFFFFFFF,
                         int(cas_backoff_ns), int(mirror_bits), 0 if deep_grid else -1, int(ticket_lanes),
                         0 if l2_persist else -1,
                         int(smem_path) if not isinstance(smem_path, bool) else (1 if smem_path else -1),
                         int(relabel) if not isinstance(relabel, bool) else (1 if relabel else -1),
                         int(level_bits))


# bfs / BfsPlan keyword options that map one to one onto bfs_opts fields
_OPT_KEYS = ("variant", "capacity", "threads", "chunk", "timeout_s", "backoff_ns", "parents", "hub_queue",
             "debug_delay_ns", "debug_delay_seed", "cas_backoff_ns", "mirror_bits", "deep_grid", "ticket_lanes",
             "l2_persist", "smem_path", "relabel", "level_bits")


def _stats_dict(st: _lib.bfs_stats) -> dict:
    return {f: getattr(st, f) for f, _ in st._fields_}


def _empty_like_graph(row_ptr, n):
    if _is_tensor(row_ptr):
        torch = _torch()
        return torch.empty(n, dtype=torch.int32, device=row_ptr.device)
    return np.empty(n, dtype=np.int32)


def bfs(row_ptr, col, root: int, level=None, parent=None, *, want_parent: bool = True, stream=None,
        device: int = 0, **opts):
    """One-shot `bfs_run_ex`: returns (level, parent, stats).

    Graph arrays may be CUDA tensors (used in place) or host numpy arrays
    (staged to the device by the library). Outputs default to the graph's
    kind of memory. `opts`: the bfs_opts fields (variant, capacity, threads,
    chunk, timeout_s, backoff_ns, parents, hub_queue, debug_delay_ns,
    debug_delay_seed, cas_backoff_ns, mirror_bits, deep_grid, ticket_lanes, l2_persist,
    smem_path: 0 auto, -1 / False off, 1 / True required; relabel: 0 auto, -1 / False off,
    1 / True on; level_bits: test-only cap of the tokens' level field).
    """
    bad = set(opts) - set(_OPT_KEYS)
    if bad:
        raise TypeError(f"unknown options {sorted(bad)}")
    g = _csr(row_ptr, col)
    n = g.n_vertices
    if level is None:
        level = _empty_like_graph(row_ptr, n)
    if parent is None and want_parent:
        parent = _empty_like_graph(row_ptr, n)
    o = _opts(stream=_stream_ptr(stream, row_ptr),
              device=row_ptr.device.index if _is_tensor(row_ptr) and row_ptr.is_cuda else device, **opts)
    st = _lib.bfs_stats()
    check(lib().bfs_run_ex(ctypes.byref(g), int(root), _ptr(level), _ptr(parent), ctypes.byref(o),
                           ctypes.byref(st)), "bfs_run_ex")
    return level, parent, _stats_dict(st)


class BfsPlan:
    """`bfs_plan_create` / `bfs_plan_run` / `bfs_plan_destroy`.

    Static allocation before launch: graph view, queue, W and the
    chunk table live for the plan's lifetime; `run` only launches.
    """

    def __init__(self, row_ptr, col, *, stream=None, device: int = 0, **opts):
        bad = set(opts) - set(_OPT_KEYS)
        if bad:
            raise TypeError(f"unknown options {sorted(bad)}")
        self._keep = (row_ptr, col)  # device arrays must outlive the plan
        self._g = _csr(row_ptr, col)
        self.n_vertices = self._g.n_vertices
        self.nnz = self._g.nnz
        self.device = row_ptr.device.index if _is_tensor(row_ptr) and row_ptr.is_cuda else device
        self._opts = _opts(stream=_stream_ptr(stream, row_ptr), device=self.device, **opts)
        self.regrows = 0
        self._h = None
        self._create()

    def _create(self):
        h = ctypes.c_void_p()
        check(lib().bfs_plan_create(ctypes.byref(self._g), ctypes.byref(self._opts), ctypes.byref(h)),
              "bfs_plan_create")
        self._h = h

    # the largest queue the library builds (tq_create: C <= 2^31)
    MAX_CAPACITY = 1 << 31
    MAX_REGROWS = 12

    def _grow(self) -> bool:
        """Queue-full answer of the paper: re-create the plan with
        twice the queue capacity (the chunk queue follows it). False once the
        capacity cannot grow any more or MAX_REGROWS retries were spent."""
        cap = self._opts.capacity or 2 * max(self.n_vertices, 1 << 15)
        new = min(2 * max(cap, 1 << 16), self.MAX_CAPACITY)
        if new <= (self._opts.capacity or 0) or self.regrows >= self.MAX_REGROWS:
            return False
        self._opts.capacity = new
        self.close()
        self._create()
        self.regrows += 1
        return True

    def run(self, root: int, level=None, parent=None, grow_on_full: bool = False) -> dict:
        """One BFS. With grow_on_full, a queue-full abort (TQ_ERR_QUEUE_FULL)
        is answered as the paper suggests: re-create the plan with
        twice the queue capacity and run again (counted in `regrows`), at most
        MAX_REGROWS times and never past MAX_CAPACITY; then the error is raised."""
        while True:
            st = _lib.bfs_stats()
            status = lib().bfs_plan_run(self._h, int(root), _ptr(level), _ptr(parent), ctypes.byref(st))
            if status == _lib.TQ_ERR_QUEUE_FULL and grow_on_full and self._grow():
                continue
            check(status, "bfs_plan_run")
            return _stats_dict(st)

    def set_tickets(self, t_main: int, t_chunk: int = 0):
        """`bfs_plan_set_tickets`: restart the queues at these tickets (tests of
        the 32-bit sequence-tag wrap)."""
        check(lib().bfs_plan_set_tickets(self._h, int(t_main), int(t_chunk)), "bfs_plan_set_tickets")

    def tickets(self) -> tuple:
        """`bfs_plan_get_tickets`: (main-queue ticket, chunk-queue ticket) where
        the next run starts."""
        a, b = ctypes.c_uint64(), ctypes.c_uint64()
        check(lib().bfs_plan_get_tickets(self._h, ctypes.byref(a), ctypes.byref(b)), "bfs_plan_get_tickets")
        return a.value, b.value

    def run_batch(self, roots, level=None, parent=None, stride: int | None = None) -> list:
        """`bfs_plan_run_batch`: root i writes level[i * stride:] / parent[...].
        stride defaults to n_vertices when the outputs hold len(roots) rows,
        else 0 (one reused buffer). Host outputs are copied on a second stream
        overlapped with the next BFS. Returns the per-root statistics."""
        r = np.ascontiguousarray(np.asarray(roots, dtype=np.int32))
        n = r.size
        if stride is None:
            size = level.shape[0] if level is not None else (parent.shape[0] if parent is not None else 0)
            stride = self.n_vertices if size >= n * self.n_vertices and n > 1 else 0
        sts = (_lib.bfs_stats * max(n, 1))()
        check(lib().bfs_plan_run_batch(self._h, r.ctypes.data, n, _ptr(level), _ptr(parent), int(stride),
                                       ctypes.cast(sts, ctypes.c_void_p)), "bfs_plan_run_batch")
        return [_stats_dict(sts[i]) for i in range(n)]

    def launch(self, root: int, level=None, parent=None):
        """Enqueue one BFS on the plan's stream and return (bfs_plan_launch)."""
        check(lib().bfs_plan_launch(self._h, int(root), _ptr(level), _ptr(parent)), "bfs_plan_launch")

    def wait(self) -> dict:
        """Block until the launched BFS finished; its statistics (bfs_plan_wait)."""
        st = _lib.bfs_stats()
        check(lib().bfs_plan_wait(self._h, ctypes.byref(st)), "bfs_plan_wait")
        return _stats_dict(st)

    def close(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value:
            lib().bfs_plan_destroy(h)
        self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


class SsspPlan(BfsPlan):
    """`sssp_plan_create` / `sssp_plan_run`: label-correcting shortest paths on
    the same queue and persistent kernel (include/tq.h, NEXT row 4). `weights`
    is int32[nnz] (>= 1), host or device like the CSR."""

    def __init__(self, row_ptr, col, weights, *, stream=None, device: int = 0, **opts):
        self._w = weights
        opts = dict(opts, variant="rf_an", parents="min_id")
        super().__init__(row_ptr, col, stream=stream, device=device, **opts)

    def _create(self):
        h = ctypes.c_void_p()
        check(lib().sssp_plan_create(ctypes.byref(self._g), _ptr(self._w), ctypes.byref(self._opts),
                                     ctypes.byref(h)), "sssp_plan_create")
        self._h = h

    def run(self, src: int, dist=None, parent=None, grow_on_full: bool = False) -> dict:
        """dist: uint32/int32 buffer (0xFFFFFFFF = unreached)."""
        while True:
            st = _lib.bfs_stats()
            status = lib().sssp_plan_run(self._h, int(src), _ptr(dist), _ptr(parent), ctypes.byref(st))
            if status == _lib.TQ_ERR_QUEUE_FULL and grow_on_full and self._grow():
                continue
            check(status, "sssp_plan_run")
            return _stats_dict(st)


def sssp(row_ptr, col, weights, src: int, dist=None, parent=None, **opts):
    """One-shot shortest paths: returns (dist, parent, stats); dist as int32
    holding uint32 bits (0xFFFFFFFF = unreached)."""
    n = int(row_ptr.shape[0]) - 1
    if dist is None:
        dist = _empty_like_graph(row_ptr, n)
    if parent is None:
        parent = _empty_like_graph(row_ptr, n)
    with SsspPlan(row_ptr, col, weights, **opts) as p:
        st = p.run(src, dist, parent)
    return dist, parent, st


def run_concurrent(plans, roots, levels=None, parents=None):
    """Run `roots` over several plans (each on its own stream) keeping one BFS
    in flight per plan; returns the per-root statistics in root order."""
    out = [None] * len(roots)
    busy = {}  # plan index -> root index
    nxt = 0
    k = len(plans)
    while nxt < len(roots) or busy:
        for i in range(k):
            if i not in busy and nxt < len(roots):
                plans[i].launch(roots[nxt], levels[i] if levels else None, parents[i] if parents else None)
                busy[i] = nxt
                nxt += 1
        # wait for the oldest launch first (launch order == root order)
        i = min(busy, key=busy.get)
        out[busy.pop(i)] = plans[i].wait()
    return out


class Queue:
    """A device queue object (`tq_create` ... `tq_destroy`)."""

    def __init__(self, capacity: int, device: int = 0):
        h = ctypes.c_void_p()
        check(lib().tq_create(int(capacity), int(device), ctypes.byref(h)), "tq_create")
        self._h = h

    def reset(self, stream=None):
        check(lib().tq_reset(self._h, stream), "tq_reset")

    def reset_at(self, ticket: int, stream=None):
        """`tq_reset_at`: empty queue with Front = Rear = Done = ticket."""
        check(lib().tq_reset_at(self._h, int(ticket), stream), "tq_reset_at")

    def view(self) -> _lib.tq_device_view:
        v = _lib.tq_device_view()
        check(lib().tq_device_view_get(self._h, ctypes.byref(v)), "tq_device_view_get")
        return v

    def counters(self) -> dict:
        c = _lib.tq_counters()
        check(lib().tq_counters_get(self._h, ctypes.byref(c)), "tq_counters_get")
        return {"front": c.front, "rear": c.rear, "done": c.done, "status": c.status}

    @property
    def capacity(self) -> int:
        return int(self.view().mask) + 1

    def close(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value:
            lib().tq_destroy(h)
        self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def queue_bench(variant="rf_an", *, warps: int = 0, batch: int = 32, items: int = 1 << 24,
                capacity: int = 1 << 20, work_iters: int = 0, seed: int = 3, log: bool = False,
                stream=None, timeout_s: float = 0.0, device: int = 0, depth: int = 1,
                cluster: int = 0, cas_backoff_ns: int = 0, relaxed_poll: bool = False) -> dict:
    """`tq_bench`: enqueue/dequeue throughput of one queue variant.

    depth=2 pipelines one iteration ahead (rf_an, rf_an_cta; rf_an_cluster
    always); cluster = CTAs per proxy group of rf_an_cluster (0 -> 4).
    With log=True returns 'enq_log' / 'deq_log' (ticket -> item, CUDA tensors).
    """
    enq_log = deq_log = None
    if log:
        torch = _torch()
        enq_log = torch.zeros(items, dtype=torch.int32, device=f"cuda:{device}")
        deq_log = torch.zeros(items, dtype=torch.int32, device=f"cuda:{device}")
    cfg = _lib.tq_bench_cfg(_variant(variant), int(warps), int(batch), int(items), int(capacity),
                            int(work_iters), int(seed), int(log), _ptr(enq_log), _ptr(deq_log),
                            _stream_ptr(stream), float(timeout_s), int(device), int(depth), int(cluster),
                            int(cas_backoff_ns), int(bool(relaxed_poll)))
    res = _lib.tq_bench_result()
    status = lib().tq_bench(ctypes.byref(cfg), ctypes.byref(res))
    out = {f: getattr(res, f) for f, _ in res._fields_}
    out["status"] = status
    if log:
        out["enq_log"], out["deq_log"] = enq_log, deq_log
    if status not in (_lib.TQ_OK,):
        raise TQError(status, "tq_bench")
    return out


def persistent_threads(variant="rf_an", device: int = 0) -> int:
    t = ctypes.c_int()
    check(lib().tq_persistent_threads(_variant(variant), 256, int(device), ctypes.byref(t)),
          "tq_persistent_threads")
    return t.value


def probe_ceiling(table_bytes: int, probes: int = 1 << 28, device: int = 0, stream=None) -> float:
    """G random L2 byte probes per second on this GPU (tq_probe_ceiling): the
    ceiling of the BFS expansion's mirror probes."""
    g = ctypes.c_double()
    check(lib().tq_probe_ceiling(int(device), int(table_bytes), int(probes), _stream_ptr(stream),
                                 ctypes.byref(g)), "tq_probe_ceiling")
    return g.value


def memory_trim(device: int = 0) -> None:
    """`tq_memory_trim`: release the library pool's cached device memory."""
    check(lib().tq_memory_trim(int(device)), "tq_memory_trim")


def version() -> str:
    return lib().tq_version().decode()
