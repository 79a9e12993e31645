"""ctypes mirror of include/tq.h (argument marshalling only).

Loading fails loudly if libtq.so is missing: there is no CPU fallback.
"""
from __future__ import annotations

import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
# TQ_LIB: A/B experiments only (scripts/ab_bfs.sh loads an alternative build)
LIB_PATH = os.environ.get("TQ_LIB") or os.path.join(HERE, "libtq.so")

c_i32, c_i64, c_u32, c_u64, c_dbl, c_vp = (ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32,
                                           ctypes.c_uint64, ctypes.c_double, ctypes.c_void_p)

TQ_OK, TQ_ERR_INVALID, TQ_ERR_CUDA, TQ_ERR_NOMEM, TQ_ERR_QUEUE_FULL, TQ_ERR_TIMEOUT, \
    TQ_ERR_UNSUPPORTED = 0, -1, -2, -3, -4, -5, -6

VARIANTS = {"rf_an": 0, "per_thread_afa": 1, "cas_retry": 2, "an": 3, "atomic_ceiling": 4, "rf_an_cta": 5,
            "rf_an_cluster": 6}
STATUS_NAMES = {0: "running", 1: "finished", 2: "aborted_full", 3: "aborted_timeout"}
PARENT_RULES = {"any": 0, "min_id": 1}


class tq_device_view(ctypes.Structure):
    _fields_ = [("slots", c_vp), ("front", c_vp), ("rear", c_vp), ("done", c_vp),
                ("status", c_vp), ("mask", c_u64), ("log2_capacity", c_u32), ("reserved_", c_u32)]


class tq_counters(ctypes.Structure):
    _fields_ = [("front", c_u64), ("rear", c_u64), ("done", c_u64), ("status", c_u32)]


class tq_csr(ctypes.Structure):
    _fields_ = [("n_vertices", c_i64), ("nnz", c_i64), ("row_ptr", c_vp), ("col", c_vp)]


class bfs_opts(ctypes.Structure):
    _fields_ = [("capacity", c_u64), ("threads", ctypes.c_int), ("block", ctypes.c_int),
                ("chunk", ctypes.c_int), ("variant", ctypes.c_int), ("stream", c_vp),
                ("timeout_s", c_dbl), ("backoff_ns", ctypes.c_int), ("device", ctypes.c_int),
                ("parent_rule", ctypes.c_int), ("hub_queue", ctypes.c_int),
                ("debug_delay_ns", ctypes.c_int), ("debug_delay_seed", c_u32),
                ("cas_backoff_ns", ctypes.c_int), ("mirror_bits", ctypes.c_int), ("deep_grid", ctypes.c_int),
                ("ticket_lanes", ctypes.c_int), ("l2_persist", ctypes.c_int),
                ("smem_path", ctypes.c_int), ("relabel", ctypes.c_int), ("level_bits", ctypes.c_int)]


class bfs_stats(ctypes.Structure):
    _fields_ = [("ms", c_dbl), ("ms_kernel", c_dbl), ("traversed_edges", c_u64), ("reached", c_u64),
                ("tasks", c_u64), ("chunk_tasks", c_u64), ("edges_scanned", c_u64),
                ("min_atomics", c_u64), ("reenqueues", c_u64), ("queue_atomics", c_u64),
                ("cas_failures", c_u64), ("empty_polls", c_u64), ("tickets", c_u64),
                ("busy_cycles", c_u64), ("rounds", c_u64), ("skipped_tasks", c_u64),
                ("max_level", c_i32), ("persistent_threads", c_i32), ("mirror_bits", c_i32),
                ("ticket_lanes", c_i32), ("smem_path", c_i32),
                ("relabelled", c_i32), ("level_tokens", c_i32)]


class tq_bench_cfg(ctypes.Structure):
    _fields_ = [("variant", ctypes.c_int), ("warps", ctypes.c_int), ("batch", ctypes.c_int),
                ("items", c_u64), ("capacity", c_u64), ("work_iters", ctypes.c_int), ("seed", c_u64),
                ("log_mode", ctypes.c_int), ("enq_log", c_vp), ("deq_log", c_vp), ("stream", c_vp),
                ("timeout_s", c_dbl), ("device", ctypes.c_int), ("depth", ctypes.c_int),
                ("cluster", ctypes.c_int), ("cas_backoff_ns", ctypes.c_int), ("relaxed_poll", ctypes.c_int)]


class tq_bench_result(ctypes.Structure):
    _fields_ = [("ms", c_dbl), ("items", c_u64), ("enq", c_u64), ("deq", c_u64), ("atomics", c_u64),
                ("cas_failures", c_u64), ("empty_retries", c_u64), ("sum_enq", c_u64),
                ("sum_deq", c_u64), ("xor_enq", c_u64), ("xor_deq", c_u64), ("warps", c_i32),
                ("status", c_i32)]


# every symbol include/tq.h declares (checked by tests/test_boundary.py)
EXPORTS = {
    "tq_create": (ctypes.c_int, [c_u64, ctypes.c_int, ctypes.POINTER(c_vp)]),
    "tq_destroy": (ctypes.c_int, [c_vp]),
    "tq_reset": (ctypes.c_int, [c_vp, c_vp]),
    "tq_reset_at": (ctypes.c_int, [c_vp, c_u64, c_vp]),
    "tq_device_view_get": (ctypes.c_int, [c_vp, ctypes.POINTER(tq_device_view)]),
    "tq_counters_get": (ctypes.c_int, [c_vp, ctypes.POINTER(tq_counters)]),
    "bfs_run": (ctypes.c_int, [ctypes.POINTER(tq_csr), c_i32, c_vp, c_vp]),
    "bfs_run_ex": (ctypes.c_int, [ctypes.POINTER(tq_csr), c_i32, c_vp, c_vp, ctypes.POINTER(bfs_opts),
                                  ctypes.POINTER(bfs_stats)]),
    "bfs_plan_create": (ctypes.c_int, [ctypes.POINTER(tq_csr), ctypes.POINTER(bfs_opts),
                                       ctypes.POINTER(c_vp)]),
    "bfs_plan_run": (ctypes.c_int, [c_vp, c_i32, c_vp, c_vp, ctypes.POINTER(bfs_stats)]),
    "bfs_plan_destroy": (ctypes.c_int, [c_vp]),
    "bfs_plan_set_tickets": (ctypes.c_int, [c_vp, c_u64, c_u64]),
    "bfs_plan_get_tickets": (ctypes.c_int, [c_vp, ctypes.POINTER(c_u64), ctypes.POINTER(c_u64)]),
    "bfs_plan_launch": (ctypes.c_int, [c_vp, c_i32, c_vp, c_vp]),
    "bfs_plan_wait": (ctypes.c_int, [c_vp, ctypes.POINTER(bfs_stats)]),
    "bfs_plan_run_batch": (ctypes.c_int, [c_vp, c_vp, c_i32, c_vp, c_vp, c_i64, c_vp]),
    "sssp_plan_create": (ctypes.c_int, [ctypes.POINTER(tq_csr), c_vp, ctypes.POINTER(bfs_opts),
                                        ctypes.POINTER(c_vp)]),
    "sssp_plan_run": (ctypes.c_int, [c_vp, c_i32, c_vp, c_vp, ctypes.POINTER(bfs_stats)]),
    "sssp_run_ex": (ctypes.c_int, [ctypes.POINTER(tq_csr), c_vp, c_i32, c_vp, c_vp, ctypes.POINTER(bfs_opts),
                                   ctypes.POINTER(bfs_stats)]),
    "tq_bench": (ctypes.c_int, [ctypes.POINTER(tq_bench_cfg), ctypes.POINTER(tq_bench_result)]),
    "tq_strerror": (ctypes.c_char_p, [ctypes.c_int]),
    "tq_persistent_threads": (ctypes.c_int, [ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                             ctypes.POINTER(ctypes.c_int)]),
    "tq_version": (ctypes.c_char_p, []),
    "tq_memory_trim": (ctypes.c_int, [ctypes.c_int]),
    "tq_struct_size": (ctypes.c_size_t, [ctypes.c_char_p]),
    "tq_probe_ceiling": (ctypes.c_int, [ctypes.c_int, c_u64, c_u64, c_vp, ctypes.POINTER(c_dbl)]),
}

STRUCTS = {"tq_csr": tq_csr, "bfs_opts": bfs_opts, "bfs_stats": bfs_stats, "tq_device_view": tq_device_view,
           "tq_counters": tq_counters, "tq_bench_cfg": tq_bench_cfg, "tq_bench_result": tq_bench_result}

_lib = None


class TQError(RuntimeError):
    def __init__(self, status: int, what: str = ""):
        self.status = status
        msg = lib().tq_strerror(status).decode() if _lib is not None else str(status)
        super().__init__(f"{what}: {msg} (tq_status {status})" if what else msg)


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(
                f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
                "(nvcc, sm_100a). There is no CPU fallback.")
        L = ctypes.CDLL(LIB_PATH)
        for name, (res, args) in EXPORTS.items():
            if os.environ.get("TQ_LIB") and not hasattr(L, name):
                continue  # A/B runs of an older build: entry points it predates stay unbound
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def check(status: int, what: str = ""):
    if status != TQ_OK:
        raise TQError(status, what)
