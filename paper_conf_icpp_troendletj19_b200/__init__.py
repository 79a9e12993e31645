"""B200-native retry-free, arbitrary-n task queue and persistent-thread BFS.

Troendle, Ta & Jang, "A Specialized Concurrent Queue for Scheduling Irregular
Workloads on GPUs", ICPP 2019. The product is `libtq.so` (CUDA for sm_100a
behind the C ABI in include/tq.h); this package is its thin Python binding.
"""
from .api import (BfsPlan, Queue, SsspPlan, TQError, VARIANTS, bfs, memory_trim, persistent_threads,
                  probe_ceiling, queue_bench, run_concurrent, sssp, version)

__all__ = ["BfsPlan", "Queue", "SsspPlan", "TQError", "VARIANTS", "bfs", "memory_trim", "persistent_threads",
           "probe_ceiling", "queue_bench", "run_concurrent", "sssp", "version"]
