"""One tq_bench launch per configuration, for ncu (-k regex:bench): the queue
micro-benchmark at full occupancy -- RF/AN warp proxy at b = 1 (bound by the
same-address atomic rate on Front / Rear) and b = 32, the pipelined CTA proxy at
b = 32, and the per-thread-AFA comparator."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_troendletj19_b200 as tq

for v, b, d in (("rf_an", 1, 1), ("rf_an", 32, 1), ("rf_an_cta", 32, 2), ("per_thread_afa", 32, 1)):
    r = tq.queue_bench(v, warps=0, batch=b, items=1 << 24, capacity=1 << 22, seed=3, depth=d, timeout_s=60)
    print(v, b, d, r["warps"], round(2 * r["items"] / (r["ms"] * 1e-3) / 1e6, 1), "Mops/s", flush=True)
