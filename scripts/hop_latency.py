"""Per-hop latency of the persistent BFS on a path graph (one vertex per
level: the pure dependent chain publish -> poll -> prolog -> col -> atomicMin
-> enqueue), vs persistent thread count; compare with the grid's us/level."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_icpp_troendletj19_b200 as tq
from inputs import edges_to_csr

n = int(sys.argv[1]) if len(sys.argv) > 1 else 20000
g = edges_to_csr(np.arange(n - 1), np.arange(1, n), n, "path")
rp, col = torch.from_numpy(g.row_ptr).cuda(), torch.from_numpy(g.col).cuda()
lv = torch.empty(n, dtype=torch.int32, device="cuda")
pa = torch.empty(n, dtype=torch.int32, device="cuda")
for threads in (32, 256, 2048, 16384, 0):
    for backoff in (-1, 256):
        with tq.BfsPlan(rp, col, threads=threads, backoff_ns=backoff, timeout_s=60) as plan:
            plan.run(0, lv, pa)
            ms = min(plan.run(0, lv, pa)["ms_kernel"] for _ in range(3))
            st = plan.run(0, lv, pa)
        print(json.dumps({"n": n, "threads": st["persistent_threads"], "backoff": backoff, "ms": round(ms, 3),
                          "us_per_hop": round(ms * 1e3 / (n - 1), 3)}), flush=True)
