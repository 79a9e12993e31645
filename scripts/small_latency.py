"""Fixed and per-level latency of one BFS on tiny graphs (config 1 regime):
kernel and device time (median of 30) for a 2-vertex edge, paths of 10 / 100,
a 1,000-leaf star, R-MAT scale 10 and Kronecker scale 14, at several
persistent thread counts and ticket-holding lanes per warp (argv[1], e.g.
"0,1,4,32"; 0 = the plan's automatic choice)."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_icpp_troendletj19_b200 as tq
from inputs import edges_to_csr, kronecker_csr, sample_roots

graphs = {
    "edge2": (edges_to_csr(np.array([0]), np.array([1]), 2, "e2"), 0),
    "path10": (edges_to_csr(np.arange(9), np.arange(1, 10), 10, "p10"), 0),
    "path100": (edges_to_csr(np.arange(99), np.arange(1, 100), 100, "p100"), 0),
    "star1000": (edges_to_csr(np.zeros(1000, dtype=np.int64), np.arange(1, 1001), 1001, "s1k"), 0),
}
g = kronecker_csr(10, 16, 1)
graphs["rmat10"] = (g, int(sample_roots(g.row_ptr, 1, 2)[0]))
g = kronecker_csr(14, 16, 1)
graphs["kron14"] = (g, int(sample_roots(g.row_ptr, 1, 2)[0]))
LANES = [int(x) for x in (sys.argv[1].split(",") if len(sys.argv) > 1 else ["0"])]
for name, (g, root) in graphs.items():
    rp, col = torch.from_numpy(g.row_ptr).cuda(), torch.from_numpy(g.col).cuda()
    lv = torch.empty(g.n_vertices, dtype=torch.int32, device="cuda")
    for th, tl in [(th, tl) for th in (1024, 37888, 0) for tl in LANES]:
        with tq.BfsPlan(rp, col, threads=th, ticket_lanes=tl) as plan:
            for _ in range(3):
                plan.run(root, lv, None)
            sts = [plan.run(root, lv, None) for _ in range(30)]
        print(json.dumps({"graph": name, "threads": sts[0]["persistent_threads"], "ticket_lanes": tl,
                          "levels": sts[0]["max_level"] + 1,
                          "kernel_us": round(statistics.median(s["ms_kernel"] for s in sts) * 1e3, 1),
                          "dev_us": round(statistics.median(s["ms"] for s in sts) * 1e3, 1),
                          "empty_polls": sts[0]["empty_polls"], "tasks": sts[0]["tasks"]}), flush=True)
