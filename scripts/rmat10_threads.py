"""Config 1 (R-MAT scale 10) latency by persistent thread count: device time of
init + kernel + unpack (median of 50) and the host wall time of bfs_plan_run."""
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import bench
import paper_conf_icpp_troendletj19_b200 as tq

rp, col = bench.make_graph("kron", 10, 16, torch.device("cuda", 0))
roots = bench.pick_roots("kron", rp.cpu().numpy(), 16)
lv = torch.empty(rp.numel() - 1, dtype=torch.int32, device="cuda")
pa = torch.empty_like(lv)
for th in (256, 1024, 4096, 16384, 37888, 0):
    for bo in (0, -1):
        with tq.BfsPlan(rp, col, threads=th, backoff_ns=bo) as plan:
            for r in roots[:4]:
                plan.run(r, lv, pa)
            dev, wall = [], []
            for i in range(50):
                t = time.perf_counter()
                st = plan.run(roots[i % 16], lv, pa)
                wall.append((time.perf_counter() - t) * 1e6)
                dev.append(st["ms"] * 1e3)
        print(json.dumps({"threads": st["persistent_threads"], "backoff_ns": bo,
                          "dev_us_median": round(statistics.median(dev), 1),
                          "kernel_us_median": round(st["ms_kernel"] * 1e3, 1),
                          "wall_us_median": round(statistics.median(wall), 1)}), flush=True)
