"""One warm-up BFS then one BFS to be captured by ncu (-k regex:bfs_persistent -s 1 -c 1)."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import bench
import paper_conf_icpp_troendletj19_b200 as tq

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="kron24x8")
ap.add_argument("--variant", default="rf_an")
ap.add_argument("--runs", type=int, default=2)
args = ap.parse_args()
kind, a, ef, nr = bench.WORKLOADS[args.workload]
dev = torch.device("cuda", 0)
rp, col = bench.make_graph(kind, a, ef, dev)
roots = bench.pick_roots(kind, rp.cpu().numpy(), nr)
n = rp.numel() - 1
plan = tq.BfsPlan(rp, col, variant=args.variant)
lv = torch.empty(n, dtype=torch.int32, device=dev)
pa = torch.empty(n, dtype=torch.int32, device=dev)
for i in range(args.runs):
    st = plan.run(roots[0], lv, pa, grow_on_full=True)
    print({k: st[k] for k in ("ms", "ms_kernel", "traversed_edges", "reached", "tasks", "chunk_tasks",
                              "edges_scanned", "min_atomics", "reenqueues", "queue_atomics",
                              "empty_polls", "max_level", "busy_cycles", "rounds", "skipped_tasks")})
