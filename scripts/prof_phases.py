"""Per-phase SM-cycle breakdown of the persistent kernel (A/B builds with
-DTQ_AB_PROF print a TQPROF line to stderr per run).  TQ_LIB selects the build."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import bench
import paper_conf_icpp_troendletj19_b200 as tq

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="kron24x8")
ap.add_argument("--runs", type=int, default=3)
args = ap.parse_args()
kind, a, ef, nr = bench.WORKLOADS[args.workload]
dev = torch.device("cuda", 0)
rp, col = bench.make_graph(kind, a, ef, dev)
roots = bench.pick_roots(kind, rp.cpu().numpy(), nr)
plan = tq.BfsPlan(rp, col)
n = rp.numel() - 1
lv = torch.empty(n, dtype=torch.int32, device=dev)
for i in range(args.runs):
    st = plan.run(roots[i % len(roots)], lv, None, grow_on_full=True)
    print({k: st[k] for k in ("ms_kernel", "tasks", "edges_scanned", "rounds", "busy_cycles", "empty_polls")},
          flush=True)
