"""SSSP on the queue (NEXT row 4) at scale: Kronecker graphs with seeded
weights in [1, wmax]; kernel ms, edges relaxed per second, redundancy, and an
element-by-element check of every distance against the Dijkstra oracle for the
first source."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import inputs.gpu as gg
import oracle
import paper_conf_icpp_troendletj19_b200 as tq
from inputs import sample_roots

ap = argparse.ArgumentParser()
ap.add_argument("--scale", type=int, default=24)
ap.add_argument("--wmax", type=int, default=255)
ap.add_argument("--roots", type=int, default=3)
ap.add_argument("--check", type=int, default=1)
args = ap.parse_args()
gg.build()
rp, col = gg.kronecker_csr_cuda(args.scale, 16, 1)
w = gg.edge_weights_cuda(rp, col, 3, args.wmax)
rp_h = rp.cpu().numpy()
roots = [int(r) for r in sample_roots(rp_h, args.roots, 2)]
n = rp.numel() - 1
dist = torch.empty(n, dtype=torch.int32, device="cuda")
parent = torch.empty_like(dist)
with tq.SsspPlan(rp, col, w) as plan:
    plan.run(roots[0], dist, parent, grow_on_full=True)
    for i, r in enumerate(roots):
        st = plan.run(r, dist, parent, grow_on_full=True)
        st["regrows"] = plan.regrows
        rec = {"scale": args.scale, "wmax": args.wmax, "src": r, "ms_kernel": round(st["ms_kernel"], 3),
               "reached": st["reached"], "edges_scanned": st["edges_scanned"],
               "g_edges_per_s": round(st["edges_scanned"] / st["ms_kernel"] / 1e6, 2),
               "undirected_edges_reached": st["traversed_edges"],
               "gteps_equiv": round(st["traversed_edges"] / st["ms_kernel"] / 1e6, 2),
               "tasks": st["tasks"], "reenqueues": st["reenqueues"], "skipped": st["skipped_tasks"],
               "queue_regrows": st["regrows"], "tickets": st["tickets"]}
        if i < args.check:
            d_o, p_o, _ = oracle.sssp(rp_h, col.cpu().numpy(), w.cpu().numpy(), r)
            rec["dist_identical"] = bool(np.array_equal(dist.cpu().numpy().view(np.uint32), d_o))
            rec["parent_identical"] = bool(np.array_equal(parent.cpu().numpy(), p_o))
        print(json.dumps(rec), flush=True)
