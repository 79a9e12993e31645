"""Interleaved A/B of BFS plan options on one graph (same process, same
graph, alternating plans): mean persistent-kernel ms per option set.

  python scripts/ab_opts.py --workload kron24x8 --roots 6 --reps 3 \
      --opts "{}" "{\"hub_queue\": false}"
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import bench
import paper_conf_icpp_troendletj19_b200 as tq

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="kron24x8")
ap.add_argument("--roots", type=int, default=6)
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--opts", nargs="+", default=["{}"])
ap.add_argument("--check", action="store_true", help="levels of every run vs the first option's")
args = ap.parse_args()
kind, a, ef, nr = bench.WORKLOADS[args.workload]
dev = torch.device("cuda", 0)
rp, col = bench.make_graph(kind, a, ef, dev)
roots = bench.pick_roots(kind, rp.cpu().numpy(), max(nr, args.roots))[: args.roots]
n = rp.numel() - 1
lv = torch.empty(n, dtype=torch.int32, device=dev)
pa = torch.empty(n, dtype=torch.int32, device=dev)
optsets = [json.loads(o) for o in args.opts]
plans = [tq.BfsPlan(rp, col, timeout_s=60, **o) for o in optsets]
for p in plans:  # warm-up
    p.run(roots[0], lv, pa)
ref = {}
res = {i: [] for i in range(len(plans))}
for rep in range(args.reps):
    for r in roots:
        for i, p in enumerate(plans):
            st = p.run(r, lv, pa)
            if args.check:
                if i == 0:
                    ref[r] = lv.clone()
                else:
                    assert torch.equal(ref[r], lv), (r, optsets[i])
            res[i].append(st)
for i, sts in res.items():
    ms = [s["ms_kernel"] for s in sts]
    te = sum(s["traversed_edges"] for s in sts)
    scanned = sum(s["edges_scanned"] for s in sts)
    print(json.dumps({"workload": args.workload, "opts": optsets[i], "n": len(ms),
                      "ms_mean": round(statistics.mean(ms), 4), "ms_min": round(min(ms), 4),
                      "gteps_kernel": round(te / (sum(ms) * 1e-3) / 1e9, 2),
                      "scan_x": round(scanned / max(2 * te, 1), 3),
                      "min_atomics_per_edge": round(sum(s["min_atomics"] for s in sts) / max(scanned, 1), 4),
                      "threads": sts[0]["persistent_threads"]}), flush=True)
