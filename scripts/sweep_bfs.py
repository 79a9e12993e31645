"""Option sweep of the BFS on one workload: prints ms and redundancy stats."""
import argparse
import itertools
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import bench
import paper_conf_icpp_troendletj19_b200 as tq

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="kron24x8")
ap.add_argument("--chunks", default="256")
ap.add_argument("--threads", default="0")
ap.add_argument("--backoff", default="0")
ap.add_argument("--variants", default="rf_an")
ap.add_argument("--roots", type=int, default=2)
ap.add_argument("--parents", default="any")
ap.add_argument("--hubq", default="1")
args = ap.parse_args()
kind, a, ef, nr = bench.WORKLOADS[args.workload]
dev = torch.device("cuda", 0)
rp, col = bench.make_graph(kind, a, ef, dev)
roots = bench.pick_roots(kind, rp.cpu().numpy(), nr)[: args.roots]
n = rp.numel() - 1
lv = torch.empty(n, dtype=torch.int32, device=dev)
pa = torch.empty(n, dtype=torch.int32, device=dev)
for var, ch, th, bo in itertools.product(args.variants.split(","), map(int, args.chunks.split(",")),
                                         map(int, args.threads.split(",")), map(int, args.backoff.split(","))):
    plan = tq.BfsPlan(rp, col, variant=var, chunk=ch, threads=th, backoff_ns=bo, timeout_s=60,
                      parents=args.parents, hub_queue=args.hubq == "1")
    plan.run(roots[0], lv, pa)
    for r in roots:
        st = plan.run(r, lv, pa)
        ideal = 2 * st["traversed_edges"]
        print(json.dumps({"var": var, "chunk": ch, "threads": st["persistent_threads"], "backoff": bo, "root": r,
                          "ms": round(st["ms_kernel"], 3), "gteps": round(st["traversed_edges"] / st["ms"] / 1e6, 2),
                          "scan_x": round(st["edges_scanned"] / max(ideal, 1), 3),
                          "reenq_frac": round(st["reenqueues"] / max(st["reached"], 1), 3),
                          "tasks": st["tasks"], "chunk_tasks": st["chunk_tasks"], "min_atomics": st["min_atomics"],
                          "qatom": st["queue_atomics"], "empty": st["empty_polls"], "maxlev": st["max_level"],
                          "tok_per_cycle": round(st["tasks"] / max(st["busy_cycles"], 1), 2),
                          "rounds_per_cycle": round(st["rounds"] / max(st["busy_cycles"], 1), 2),
                          "round_fill": round(st["edges_scanned"] / max(128 * st["rounds"], 1), 3),
                          "skipped": st["skipped_tasks"]}), flush=True)
    plan.close()
