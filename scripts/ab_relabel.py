"""A/B of bfs_opts.relabel on the bench graphs: per-root persistent-kernel ms
and whole-run ms (init + kernel + unpack), plan build seconds, interleaved
over reps (results/relabel_r02.log)."""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import bench
import paper_conf_icpp_troendletj19_b200 as tq

ap = argparse.ArgumentParser()
ap.add_argument("--workloads", default="kron24x8,kron26x64,grid4096")
ap.add_argument("--roots", type=int, default=6)
ap.add_argument("--reps", type=int, default=3)
args = ap.parse_args()
dev = torch.device("cuda", 0)
for wl in args.workloads.split(","):
    kind, a, ef, nr = bench.WORKLOADS[wl]
    rp, col = bench.make_graph(kind, a, ef, dev)
    roots = bench.pick_roots(kind, rp.cpu().numpy(), nr)[: (1 if kind == "grid" else args.roots)]
    n = rp.numel() - 1
    lv = torch.empty(n, dtype=torch.int32, device=dev)
    pa = torch.empty_like(lv)
    plans = {}
    for rl in (-1, 1):
        torch.cuda.synchronize()
        t = time.perf_counter()
        plans[rl] = tq.BfsPlan(rp, col, relabel=rl)
        torch.cuda.synchronize()
        build_s = time.perf_counter() - t
        plans[rl].run(roots[0], lv, pa, grow_on_full=True)
        plans[rl].build_s = build_s
    res = {rl: {"k": [], "t": []} for rl in plans}
    for rep in range(args.reps):
        for rl, plan in plans.items():
            for r in roots:
                st = plan.run(r, lv, pa, grow_on_full=True)
                res[rl]["k"].append(st["ms_kernel"])
                res[rl]["t"].append(st["ms"])
    for rl, plan in plans.items():
        k, t = res[rl]["k"], res[rl]["t"]
        print(json.dumps({"workload": wl, "relabel": rl, "relabelled": st["relabelled"] if rl > 0 else 0,
                          "kernel_ms_mean": round(sum(k) / len(k), 3), "kernel_ms_min": round(min(k), 3),
                          "run_ms_mean": round(sum(t) / len(t), 3), "plan_build_s": round(plan.build_s, 3)}),
              flush=True)
        plan.close()
