"""Multi-root throughput with K concurrent BFS plans on K streams (each with
1/K of the persistent grid): fills the low-parallelism first and last levels
of each BFS with another root's work."""
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
ap.add_argument("--workload", default="kron26x64")
ap.add_argument("--roots", type=int, default=16)
ap.add_argument("--ks", default="1,2,3,4")
ap.add_argument("--occ-scale", default="1.0")
args = ap.parse_args()
kind, a, ef, nr = bench.WORKLOADS[args.workload]
dev = torch.device("cuda", 0)
rp, col = bench.make_graph(kind, a, ef, dev)
roots = bench.pick_roots(kind, rp.cpu().numpy(), nr)[: args.roots]
full = tq.persistent_threads()
for k in map(int, args.ks.split(",")):
    for sc in map(float, args.occ_scale.split(",")):
        streams = [torch.cuda.Stream() for _ in range(k)]
        plans = [tq.BfsPlan(rp, col, stream=s, threads=int(full * sc / k) // 256 * 256) for s in streams]
        tq.run_concurrent(plans, roots[:k])  # warm-up
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        st = tq.run_concurrent(plans, roots)
        torch.cuda.synchronize()
        sec = time.perf_counter() - t0
        te = sum(s["traversed_edges"] for s in st)
        print(json.dumps({"k": k, "occ_scale": sc, "threads_per_plan": st[0]["persistent_threads"],
                          "roots": len(roots), "s": round(sec, 4), "gteps": round(te / sec / 1e9, 2)}), flush=True)
        for p in plans:
            p.close()
        del plans
        torch.cuda.empty_cache()
