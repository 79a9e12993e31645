"""Weak-scaling sweep of the queue micro-benchmark's proxy groups (fixed
iterations per warp): warp / CTA proxies in the paper's order (depth 1) and
pipelined one iteration ahead (depth 2), and thread-block-cluster proxies
(always pipelined).  E = X(P) / (P_warps * X1), X1 = the same variant's
single-group rate per warp ("E_self") and the single-warp RF/AN rate
("E_warp1", linear from one warp).  One JSON line per run."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_troendletj19_b200 as tq

ap = argparse.ArgumentParser()
ap.add_argument("--iters", type=int, default=4096)
ap.add_argument("--batches", default="1,8,32")
ap.add_argument("--configs", default="rf_an:1:0,rf_an_cta:1:0,rf_an_cta:2:0,"
                                      "rf_an_cluster:2:2,rf_an_cluster:2:4,rf_an_cluster:2:8,rf_an_cluster:2:16")
ap.add_argument("--out", default=None)
args = ap.parse_args()
out = open(args.out, "a") if args.out else None


def run(v, d, c, w, b):
    items = w * b * args.iters
    r = tq.queue_bench(v, warps=w, batch=b, items=items, seed=3, timeout_s=60, depth=d, cluster=c,
                       capacity=1 << 22)
    return r, 2 * r["items"] / (r["ms"] * 1e-3) / 1e6


for b in [int(x) for x in args.batches.split(",")]:
    _, x1 = run("rf_an", 1, 0, 1, b)
    for cfg in args.configs.split(","):
        v, d, c = cfg.split(":")
        d, c = int(d), int(c)
        try:
            full = tq.queue_bench(v, warps=0, batch=b, items=1 << 24, depth=d, cluster=c, capacity=1 << 22)["warps"]
        except tq.TQError as e:
            print(json.dumps({"v": v, "depth": d, "cluster": c, "b": b, "error": str(e)}), flush=True)
            continue
        g = {"rf_an": 1, "rf_an_cta": 8, "rf_an_cluster": 8 * max(c, 1)}[v]
        # a CTA group may be a single warp (1-warp blocks): its own linear baseline
        ws = sorted({w for w in (1, 8, 64, 128, 512, 1024, 2048, 4096)
                     if (w % g == 0 or (v == "rf_an_cta" and w == 1)) and w <= full} | {full})
        base = None
        for w in ws:
            try:
                r, mops = run(v, d, c, w, b)
            except tq.TQError as e:
                print(json.dumps({"v": v, "depth": d, "cluster": c, "b": b, "warps": w, "error": str(e)}), flush=True)
                continue
            if base is None:
                base = mops / w
            rec = {"v": v, "depth": d, "cluster": c, "b": b, "warps": w, "threads": 32 * w,
                   "ms": round(r["ms"], 3), "mops": round(mops, 1), "E_self": round(mops / (base * w), 3),
                   "E_warp1": round(mops / (x1 * w), 3), "atomics_per_item": round(r["atomics"] / r["items"], 4)}
            print(json.dumps(rec), flush=True)
            if out:
                out.write(json.dumps(rec) + "\n")
                out.flush()
