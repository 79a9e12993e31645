"""Queue micro-benchmark sweep (BASELINE.json configs[1]; Fig 4 / Fig 5 analogue).

Persistent warps 1 .. full B200, batch b in {1..32}, variants RF/AN,
per-thread AFA, CAS-retry (BASE), AN, plus the same-address atomic ceiling.
Every run's item multiset is checked against the generator (count/sum/xor).
Writes one JSON line per run to --out and prints a summary table.

    python scripts/queue_sweep.py --out results/queue_sweep_r01.jsonl
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import paper_conf_icpp_troendletj19_b200 as tq
from inputs import fingerprint, item_of

ap = argparse.ArgumentParser()
ap.add_argument("--out", default="gpurun_out/queue_sweep.jsonl")
ap.add_argument("--variants", default="rf_an,rf_an_cta,per_thread_afa,cas_retry,an,atomic_ceiling")
ap.add_argument("--batches", default="1,2,4,8,16,32")
ap.add_argument("--capacity", type=int, default=1 << 20)
ap.add_argument("--big-capacity", type=int, default=1 << 26)
ap.add_argument("--per-warp-items", type=int, default=1 << 13)
ap.add_argument("--max-items", type=int, default=1 << 24)
ap.add_argument("--target-s", type=float, default=0.25)
args = ap.parse_args()

full = tq.queue_bench("rf_an", warps=0, batch=32, items=1 << 22)["warps"]
warps_list = sorted({1 << i for i in range(0, 16) if (1 << i) < full} | {448, full})  # 448 = paper's 14,336 thr
os.makedirs(os.path.dirname(args.out) or ".", exist_ok=True)
fp_cache = {}
rows = []
with open(args.out, "w") as f:
    for variant in args.variants.split(","):
        for b in map(int, args.batches.split(",")):
            rate = None  # items/s at the previous point: sizes the next run to ~target seconds
            for w in warps_list:
                for cap in ([args.capacity] + ([args.big_capacity] if w == full else [])):
                    items = min(args.max_items, max(w * b * 64, w * args.per_warp_items))
                    if rate is not None:
                        items = int(min(items, max(w * b * 16, rate * args.target_s)))
                    try:
                        r = tq.queue_bench(variant, warps=w, batch=b, items=items, capacity=cap, seed=3,
                                           timeout_s=60)
                    except tq.TQError as e:
                        rec = {"variant": variant, "batch": b, "warps": w, "capacity": cap, "error": str(e)}
                        f.write(json.dumps(rec) + "\n")
                        continue
                    n = r["items"]
                    ok = None
                    if variant != "atomic_ceiling":
                        if n not in fp_cache:
                            fp_cache[n] = fingerprint(item_of(3, np.arange(n)))
                        ok = (r["deq"], r["sum_deq"], r["xor_deq"]) == fp_cache[n] and \
                             (r["enq"], r["sum_enq"], r["xor_enq"]) == fp_cache[n]
                    s = r["ms"] * 1e-3
                    rec = {"variant": variant, "batch": b, "warps": w, "threads": 32 * w, "capacity": cap,
                           "items": n, "ms": r["ms"], "items_per_s": n / s,
                           "mops": (2 * n / s / 1e6) if variant != "atomic_ceiling" else None,
                           "atomics_per_s": r["atomics"] / s, "atomics_per_item": r["atomics"] / n,
                           "cas_failures": r["cas_failures"], "empty_retries": r["empty_retries"],
                           "conserved": ok}
                    f.write(json.dumps(rec) + "\n")
                    f.flush()
                    rows.append(rec)
                    rate = n / s

# summary: throughput at full warps, scaling efficiency vs 1 warp
print(f"full persistent warps = {full} ({32 * full} threads)")
print(f"{'variant':16s} {'b':>3s} {'Mops@1w':>10s} {'Mops@full':>10s} {'atom/item':>9s} {'E(full)':>8s} {'E(448w)':>8s} cons")
for variant in args.variants.split(","):
    for b in map(int, args.batches.split(",")):
        sel = {r["warps"]: r for r in rows if r["variant"] == variant and r["batch"] == b
               and r["capacity"] == args.capacity}
        if 1 not in sel or full not in sel:
            continue
        key = "mops" if variant != "atomic_ceiling" else "atomics_per_s"
        x1, xf = sel[1][key], sel[full][key]
        e_full = (xf / x1) / full
        e448 = (sel[448][key] / x1) / 448 if 448 in sel else float("nan")
        cons = all(r["conserved"] in (True, None) for r in sel.values())
        scale = 1.0 if key == "mops" else 1e-6
        print(f"{variant:16s} {b:3d} {x1 * scale:10.1f} {xf * scale:10.1f} {sel[full]['atomics_per_item']:9.3f} "
              f"{e_full:8.3f} {e448:8.3f} {cons}")
