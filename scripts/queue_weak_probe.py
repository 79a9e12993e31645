import json, sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_troendletj19_b200 as tq
full = tq.queue_bench("rf_an", warps=0, batch=32, items=1 << 22)["warps"]
for v in ("rf_an", "rf_an_cta"):
    for b in (1, 8, 32):
        base = None
        for w in (1, 8, 64, 512, 2048, 4096, full):
            for it in (1024, 8192):
                items = w * b * it
                if items >= 1 << 32: continue
                r = tq.queue_bench(v, warps=w, batch=b, items=items, seed=3, timeout_s=60)
                mops = 2 * r["items"] / (r["ms"] * 1e-3) / 1e6
                if w == 1 and it == 8192: base = mops
                E = mops / (base * w) if base else None
                print(json.dumps({"v": v, "b": b, "warps": w, "iters": it, "ms": round(r["ms"], 3), "mops": round(mops, 1), "E": E and round(E, 3)}), flush=True)
