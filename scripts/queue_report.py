"""Markdown report of a queue sweep JSONL (scripts/queue_sweep.py)."""
import json
import sys

rows = [json.loads(l) for l in open(sys.argv[1]) if '"ms"' in l]
cap = min(r["capacity"] for r in rows)
full = max(r["warps"] for r in rows)
ceil = {r["batch"]: r for r in rows if r["variant"] == "atomic_ceiling" and r["warps"] == full and r["capacity"] == cap}
r_atom = max(r["atomics_per_s"] for r in ceil.values()) if ceil else float("nan")
out = [f"# Queue micro-benchmark (BASELINE.json configs[1]) — `{sys.argv[1]}`", "",
       f"Full persistent grid = {full} warps ({32 * full} threads); queue capacity {cap} slots "
       f"(2^{cap.bit_length() - 1}) unless noted. ops = enqueues + dequeues (2 per item). Every run's item "
       "multiset was checked against the generator (count / sum / xor of splitmix64).", "",
       f"Same-address atomic ceiling measured in the same run (ATOMIC_CEILING, proxy atomicAdd loop): "
       f"R_atom = {r_atom / 1e9:.2f} G atomics/s per counter.", ""]
variants = ["rf_an", "per_thread_afa", "an", "cas_retry"]
for b in (1, 8, 32):
    out.append(f"## batch b = {b}: throughput (M ops/s) vs persistent threads, E = (X(P)/X(1 warp))/P")
    ws = sorted({r["warps"] for r in rows})
    out.append("| threads | " + " | ".join(variants) + " |")
    out.append("|---|" + "---|" * len(variants))
    base = {v: next((r["mops"] for r in rows if r["variant"] == v and r["batch"] == b and r["warps"] == 1
                     and r["capacity"] == cap), None) for v in variants}
    for w in ws:
        cells = []
        for v in variants:
            r = next((r for r in rows if r["variant"] == v and r["batch"] == b and r["warps"] == w
                      and r["capacity"] == cap), None)
            if r is None:
                cells.append("")
            else:
                e = r["mops"] / base[v] / w if base[v] else float("nan")
                cells.append(f"{r['mops']:.1f} (E {e:.2f})")
        out.append(f"| {32 * w} | " + " | ".join(cells) + " |")
    out.append("")
out.append("## Atomics per item at full occupancy (Fig 5 retry-ratio analogue)")
out.append("| b | " + " | ".join(variants) + " | BASE / RF-AN |")
out.append("|---|" + "---|" * (len(variants) + 1))
for b in sorted({r["batch"] for r in rows}):
    a = {v: next((r["atomics_per_item"] for r in rows if r["variant"] == v and r["batch"] == b
                  and r["warps"] == full and r["capacity"] == cap), float("nan")) for v in variants}
    out.append(f"| {b} | " + " | ".join(f"{a[v]:.3f}" for v in variants) +
               f" | {a['cas_retry'] / a['rf_an']:.0f}x |")
out.append("")
big = [r for r in rows if r["capacity"] != cap and r["variant"] == "rf_an"]
if big:
    out.append(f"## RF/AN at full occupancy with C = {big[0]['capacity']} slots (HBM-resident ring)")
    out.append("| b | M ops/s |")
    out.append("|---|---|")
    for r in sorted(big, key=lambda r: r["batch"]):
        out.append(f"| {r['batch']} | {r['mops']:.1f} |")
print("\n".join(out))
