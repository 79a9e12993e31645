"""The paper's synthetic dataset on B200 (NEXT row 2; Table 3
synthetic row P:369/Fig 4a/b P:363-365).

Reading R13: heap-ordered 4-ary tree, 10,485,760 vertices,
children of i are 4i+1..4i+4. BFS from vertex 0 with each queue variant
(BASE = CAS-retry, AN, RF/AN, plus per-thread AFA) over persistent thread
counts from one warp to the full GPU; levels are checked against the closed
form level(i) = floor(log4(3i+1)) on every run. Prints one JSON line per run
and a summary (kernel ms, speedup vs the smallest thread count).
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import inputs.gpu as gg
import paper_conf_icpp_troendletj19_b200 as tq

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=10485760)
ap.add_argument("--variants", default="rf_an,per_thread_afa,an,cas_retry")
ap.add_argument("--threads", default="256,1024,4096,14336,16384,65536,0")
ap.add_argument("--timeout", type=float, default=30.0)
ap.add_argument("--out", default="gpurun_out/paper_synthetic.jsonl")
args = ap.parse_args()

gg.build()
rp, col = gg.tree4_csr_cuda(args.n)
n = args.n
i = torch.arange(n, device="cuda", dtype=torch.int64)
x = 3 * i + 1
exp = torch.zeros(n, dtype=torch.int64, device="cuda")
k, p4 = 0, 1
while p4 * 4 <= int(x.max()):
    k += 1
    p4 *= 4
    exp[x >= p4] = k
level = torch.empty(n, dtype=torch.int32, device="cuda")
parent = torch.empty_like(level)
rows = []
with open(args.out, "w") as f:
    for v in args.variants.split(","):
        for th in map(int, args.threads.split(",")):
            try:
                with tq.BfsPlan(rp, col, variant=v, threads=th, timeout_s=args.timeout) as plan:
                    plan.run(0, level, parent)  # warm-up
                    st = plan.run(0, level, parent)
                ok = bool(torch.equal(level.long(), exp))
                rec = {"variant": v, "threads": st["persistent_threads"], "ms_kernel": st["ms_kernel"],
                       "ms": st["ms"], "levels_ok": ok, "queue_atomics": st["queue_atomics"],
                       "cas_failures": st["cas_failures"], "tasks": st["tasks"], "reached": st["reached"]}
            except tq.TQError as e:
                rec = {"variant": v, "threads": th, "error": str(e)}
            f.write(json.dumps(rec) + "\n")
            f.flush()
            print(json.dumps(rec), flush=True)
            rows.append(rec)

print("--- kernel ms (speedup vs the smallest thread count) ---")
for v in args.variants.split(","):
    sel = [r for r in rows if r["variant"] == v and "ms_kernel" in r]
    if not sel:
        continue
    t0 = sel[0]["ms_kernel"]
    print(v, " ".join(f"{r['threads']}:{r['ms_kernel']:.2f}({t0 / r['ms_kernel']:.1f}x)" for r in sel))
