"""Table 3 / Fig 5 analogue on the B200 configs (§5.3, P:367-382,
P:417-427): BFS kernel time and queue atomics per task of the four queue
variants -- BASE (CAS-retry), AN, RF/AN, per-thread AFA -- at the paper's
14,336 persistent threads and at the full GPU, the CAS queues naive and with a
bounded randomised back-off.  Every run's levels are checked (closed form for
the tree and the grid, the oracle for Kronecker).  One JSON line per run.

  python scripts/variant_table.py --graphs tree,kron24,grid --out results/variant_table_r02.jsonl
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import bench
import inputs.gpu as gg
import oracle
import paper_conf_icpp_troendletj19_b200 as tq

ap = argparse.ArgumentParser()
ap.add_argument("--graphs", default="tree,kron24,grid")
ap.add_argument("--threads", default="14336,0")
ap.add_argument("--timeout", type=float, default=20.0)
ap.add_argument("--backoff", type=int, default=2048)
ap.add_argument("--out", default=None)
args = ap.parse_args()
gg.build()
out = open(args.out, "a") if args.out else None


def graph(name):
    if name == "tree":
        n = 10485760
        rp, col = gg.tree4_csr_cuda(n)
        i = torch.arange(n, device="cuda", dtype=torch.int64)
        x, exp, k, p4 = 3 * i + 1, torch.zeros(n, dtype=torch.int64, device="cuda"), 0, 1
        while p4 * 4 <= int(x.max()):
            k, p4 = k + 1, p4 * 4
            exp[x >= p4] = k
        return rp, col, 0, exp.int()
    if name == "grid":
        rows = 4096
        rp, col = gg.grid_csr_cuda(rows)
        v = torch.arange(rows * rows, device="cuda", dtype=torch.int64)
        return rp, col, 0, (v // rows + v % rows).int()
    scale = int(name[4:])
    rp, col = gg.kronecker_csr_cuda(scale, 16, bench.GRAPH_SEED)
    root = bench.pick_roots("kron", rp.cpu().numpy(), 1)[0]
    lv, _, _ = oracle.bfs(rp.cpu().numpy(), col.cpu().numpy(), root, parents=False)
    return rp, col, root, torch.from_numpy(lv).cuda()


for name in args.graphs.split(","):
    rp, col, root, exp = graph(name)
    lv = torch.empty(rp.numel() - 1, dtype=torch.int32, device="cuda")
    for th in map(int, args.threads.split(",")):
        for v, bo in (("rf_an", 0), ("per_thread_afa", 0), ("an", 0), ("an", args.backoff), ("cas_retry", 0),
                      ("cas_retry", args.backoff)):
            rec = {"graph": name, "variant": v, "cas_backoff_ns": bo, "threads_req": th}
            try:
                with tq.BfsPlan(rp, col, variant=v, threads=th, timeout_s=args.timeout, cas_backoff_ns=bo) as plan:
                    plan.run(root, lv, None)  # warm-up (and the deep-graph grid decision)
                    st = plan.run(root, lv, None)
                rec.update({"threads": st["persistent_threads"], "ms_kernel": round(st["ms_kernel"], 3),
                            "levels_ok": bool(torch.equal(lv, exp)), "tasks": st["tasks"],
                            "queue_atomics": st["queue_atomics"], "cas_failures": st["cas_failures"],
                            "atomics_per_task": round(st["queue_atomics"] / max(st["tasks"], 1), 4),
                            "gteps": round(st["traversed_edges"] / (st["ms_kernel"] * 1e-3) / 1e9, 3)})
            except tq.TQError as e:
                rec["error"] = str(e)
            print(json.dumps(rec), flush=True)
            if out:
                out.write(json.dumps(rec) + "\n")
                out.flush()
    del rp, col
    torch.cuda.empty_cache()
