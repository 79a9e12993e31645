"""Experiment: how much does a degree-descending vertex relabelling (hubs get
the smallest ids, so their mirror bytes / W words share a few L2 lines) change
the persistent BFS time?  Builds the relabelled CSR with torch on the device
(experiment only) and times the same roots on both graphs."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import bench
import paper_conf_icpp_troendletj19_b200 as tq

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="kron24x8")
ap.add_argument("--roots", type=int, default=4)
ap.add_argument("--mode", default="sorted", choices=["sorted", "strided", "compact", "isorted"])
ap.add_argument("--hub-shift", type=int, default=7)
ap.add_argument("--hubs", type=int, default=1 << 17)
ap.add_argument("--cache", type=int, default=1, help="strided: enable the hub level cache")
args = ap.parse_args()
kind, a, ef, nr = bench.WORKLOADS[args.workload]
dev = torch.device("cuda", 0)
rp, col = bench.make_graph(kind, a, ef, dev)
roots = bench.pick_roots(kind, rp.cpu().numpy(), nr)[: args.roots]
n = rp.numel() - 1
deg = rp[1:] - rp[:-1]
if args.mode in ("sorted", "isorted"):
    new2old = torch.sort(deg, descending=True, stable=True).indices
    if args.mode == "isorted":  # top H ranks interleaved over the region's 128-byte lines
        H = min(args.hubs, n) // 128 * 128
        NL = H // 128
        r = torch.arange(H, device=dev)
        pos = (r % NL) * 128 + r // NL
        top = new2old[:H].clone()
        new2old[pos] = top
    old2new = torch.empty_like(new2old)
    old2new[new2old] = torch.arange(n, device=dev)
elif args.mode == "compact":  # top-H degree vertices moved to ids 0..H-1 (swaps), the rest unchanged
    H = args.hubs
    top = torch.sort(deg, descending=True, stable=True).indices[:H]
    is_hub = torch.zeros(n, dtype=torch.bool, device=dev)
    is_hub[top] = True
    is_slot = torch.zeros(n, dtype=torch.bool, device=dev)
    is_slot[:H] = True
    A = torch.nonzero(is_hub & ~is_slot).flatten()
    B = torch.nonzero(is_slot & ~is_hub).flatten()
    new2old = torch.arange(n, device=dev)
    new2old[A] = B
    new2old[B] = A
    old2new = new2old
    print("hubs", H, "moved", A.numel(), "hub edge share %.3f" % (float(deg[top].sum()) / float(deg.sum())))
else:  # top-H degree vertices moved to ids k << shift (swaps), the rest unchanged
    S = 1 << args.hub_shift
    H = min(args.hubs, (n + S - 1) // S)
    top = torch.sort(deg, descending=True, stable=True).indices[:H]
    is_hub = torch.zeros(n, dtype=torch.bool, device=dev)
    is_hub[top] = True
    is_slot = torch.zeros(n, dtype=torch.bool, device=dev)
    is_slot[torch.arange(H, device=dev) * S] = True
    A = torch.nonzero(is_hub & ~is_slot).flatten()
    B = torch.nonzero(is_slot & ~is_hub).flatten()
    new2old = torch.arange(n, device=dev)
    new2old[A] = B
    new2old[B] = A
    old2new = new2old
    print("hubs", H, "moved", A.numel(), "hub edge share %.3f" % (float(deg[top].sum()) / float(deg.sum())))
    if args.cache:
        os.environ["TQ_HUB_SHIFT"] = str(args.hub_shift)
        os.environ["TQ_HUB_N"] = str(H)
deg_new = deg[new2old]
rp_new = torch.zeros(n + 1, dtype=torch.int64, device=dev)
rp_new[1:] = torch.cumsum(deg_new, 0)
col_new = torch.empty_like(col)
step = 1 << 22  # rows per piece (bounded temporaries)
for i0 in range(0, n, step):
    i1 = min(n, i0 + step)
    d = deg_new[i0:i1]
    src_start = rp[new2old[i0:i1]]
    rows = torch.repeat_interleave(torch.arange(i0, i1, device=dev), d)
    off = torch.arange(int(rp_new[i0]), int(rp_new[i1]), device=dev) - rp_new[rows]
    col_new[int(rp_new[i0]):int(rp_new[i1])] = old2new[col[src_start.repeat_interleave(d) + off].long()].int()
    del rows, off, src_start
torch.cuda.synchronize()
del deg, deg_new
lv = torch.empty(n, dtype=torch.int32, device=dev)
lv2 = torch.empty(n, dtype=torch.int32, device=dev)
res = {}
hub_env = {k: os.environ.pop(k) for k in ("TQ_HUB_SHIFT", "TQ_HUB_N") if k in os.environ}
for name, (r_, c_) in {"orig": (rp, col), "relabel": (rp_new, col_new)}.items():
    if name == "relabel":
        os.environ.update(hub_env)
    plan = tq.BfsPlan(r_, c_)
    for k in hub_env:
        os.environ.pop(k, None)
    ms = []
    for rep in range(2):
        for r in roots:
            rr = r if name == "orig" else int(old2new[r])
            st = plan.run(rr, lv if name == "orig" else lv2, None, grow_on_full=True)
            ms.append(st["ms_kernel"])
            if rep == 0 and r == roots[0]:
                print(name, {k: st[k] for k in ("tasks", "edges_scanned", "min_atomics", "persistent_threads")})
            if name == "relabel" and rep == 0:
                plan0 = tq.BfsPlan(rp, col)
                plan0.run(r, lv, None)
                plan0.close()
                assert torch.equal(lv, lv2[old2new]), "levels differ"
    plan.close()
    res[name] = ms
    print(name, "ms_kernel mean %.3f min %.3f" % (sum(ms) / len(ms), min(ms)), flush=True)
