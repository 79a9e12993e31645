"""Where the end-to-end (host buffers) time of bench.py's e2e leg goes:
plan creation from a pinned host CSR (H2D + allocations + chunk table),
run_batch with device outputs, run_batch with pinned host outputs, and the
raw H2D / D2H copy bandwidth of this box."""
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
args = ap.parse_args()
kind, a, ef, nr = bench.WORKLOADS[args.workload]
dev = torch.device("cuda", 0)
rp, col = bench.make_graph(kind, a, ef, dev)
roots = bench.pick_roots(kind, rp.cpu().numpy(), nr)[: args.roots]
n = rp.numel() - 1
out = {}


def tick():
    torch.cuda.synchronize(dev)
    return time.perf_counter()


# raw copy bandwidth from / to pinned host memory
col_pin = torch.empty(col.numel(), dtype=torch.int32, pin_memory=True)
rp_pin = torch.empty(n + 1, dtype=torch.int64, pin_memory=True)
t0 = tick()
col_pin.copy_(col)
t1 = tick()
out["d2h_GBps_col"] = round(col.numel() * 4 / (t1 - t0) / 1e9, 1)
rp_pin.copy_(rp)
t0 = tick()
col.copy_(col_pin)
t1 = tick()
out["h2d_GBps_col"] = round(col.numel() * 4 / (t1 - t0) / 1e9, 1)
lv_pin = torch.empty(n, dtype=torch.int32, pin_memory=True)
pa_pin = torch.empty(n, dtype=torch.int32, pin_memory=True)
lv_d = torch.empty(n, dtype=torch.int32, device=dev)
pa_d = torch.empty(n, dtype=torch.int32, device=dev)
for rep in range(2):
    t0 = tick()
    plan = tq.BfsPlan(rp_pin.numpy(), col_pin.numpy())
    t1 = tick()
    out[f"create_host_csr_s_{rep}"] = round(t1 - t0, 3)
    plan.run(roots[0], lv_d, pa_d)
    t0 = tick()
    sts = plan.run_batch(roots, lv_d, pa_d, stride=0)
    t1 = tick()
    out[f"batch_dev_out_ms_per_root_{rep}"] = round((t1 - t0) / len(roots) * 1e3, 2)
    out[f"batch_dev_out_event_ms_per_root_{rep}"] = round(sum(s["ms"] for s in sts) / len(roots), 2)
    t0 = tick()
    sts = plan.run_batch(roots, lv_pin.numpy(), pa_pin.numpy(), stride=0)
    t1 = tick()
    out[f"batch_host_out_ms_per_root_{rep}"] = round((t1 - t0) / len(roots) * 1e3, 2)
    out[f"batch_host_out_event_ms_per_root_{rep}"] = round(sum(s["ms"] for s in sts) / len(roots), 2)
    t0 = time.perf_counter()
    plan.close()
    out[f"destroy_s_{rep}"] = round(time.perf_counter() - t0, 3)
t0 = tick()
plan = tq.BfsPlan(rp, col)
t1 = tick()
out["create_dev_csr_s"] = round(t1 - t0, 3)
plan.close()
print(json.dumps(out), flush=True)
