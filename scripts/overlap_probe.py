"""Does a D2H copy overlap the persistent BFS kernel?  Times one BFS alone, a
537 MB D2H alone, and both issued together (BFS on the plan's stream, the copy
on a side stream), for the plan on the legacy default stream and on a
non-blocking stream."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import bench
import paper_conf_icpp_troendletj19_b200 as tq

kind, a, ef, nr = bench.WORKLOADS[sys.argv[1] if len(sys.argv) > 1 else "kron26x64"]
dev = torch.device("cuda", 0)
rp, col = bench.make_graph(kind, a, ef, dev)
root = int(bench.pick_roots(kind, rp.cpu().numpy(), nr)[0])
n = rp.numel() - 1
lv = torch.empty(n, dtype=torch.int32, device=dev)
pa = torch.empty(n, dtype=torch.int32, device=dev)
src = torch.empty(2 * n, dtype=torch.int32, device=dev)
dst = torch.empty(2 * n, dtype=torch.int32, pin_memory=True)
side = torch.cuda.Stream(dev)
out = {}


def tick():
    torch.cuda.synchronize(dev)
    return time.perf_counter()


for name, stream in (("legacy", None), ("nonblocking", torch.cuda.Stream(dev))):
    plan = tq.BfsPlan(rp, col, stream=stream)
    plan.run(root, lv, pa)
    t0 = tick()
    plan.run(root, lv, pa)
    t1 = tick()
    out[f"{name}_bfs_ms"] = round((t1 - t0) * 1e3, 2)
    with torch.cuda.stream(side):
        dst.copy_(src, non_blocking=True)
    t2 = tick()
    out[f"{name}_copy_ms"] = round((t2 - t1) * 1e3, 2)
    t0 = tick()
    plan.launch(root, lv, pa)
    with torch.cuda.stream(side):
        dst.copy_(src, non_blocking=True)
    plan.wait()
    t1 = tick()
    out[f"{name}_both_ms"] = round((t1 - t0) * 1e3, 2)
    # copy first, then an independent BFS / an independent torch kernel
    main = stream if stream is not None else torch.cuda.current_stream(dev)
    e0, e1, e2, e3 = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
    e0.record(main)
    with torch.cuda.stream(side):
        dst.copy_(src, non_blocking=True)
    e1.record(main)
    plan.launch(root, lv, pa)
    e2.record(main)
    plan.wait()
    torch.cuda.synchronize(dev)
    out[f"{name}_copy_then_bfs_start_end"] = [round(e0.elapsed_time(e1), 2), round(e0.elapsed_time(e2), 2)]
    x = torch.empty(1 << 28, device=dev)
    e0.record(main)
    with torch.cuda.stream(side):
        dst.copy_(src, non_blocking=True)
    e1.record(main)
    with torch.cuda.stream(main):
        x.mul_(2.0)
    e2.record(main)
    torch.cuda.synchronize(dev)
    out[f"{name}_copy_then_torchkernel_start_end"] = [round(e0.elapsed_time(e1), 2), round(e0.elapsed_time(e2), 2)]
    e0.record(main)
    with torch.cuda.stream(side):
        dst.copy_(src, non_blocking=True)
    e1.record(main)
    with torch.cuda.stream(side):
        e3.record(side)
    torch.cuda.synchronize(dev)
    out[f"{name}_copy_then_emptyevent"] = [round(e0.elapsed_time(e1), 2), round(e0.elapsed_time(e3), 2)]
    del x
    # manual two-buffer pipeline: BFS i+1 runs while root i's outputs drain
    bufs = [torch.empty(2, n, dtype=torch.int32, device=dev) for _ in range(2)]
    ev_bfs = [torch.cuda.Event() for _ in range(2)]
    ev_cp = [torch.cuda.Event() for _ in range(2)]
    main = stream if stream is not None else torch.cuda.current_stream(dev)
    hl = torch.empty(2, n, dtype=torch.int32, pin_memory=True)
    K = 8
    t0 = tick()
    for i in range(K):
        b = i & 1
        main.wait_event(ev_cp[b])
        plan.launch(root, bufs[b][0], bufs[b][1])
        ev_bfs[b].record(main)
        side.wait_event(ev_bfs[b])
        with torch.cuda.stream(side):
            hl.copy_(bufs[b], non_blocking=True)
        ev_cp[b].record(side)
        plan.wait()
    t1 = tick()
    out[f"{name}_manual_pipeline_ms_per_root"] = round((t1 - t0) * 1e3 / K, 2)
    # the same pipeline with timestamps: [bfs start, bfs end, copy start, copy end] (ms)
    base = torch.cuda.Event(enable_timing=True)
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(4)] for _ in range(4)]
    base.record(main)
    host = []
    for i in range(4):
        b = i & 1
        main.wait_event(ev_cp[b])
        evs[i][0].record(main)
        hl0 = time.perf_counter()
        plan.launch(root, bufs[b][0], bufs[b][1])
        hl1 = time.perf_counter()
        evs[i][1].record(main)
        ev_bfs[b].record(main)
        side.wait_event(ev_bfs[b])
        evs[i][2].record(side)
        h0 = time.perf_counter()
        with torch.cuda.stream(side):
            hl.copy_(bufs[b], non_blocking=True)
        h1 = time.perf_counter()
        evs[i][3].record(side)
        ev_cp[b].record(side)
        plan.wait()
        h2 = time.perf_counter()
        host.append([round((hl1 - hl0) * 1e3, 2), round((h1 - h0) * 1e3, 2), round((h2 - h1) * 1e3, 2)])
    torch.cuda.synchronize(dev)
    out[f"{name}_host_copy_wait_ms"] = host
    out[f"{name}_timeline"] = [[round(base.elapsed_time(e), 2) for e in row] for row in evs]
    t0 = tick()
    plan.run_batch([root] * K, hl[0].numpy(), hl[1].numpy(), stride=0)
    t1 = tick()
    out[f"{name}_run_batch_host_ms_per_root"] = round((t1 - t0) * 1e3 / K, 2)
    t0 = tick()
    plan.run_batch([root] * K, hl[0].numpy(), None, stride=0)
    t1 = tick()
    out[f"{name}_run_batch_host_level_only_ms_per_root"] = round((t1 - t0) * 1e3 / K, 2)
    plan.close()
print(json.dumps(out), flush=True)
