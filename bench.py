#!/usr/bin/env python
"""Benchmark: batched multi-root persistent-thread BFS on the retry-free,
arbitrary-n queue (BASELINE.json configs[4]: Kronecker scale 26, edgefactor
16, 64 roots split across the ranks, graph replicated, NCCL stats gather).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl tq|reference]
                    [--workload kron26x64|kron24x64|kron24x8|grid4096|rmat10]

A step is one pass of the whole hot path over one batch: for every root of
this rank's share, queue/state init (a2) + persistent BFS (a3-a8) + unpack
and stats (a9). The metric is GTEPS = sum over roots of traversed edges
(undirected, deduplicated, loop-free edges with a reached endpoint; DESIGN.md
R16) / the step time (max over ranks). Rank 0 prints ONE JSON line.

--impl reference runs the oracle (oracle/, the plain sequential C BFS) on the
host cores, on a bounded sample of the same workload (rank 0 only).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

WORKLOADS = {
    # name: (kind, scale/rows, edgefactor, n_roots)
    "kron26x64": ("kron", 26, 16, 64),
    "kron24x64": ("kron", 24, 16, 64),
    "kron24x8": ("kron", 24, 16, 8),
    "grid4096": ("grid", 4096, 0, 1),
    "rmat10": ("kron", 10, 16, 16),
    "kron20x16": ("kron", 20, 16, 16),  # tests: a quick multi-root batch
}
GRAPH_SEED, ROOT_SEED = 1, 2


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi-equivalent clock / throttle sampling (NVML) during the timed region."""

    REASONS = {
        0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
        0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
        0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
    }

    def __init__(self, index: int):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit and name != "gpu_idle":
                        self.reasons.add(name)
            except Exception:
                pass
            self._stop.wait(0.1)

    def __enter__(self):
        if self.nv:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.nv:
            self.t.join()

    def summary(self):
        s = sorted(self.samples)
        return {"sm_mhz": s[len(s) // 2] if s else None, "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(s)}


def free_port():
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def make_graph(kind, a, ef, device):
    import inputs.gpu as gg
    gg.build()
    if kind == "kron":
        return gg.kronecker_csr_cuda(a, ef, GRAPH_SEED, device=device)
    return gg.grid_csr_cuda(a, a, device=device)


def pick_roots(kind, row_ptr_host, n_roots):
    from inputs import sample_roots
    if kind == "grid":
        return [0]  # corner: 8,191 levels (R17)
    return [int(r) for r in sample_roots(row_ptr_host, n_roots, ROOT_SEED)]


def algorithmic_bytes(traversed_edges, reached):
    """SURVEY §8(d) per-unit figures for the persistent kernel (DESIGN.md
    "Algorithmic bytes"): 12 B per directed CSR entry of a reached vertex
    (4 B col + 8 B W prefilter) and 56 B per reached vertex (16 B row_ptr,
    24 B queue slot write/poll/reset, 8 B W install, 8 B fresh level read)."""
    return 12 * 2 * traversed_edges + 56 * reached


def cpu_oracle_sample(row_ptr, col, roots, budget_s=20.0, check=None):
    """Time the oracle (as it stands, 1 core) on roots of the same graph until
    the budget is spent; returns (teps, sample description, levels of root 0)."""
    import oracle
    te_sum, sec_sum, done, lv0 = 0, 0.0, [], None
    for r in roots:
        lv, _, info = oracle.bfs(row_ptr, col, r, parents=False)
        te_sum += info["traversed_edges"]
        sec_sum += info["seconds_levels"]
        done.append(r)
        if lv0 is None:
            lv0 = lv
        if sec_sum >= budget_s:
            break
    return te_sum / sec_sum, done, sec_sum, lv0


def _median(xs):
    xs = sorted(xs)
    return xs[len(xs) // 2] if xs else None


def _mirror_bytes(n):
    return n if n <= (1 << 25) else (n + 7) // 8 * 4  # byte / nibble mirror (R8)


def _roofline(stats_list, hbm_peak, peak_src, probe_g=None):
    """HBM roofline (SURVEY §8(d) algorithmic bytes / CUDA-event kernel time,
    per launch) and the L2 random-probe roofline of the persistent kernel."""
    runs = len(stats_list)
    te = sum(s["traversed_edges"] for s in stats_list)
    reached = sum(s["reached"] for s in stats_list)
    kern_s = sum(s["ms_kernel"] for s in stats_list) * 1e-3 / runs
    alg = algorithmic_bytes(te, reached) / runs
    out = {"bound": "hbm", "achieved": round(alg / kern_s / 1e9, 1), "peak": hbm_peak, "unit": "GB/s",
           "frac": round(alg / kern_s / 1e9 / hbm_peak, 4), "peak_source": peak_src,
           "alg_bytes_per_launch": int(alg), "avg_launch_ms": round(kern_s * 1e3, 4)}
    if probe_g:
        scanned = sum(s["edges_scanned"] for s in stats_list) / runs
        out["l2_probe"] = {"achieved": round(scanned / kern_s / 1e9, 1), "peak": round(probe_g, 1),
                           "unit": "G CSR entries/s vs G random L2 probes/s",
                           "frac": round(scanned / kern_s / 1e9 / probe_g, 4)}
    return out


def _cpu_info():
    return {"nproc": os.cpu_count(), "cpu_model": cpu_model()}


def config_rmat10(tq, dev, local, args):
    """BASELINE.json configs[0]: R-MAT scale 10, single-root BFS, GPU us beside
    the CPU oracle's ms (median of 20 each), every sampled root checked."""
    import numpy as np
    import torch
    import oracle
    rp, col = make_graph("kron", 10, 16, dev)
    rp_h, col_h = rp.cpu().numpy(), col.cpu().numpy()
    roots = pick_roots("kron", rp_h, 16)
    n = rp.numel() - 1
    lv = torch.empty(n, dtype=torch.int32, device=dev)
    pa = torch.empty_like(lv)
    out = {"workload": "rmat10", "graph": "kron 10 ef16", "n_vertices": n, "nnz": int(col.numel()),
           "roots": len(roots)}
    with ClockSampler(local) as clk:
        ok_lv, ok_pa, ok_min = True, True, True
        with tq.BfsPlan(rp, col, variant=args.variant, device=local) as plan, \
                tq.BfsPlan(rp, col, variant=args.variant, device=local, parents="min_id") as pmin:
            for r in roots[:3]:
                plan.run(r, lv, pa)
            us, te = [], 0
            for i in range(20):
                st = plan.run(roots[i % len(roots)], lv, pa)
                us.append(st["ms"] * 1e3)
                te += st["traversed_edges"]
            smem = bool(st["smem_path"])
            for r in roots:  # parity of every sampled root (default and min-id rules)
                plan.run(r, lv, pa)
                lo, po, _ = oracle.bfs(rp_h, col_h, r)
                lvh, pah = lv.cpu().numpy(), pa.cpu().numpy()
                ok_lv &= bool(np.array_equal(lvh, lo))
                ok_pa &= oracle.validate_tree(rp_h, col_h, r, lvh, pah)[0] == 0
                pmin.run(r, lv, pa)
                ok_min &= bool(np.array_equal(lv.cpu().numpy(), lo) and np.array_equal(pa.cpu().numpy(), po))
        ms_o, te_o = [], 0
        for i in range(20):
            _, _, info = oracle.bfs(rp_h, col_h, roots[i % len(roots)], parents=False)
            ms_o.append(info["seconds_levels"] * 1e3)
            te_o += info["traversed_edges"]
    out.update({
        "gpu_us_median": round(_median(us), 2), "gpu_us_min": round(min(us), 2), "gpu_runs": 20,
        "gpu_path": "shared-memory queue, one 1024-thread block" if smem else "persistent grid",
        "gpu_timed": ("CUDA events around the one launch (graph load, BFS over the shared-memory queue, unpack; "
                      "bfs_stats.ms)" if smem else
                      "CUDA events around init + persistent kernel + unpack (bfs_stats.ms), graph L2-resident"),
        "gpu_gteps": round(te / (sum(us) * 1e-6) / 1e9, 4),
        "cpu_baseline": dict({"kind": "oracle", "cores": 1, "ms_median": round(_median(ms_o), 3),
                              "gteps": round(te_o / (sum(ms_o) * 1e-3) / 1e9, 4),
                              "sample": "20 sequential BFS (levels), the same roots cycled"}, **_cpu_info()),
        "parity": {"levels_identical": ok_lv, "parents_graph500_valid": ok_pa,
                   "min_id_parents_identical": ok_min, "roots_checked": len(roots)},
        "clocks": clk.summary()})
    return out


def config_grid(tq, dev, local, args, hbm_peak, peak_src):
    """BASELINE.json configs[2]: 4096 x 4096 grid from the corner (8,191
    levels): ms and us per level, median of 3 after 2 warm-up runs."""
    import numpy as np
    import torch
    import oracle
    rows = 4096
    rp, col = make_graph("grid", rows, 0, dev)
    n = rp.numel() - 1
    lv = torch.empty(n, dtype=torch.int32, device=dev)
    pa = torch.empty_like(lv)
    out = {"workload": "grid4096", "graph": "grid 4096x4096, 4-neighbour", "n_vertices": n,
           "nnz": int(col.numel()), "root": 0,
           "l2": "inputs larger than L2 (CSR %.0f MB)" % (((n + 1) * 8 + col.numel() * 4) / 1e6)}
    with ClockSampler(local) as clk:
        with tq.BfsPlan(rp, col, variant=args.variant, device=local) as plan:
            for _ in range(2):
                plan.run(0, lv, pa)
            sts = [plan.run(0, lv, pa) for _ in range(3)]
        v = torch.arange(n, device=dev, dtype=torch.int64)
        closed = bool(torch.equal(lv.long(), v // rows + v % rows))
        rp_h, col_h = rp.cpu().numpy(), col.cpu().numpy()
        rule = oracle.validate_tree(rp_h, col_h, 0, lv.cpu().numpy(), pa.cpu().numpy())[0]
        lo, _, info = oracle.bfs(rp_h, col_h, 0, parents=False)
    ms = _median([s["ms"] for s in sts])
    levels = sts[0]["max_level"] + 1
    out.update({
        "ms_median": round(ms, 3), "ms_kernel_median": round(_median([s["ms_kernel"] for s in sts]), 3),
        "us_per_level": round(ms * 1e3 / levels, 3), "levels": levels,
        "gteps": round(sts[0]["traversed_edges"] / (ms * 1e-3) / 1e9, 4),
        "persistent_threads": sts[0]["persistent_threads"],
        "roofline": _roofline(sts, hbm_peak, peak_src),
        "cpu_baseline": dict({"kind": "oracle", "cores": 1, "ms": round(info["seconds_levels"] * 1e3, 1),
                              "gteps": round(info["traversed_edges"] / info["seconds_levels"] / 1e9, 4),
                              "sample": "one sequential BFS (levels) from the corner"}, **_cpu_info()),
        "parity": {"levels_closed_form_r_plus_c": closed, "levels_identical": bool(np.array_equal(lv.cpu().numpy(), lo)),
                   "parents_graph500_valid": rule == 0},
        "clocks": clk.summary()})
    return out


def config_kron24(tq, dev, local, args, hbm_peak, peak_src):
    """BASELINE.json configs[3]: Kronecker scale 24 on one B200: one root
    (median of 5 after a warm-up) and an 8-root batch, HBM and L2-probe
    rooflines, the oracle on the first root."""
    import numpy as np
    import torch
    import oracle
    rp, col = make_graph("kron", 24, 16, dev)
    rp_h = rp.cpu().numpy()
    roots = pick_roots("kron", rp_h, 8)
    n = rp.numel() - 1
    lv = torch.empty(n, dtype=torch.int32, device=dev)
    pa = torch.empty_like(lv)
    out = {"workload": "kron24", "graph": "kron 24 ef16", "n_vertices": n, "nnz": int(col.numel()),
           "roots": roots, "l2": "inputs larger than L2 (CSR %.0f MB)" % (((n + 1) * 8 + col.numel() * 4) / 1e6)}
    with ClockSampler(local) as clk:
        with tq.BfsPlan(rp, col, variant=args.variant, device=local) as plan:
            plan.run(roots[1], lv, pa)
            single = [plan.run(roots[0], lv, pa) for _ in range(5)]
            lv0, pa0 = lv.cpu().numpy(), pa.cpu().numpy()
            batch = [plan.run(r, lv, pa) for _ in range(2) for r in roots]
        probe_g = tq.probe_ceiling(_mirror_bytes(n), 1 << 28, device=local)
        col_h = col.cpu().numpy()
        lo, _, info = oracle.bfs(rp_h, col_h, roots[0], parents=False)
        rule = oracle.validate_tree(rp_h, col_h, roots[0], lv0, pa0)[0]
    s0 = single[2]
    ms1 = _median([s["ms"] for s in single])
    out.update({
        "single_root": {"root": roots[0], "ms_median": round(ms1, 4),
                        "gteps": round(s0["traversed_edges"] / (ms1 * 1e-3) / 1e9, 3),
                        "roofline": _roofline(single, hbm_peak, peak_src, probe_g)},
        "batch8": {"gteps": round(sum(s["traversed_edges"] for s in batch) / (sum(s["ms"] for s in batch) * 1e-3) / 1e9, 3),
                   "gteps_kernel_only": round(sum(s["traversed_edges"] for s in batch) /
                                              (sum(s["ms_kernel"] for s in batch) * 1e-3) / 1e9, 3),
                   "runs": len(batch), "roofline": _roofline(batch, hbm_peak, peak_src, probe_g)},
        "cpu_baseline": dict({"kind": "oracle", "cores": 1, "ms": round(info["seconds_levels"] * 1e3, 1),
                              "gteps": round(info["traversed_edges"] / info["seconds_levels"] / 1e9, 4),
                              "sample": "one sequential BFS (levels) of the first root"}, **_cpu_info()),
        "parity": {"root": roots[0], "levels_identical": bool(np.array_equal(lv0, lo)),
                   "parents_graph500_valid": rule == 0},
        "clocks": clk.summary()})
    return out


def config_queue(tq, local, args):
    """BASELINE.json configs[1]: queue throughput and weak-scaling efficiency
    E(P) = (X(P) / P) / (X(1 group) / 1 group) at full occupancy for the warp
    proxy (the paper's) and the pipelined CTA proxy ("thread
    group"), b = 1 / 8 / 32, 1,024 iterations per warp (256 at b = 32); the
    single-group rate is the median of 5 runs of the same variant and depth.  Comparators at b = 32 (CAS queues
    naive and with a bounded back-off) and the same-address atomic ceiling.
    Every run's item multiset is checked (count, sum and xor of splitmix64
    over the items)."""
    import numpy as np
    import oracle
    from inputs import fingerprint, item_of
    iters, cap = 1024, 1 << 22

    fp_cache = {}

    def expected(n):
        # (count, sum, xor) of the n generated items, streamed in 16M chunks
        # and cached per n (the full-GPU runs of both proxies share n)
        if n not in fp_cache:
            c, sm, xr = 0, 0, 0
            for a in range(0, n, 1 << 24):
                k, s_, x_ = fingerprint(item_of(3, np.arange(a, min(n, a + (1 << 24)), dtype=np.uint64)))
                c, sm, xr = c + k, (sm + s_) & 0xFFFFFFFFFFFFFFFF, xr ^ x_
            fp_cache[n] = (c, sm, xr)
        return fp_cache[n]

    def run(v, w, b, d, items=None, relaxed=False, backoff=0):
        items = items or w * b * (iters if b < 32 else iters // 4)  # b = 32: 256 iterations per warp
        r = tq.queue_bench(v, warps=w, batch=b, items=items, capacity=cap, seed=3, depth=d, device=local,
                           timeout_s=30, relaxed_poll=relaxed, cas_backoff_ns=backoff)
        exp = expected(r["items"])
        ok = ((r["enq"], r["sum_enq"], r["xor_enq"]) == tuple(exp) and
              (r["deq"], r["sum_deq"], r["xor_deq"]) == tuple(exp))
        return r, 2 * r["items"] / (r["ms"] * 1e-3) / 1e6, ok

    full_w = tq.queue_bench("rf_an", warps=0, batch=1, items=1 << 20, capacity=cap, device=local)["warps"]
    out = {"unit": "M ops/s (enqueue + dequeue)", "capacity": cap, "iters_per_warp": {"b=1,8": iters, "b=32": iters // 4},
           "full_threads": 32 * full_w, "scaling": []}
    conserved = True
    with ClockSampler(local) as clk:
        # (relaxed arrival checks -- queue_bench(relaxed_poll=True) -- measured
        # the same E as acquire ones; not repeated here)
        w_fulls = {}
        for v, d, g, relaxed in (("rf_an", 1, 1, False), ("rf_an_cta", 2, 8, False)):
            for b in (1, 8, 32):
                t_run = time.time()
                base, base_empty = [], []
                for _ in range(5):
                    r1, x, ok = run(v, g, b, d, relaxed=relaxed)
                    base.append(x / g)
                    base_empty.append(r1["empty_retries"] / r1["items"])
                    conserved &= ok
                if (v, d) not in w_fulls:
                    w_fulls[(v, d)] = tq.queue_bench(v, warps=0, batch=b, items=1 << 22, capacity=cap, depth=d,
                                                     device=local)["warps"]
                r, x, ok = run(v, w_fulls[(v, d)], b, d, relaxed=relaxed)
                conserved &= ok
                w = r["warps"]
                out["scaling"].append({"variant": v, "depth": d, "group_warps": g, "b": b,
                                       "poll": "relaxed" if relaxed else "acquire", "threads": 32 * w,
                                       "mops": round(x, 1), "single_group_mops_per_warp": round(_median(base), 3),
                                       "E": round(x / w / _median(base), 3),
                                       "us_per_iteration": round(2 * b / (x / w), 3),
                                       "single_group_us_per_iteration": round(2 * b / _median(base), 3),
                                       "empty_polls_per_item": round(r["empty_retries"] / r["items"], 3),
                                       "single_group_empty_polls_per_item": round(_median(base_empty), 3),
                                       "atomics_per_item": round(r["atomics"] / r["items"], 4),
                                       "wall_s": round(time.time() - t_run, 2)})
        # comparators at b = 32, at the paper's 14,336 threads and at
        # full occupancy; the CAS queues naive and with a bounded back-off
        comps = []
        for v, bo in (("rf_an", 0), ("per_thread_afa", 0), ("cas_retry", 0), ("cas_retry", 2048), ("an", 0),
                      ("an", 2048)):
            for w in (448, 0):
                it = 2 if v in ("cas_retry", "an") else 16
                if not w and (v, 1) not in w_fulls:
                    w_fulls[(v, 1)] = tq.queue_bench(v, warps=0, batch=32, items=1 << 22, capacity=cap,
                                                     device=local)["warps"]
                w_run = w or w_fulls[(v, 1)]
                t_run = time.time()
                r, x, ok = run(v, w_run, 32, 1, items=w_run * 32 * it, backoff=bo)
                conserved &= ok
                comps.append({"variant": v, "cas_backoff_ns": bo, "b": 32, "threads": 32 * r["warps"],
                              "mops": round(x, 1), "atomics_per_item": round(r["atomics"] / r["items"], 4),
                              "cas_failures_per_item": round(r["cas_failures"] / r["items"], 4),
                              "wall_s": round(time.time() - t_run, 2)})
        out["comparators"] = comps
        r = tq.queue_bench("atomic_ceiling", warps=0, batch=32, items=1 << 24, capacity=cap, device=local)
        out["same_address_atomics_per_s_G"] = round(r["atomics"] / (r["ms"] * 1e-3) / 1e9, 3)
    n = 1 << 22
    sec, _ = oracle.queue_replay(cap, item_of(3, np.arange(n)), 32)
    out["cpu_baseline"] = dict({"kind": "oracle", "cores": 1, "mops": round(2 * n / sec / 1e6, 1),
                                "sample": "sequential ticket model, 2^22 items in batches of 32"}, **_cpu_info())
    out["conserved"] = bool(conserved)
    out["clocks"] = clk.summary()
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="tq", choices=["tq", "reference"])
    ap.add_argument("--workload", default=os.environ.get("TQ_BENCH_WORKLOAD", "kron26x64"),
                    choices=sorted(WORKLOADS))
    ap.add_argument("--variant", default="rf_an")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-priority", type=int, default=0, help="e2e leg: priority of the run streams")
    ap.add_argument("--e2e-relabel", type=int, default=-1,
                    help="e2e leg: bfs_opts.relabel of the per-step plans (default off: a plan rebuilt every "
                         "step for 64 roots does not win its relabelling back, results/e2e_relabel_r02.log)")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-queue", action="store_true")
    ap.add_argument("--no-configs", action="store_true", help="skip configs 1-4 (headline workload only)")
    ap.add_argument("--cpu-budget", type=float, default=20.0)
    ap.add_argument("--parents", default="any", choices=["any", "min_id"])
    ap.add_argument("--chunk", type=int, default=0, help="bfs_opts.chunk of the device leg's plan (0 = default)")
    args = ap.parse_args()

    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    kind, a, ef, n_roots = WORKLOADS[args.workload]
    hbm_peak, peak_src = peaks()

    import numpy as np
    import torch

    if args.impl == "reference":
        if rank != 0:
            return
        run_reference(args, kind, a, ef, n_roots)
        return

    # TQ_DIST_BACKEND=gloo (test only): several ranks sharing the visible
    # GPUs (device = LOCAL_RANK mod count) with host-side collectives, to
    # exercise the N > 1 path on a one-GPU box; the product path is NCCL
    backend = os.environ.get("TQ_DIST_BACKEND", "nccl")
    local = local % max(torch.cuda.device_count(), 1) if backend == "gloo" else local
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    coll_dev = dev if backend == "nccl" else None  # device of the collectives' tensors
    # The process group is created at every N, N = 1 included (a one-rank NCCL
    # group on a plain `python bench.py`), so the N > 1 code path -- barriers
    # and the NCCL all-gather of per-rank stats -- runs in every bench run.
    import torch.distributed as dist
    if "MASTER_ADDR" not in os.environ:  # plain launch: a one-rank rendezvous on loopback
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ.setdefault("MASTER_PORT", str(free_port()))
    if backend == "nccl":
        dist.init_process_group("nccl", device_id=dev, rank=rank, world_size=world)
    else:
        dist.init_process_group(backend, rank=rank, world_size=world)

    import paper_conf_icpp_troendletj19_b200 as tq
    from paper_conf_icpp_troendletj19_b200 import multiroot

    # ---- inputs (not timed): generated on the device, replicated per rank ----
    t_gen = time.time()
    row_ptr, col = make_graph(kind, a, ef, dev)
    rp_host = row_ptr.cpu().numpy()
    roots = pick_roots(kind, rp_host, n_roots)
    mine = multiroot.split_roots(roots, rank, world)
    n = int(row_ptr.numel()) - 1
    t_gen = time.time() - t_gen

    stream = torch.cuda.current_stream(dev)
    plan = tq.BfsPlan(row_ptr, col, variant=args.variant, stream=stream, device=local,
                      parents=args.parents, chunk=args.chunk)
    level = torch.empty(n, dtype=torch.int32, device=dev)
    parent = torch.empty(n, dtype=torch.int32, device=dev)

    def run_root(r):
        return plan.run(r, level, parent, grow_on_full=True)

    multiroot.run_local(run_root, mine, steps=args.warmup)
    # the expansion's second ceiling, measured live on this GPU (outside the
    # timed region): random 1-byte L2 probes over a table the size of the
    # level mirror, at the persistent kernel's shape
    mirror_bytes = n if n <= (1 << 25) else (n + 7) // 8 * 4  # byte / nibble mirror (R8)
    probe_g = tq.probe_ceiling(max(mirror_bytes, 1 << 12), 1 << 28, device=local) if kind == "kron" else None

    # ---- timed region: K steps, barrier + sync on both sides, device events ----
    if dist:
        dist.barrier()
    torch.cuda.synchronize(dev)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        e0.record(stream)
        all_stats = multiroot.run_local(run_root, mine, steps=args.steps)
        e1.record(stream)
        torch.cuda.synchronize(dev)
    if dist:
        dist.barrier()
    ms_total = e0.elapsed_time(e1)
    regrows = plan.regrows
    # outputs of the last timed root, from the long-running plan that was timed
    # (its tickets have crossed the 2^32 wrap of the sequence tags many times)
    last_root = mine[-1] if mine else None
    last_level = level.cpu().numpy() if mine else None
    last_parent = parent.cpu().numpy() if mine else None
    plan_tickets = plan.tickets()

    # NCCL all-gather of per-rank stats (the only collective; outside the data path)
    agg = multiroot.aggregate(multiroot.gather(multiroot.local_vector(all_stats, ms_total), dist, coll_dev))
    ms_max = agg["ms"]
    te_all = agg["traversed_edges"]
    reached_all = agg["reached"]
    kern_ms_all = agg["ms_kernel_sum"]
    launches = int(agg["launches"])
    runs_all = int(agg["runs"])

    gteps = te_all / (ms_max * 1e-3) / 1e9
    ms_per_step = ms_max / args.steps

    # roofline of the dominant kernel (bfs_persistent), per launch
    alg_bytes = algorithmic_bytes(te_all, reached_all) / runs_all
    avg_kernel_s = kern_ms_all / runs_all * 1e-3
    achieved = alg_bytes / avg_kernel_s / 1e9
    traffic, traffic_src = None, None
    tp = os.path.join(ROOT, "profiles", f"ncu_traffic_{args.workload}.json")
    if os.path.exists(tp):  # one committed `ncu --set full` capture of this kernel (per launch)
        tj = json.load(open(tp))
        traffic = tj.get("dram_bytes_per_launch")
        traffic_src = f"profiles/ncu_traffic_{args.workload}.json ({tj.get('capture_round', '?')})"
    s_last = all_stats[-1] if all_stats else {}
    kernel_name = ("bfs_persistent_kernel<%s, %s mirror, %d ticket lanes, %d threads>" %
                   (args.variant.upper(), {8: "byte", 4: "nibble"}.get(s_last.get("mirror_bits"), "?"),
                    s_last.get("ticket_lanes", 0), s_last.get("persistent_threads", 0)))

    probe_roof = None
    if probe_g:
        scanned = agg["edges_scanned"] / runs_all
        probe_roof = {"bound": "l2_random_probe", "achieved": round(scanned / avg_kernel_s / 1e9, 1),
                      "peak": round(probe_g, 1), "unit": "G probes/s",
                      "frac": round(scanned / avg_kernel_s / 1e9 / probe_g, 4),
                      "what": "CSR entries scanned per second of the persistent kernel (one random "
                              "32 B L2 sector each: the level-mirror probe) vs tq_probe_ceiling over a "
                              "table of the mirror's size, measured in this run"}

    # ---- e2e through the public API with host buffers (pinned), every step ----
    e2e = None
    if not args.no_e2e:
        rp_pin = torch.empty(n + 1, dtype=torch.int64, pin_memory=True)
        col_pin = torch.empty(col.numel(), dtype=torch.int32, pin_memory=True)
        rp_pin.copy_(row_ptr)
        col_pin.copy_(col)
        lv_pin = torch.empty(n, dtype=torch.int32, pin_memory=True)
        pa_pin = torch.empty(n, dtype=torch.int32, pin_memory=True)
        rp_np, col_np, lv_np, pa_np = rp_pin.numpy(), col_pin.numpy(), lv_pin.numpy(), pa_pin.numpy()
        plan.close()
        torch.cuda.empty_cache()
        # Step k+1's plan (its 9 GB H2D of the pinned host CSR, in 1 MiB
        # pieces on its own stream) is built by a helper thread while step k's
        # batch runs: every step's H2D and D2H stay inside the timed region,
        # overlapped with the BFS of the neighbouring step (ctypes releases the
        # GIL during the C calls).
        # (priority 0 = the device's least, as the library's own build stream:
        # a high-priority BFS starves the next step's relabelling kernels,
        # results/e2e_relabel_r02.log)
        streams = [torch.cuda.Stream(dev, priority=args.e2e_priority), torch.cuda.Stream(dev, priority=args.e2e_priority)]
        def make_plan(k):
            return tq.BfsPlan(rp_np, col_np, variant=args.variant, stream=streams[k % 2], device=local,
                              parents=args.parents, relabel=args.e2e_relabel)

        def run_steps(n_steps, roots_):
            """n_steps steps: step k runs every root on plan k (built from the
            pinned host CSR) while a helper thread builds plan k+1."""
            te, step_s = 0, []
            nxt = make_plan(0)
            for k in range(n_steps):
                ts0 = time.perf_counter()
                hp, box, th = nxt, {}, None
                if k + 1 < n_steps:
                    def build(k=k, box=box):
                        try:
                            box["plan"] = make_plan(k + 1)
                        except Exception as ex:  # re-raised in the main thread
                            box["error"] = ex
                    th = threading.Thread(target=build)
                    th.start()
                # one C-ABI call per step: every root's level and parent arrays
                # are copied to the (reused) pinned host buffers, D2H overlapped
                # with the next root's BFS on a second stream
                for s_ in hp.run_batch(roots_, lv_np, pa_np, stride=0):
                    te += s_["traversed_edges"]
                ts1 = time.perf_counter()
                if th is not None:
                    th.join()
                    if "error" in box:
                        raise box["error"]
                    nxt = box["plan"]
                ts2 = time.perf_counter()
                hp.close()
                step_s.append([round(ts1 - ts0, 3), round(ts2 - ts1, 3), round(time.perf_counter() - ts2, 3)])
            return te, step_s

        # untimed warm-up (as the device leg has W warm-up steps): three steps
        # of the timed loop on 2 roots each, so that the library's memory pool
        # has grown to the loop's peak (two plans alive, one being built)
        run_steps(3, mine[:2])
        if dist:
            dist.barrier()
        torch.cuda.synchronize(dev)
        t0 = time.perf_counter()
        te_e2e, step_s = run_steps(args.steps, mine)
        torch.cuda.synchronize(dev)
        sec = time.perf_counter() - t0
        secv = torch.tensor([sec, te_e2e], dtype=torch.float64, device=coll_dev)
        if dist:
            o2 = torch.empty(world * 2, dtype=torch.float64, device=coll_dev)
            dist.all_gather_into_tensor(o2, secv)
            o2 = o2.view(world, 2).cpu().numpy()
            sec_max, te_tot = float(o2[:, 0].max()), float(o2[:, 1].sum())
        else:
            sec_max, te_tot = sec, float(te_e2e)
        e2e = {"value": te_tot / sec_max / 1e9, "unit": "GTEPS",
               "h2d_bytes_per_step": int((n + 1) * 8 + col.numel() * 4),
               "d2h_bytes_per_step": int(len(mine) * n * 8),
               "step_s_batch_wait_destroy": step_s,
               "timed": "host perf_counter from the first bfs_plan_create (pinned host CSR: H2D) to the "
                        "last step's synchronised end; per step bfs_plan_run_batch (all roots, pinned host "
                        "level/parent: D2H per root) while the next step's plan (H2D) is built on a second "
                        "stream"}

    # ---- CPU baseline: the oracle, 1 core, bounded sample, rank 0 at N=1 ----
    cpu = None
    parity = None
    if rank == 0 and not args.no_cpu and last_root is not None:
        import oracle
        col_host = col.cpu().numpy()
        # the oracle's first root is the last timed root: its levels are the
        # parity reference for the timed plan's output (and part of the sample)
        sample_roots_ = [last_root] + [r for r in mine if r != last_root]
        teps, done, sec, lv0 = cpu_oracle_sample(rp_host, col_host, sample_roots_, args.cpu_budget)
        rule, bad = oracle.validate_tree(rp_host, col_host, last_root, last_level, last_parent)
        parity = {"root": int(last_root), "levels_identical": bool(np.array_equal(last_level, lv0)),
                  "parents_graph500_valid": rule == 0, "validate_rule": rule,
                  "plan_tickets_after_timed_runs": [int(t) for t in plan_tickets],
                  "what": "last timed root of the timed (long-running) plan vs the oracle"}
        cpu = {"value": teps / 1e9, "unit": "GTEPS", "cores": 1, "kind": "oracle",
               "nproc": os.cpu_count(), "cpu_model": cpu_model(),
               "sample": f"{len(done)} of the {len(roots)} roots of the same graph, sequential "
                         f"BFS levels only ({sec:.1f} s of CPU)"}

    # ---- the other BASELINE.json configs on this GPU (rank 0; after the timed
    # region and the e2e leg): config 1 (R-MAT s10, GPU us beside the oracle's
    # ms), config 2 (queue throughput + E(P)), config 3 (grid 4096^2, us per
    # level), config 4 (Kronecker s24, one root + 8 roots, rooflines) ----
    configs = None
    if rank == 0 and not args.no_configs:
        configs = {}
        for key, fn in (("2_queue", lambda: config_queue(tq, local, args)),
                        ("1_rmat10", lambda: config_rmat10(tq, dev, local, args)),
                        ("3_grid4096", lambda: config_grid(tq, dev, local, args, hbm_peak, peak_src)),
                        ("4_kron24", lambda: config_kron24(tq, dev, local, args, hbm_peak, peak_src))):
            if key == "2_queue" and args.no_queue:
                continue
            t_c = time.time()
            try:
                configs[key] = fn()
            except Exception as ex:  # report, do not lose the headline line
                configs[key] = {"error": f"{type(ex).__name__}: {ex}"}
            configs[key]["wall_s"] = round(time.time() - t_c, 1)
            torch.cuda.empty_cache()
    if dist:
        dist.barrier()

    csr_mb = ((n + 1) * 8 + col.numel() * 4) / 1e6
    if rank == 0:
        line = {
            "metric": "BFS GTEPS (batched multi-root, persistent-thread RF/AN queue)",
            "value": round(gteps, 4),
            "unit": "GTEPS",
            "n_gpus": world,
            "steps": args.steps,
            "warmup": args.warmup,
            "ms_per_step": round(ms_per_step, 3),
            "higher_is_better": True,
            "scaling": "strong",
            "vs_baseline": None,
            "dtype": "int32/int64 (integer path)",
            "data": "synthetic (seeded Kronecker/Graph500 R-MAT generated on the device)",
            "config": {"workload": args.workload, "graph": f"{kind} {a}" + (f" ef{ef}" if ef else ""),
                       "n_vertices": n, "nnz": int(col.numel()), "roots_total": len(roots),
                       "roots_per_rank": len(mine), "variant": args.variant,
                       "parallelism": f"roots split over {world} rank(s), graph replicated",
                       "l2": ("inputs larger than L2 (CSR %.0f MB > 126 MB)" % csr_mb) if csr_mb > 126 else
                             ("inputs smaller than L2 (CSR %.1f MB; not flushed between roots: a parity-size "
                              "workload, not the metric's)" % csr_mb),
                       "persistent_threads": max((st["persistent_threads"] for st in all_stats),
                                                 default=tq.persistent_threads(args.variant, device=local))},
            "roofline": {"bound": "hbm", "achieved": round(achieved, 1), "peak": hbm_peak,
                         "unit": "GB/s", "frac": round(achieved / hbm_peak, 4), "traffic": traffic,
                         "traffic_source": traffic_src, "kernel": kernel_name, "peak_source": peak_src,
                         "alg_bytes_per_launch": int(alg_bytes),
                         "avg_launch_ms": round(avg_kernel_s * 1e3, 4)},
            "roofline_l2_probe": probe_roof,
            "configs": configs,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": launches,
            "traversed_edges_total": int(te_all),
            "runs_total": runs_all,
            "process_group": {"backend": backend, "world_size": world},
            "clocks": clk.summary(),
            "parity": parity,
            "graph_gen_s": round(t_gen, 2),
            "queue_regrows": regrows,
        }
        print(json.dumps(line), flush=True)
    if dist:
        dist.destroy_process_group()


def run_reference(args, kind, a, ef, n_roots):
    """--impl reference: the oracle as it stands on the host cores."""
    import numpy as np
    import torch

    import oracle
    dev = torch.device("cuda", 0) if torch.cuda.is_available() else None
    if dev is not None:
        row_ptr, col = make_graph(kind, a, ef, dev)
        rp, cl = row_ptr.cpu().numpy(), col.cpu().numpy()
        del row_ptr, col
    else:  # CPU-only host: numpy generator (small workloads only)
        from inputs import grid_csr, kronecker_csr
        g = kronecker_csr(a, ef, GRAPH_SEED) if kind == "kron" else grid_csr(a)
        rp, cl = g.row_ptr, g.col
    roots = pick_roots(kind, rp, n_roots)
    oracle.build()

    def step(i):
        r = roots[i % len(roots)]
        _, _, info = oracle.bfs(rp, cl, r, parents=False)
        return info["traversed_edges"], info["seconds_levels"]

    for i in range(args.warmup):
        step(i)
    te, sec = 0, 0.0
    for i in range(args.steps):
        t, s = step(args.warmup + i)
        te += t
        sec += s
    v = te / sec / 1e9
    print(json.dumps({
        "impl": "reference", "metric": "BFS GTEPS (batched multi-root, persistent-thread RF/AN queue)",
        "value": round(v, 6), "unit": "GTEPS", "n_gpus": int(os.environ.get("WORLD_SIZE", 1)),
        "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(sec / args.steps * 1e3, 3),
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
        "dtype": "int32/int64 (integer path)", "data": "synthetic",
        "config": {"workload": args.workload, "graph": f"{kind} {a}" + (f" ef{ef}" if ef else ""),
                   "n_vertices": int(rp.size - 1), "nnz": int(cl.size), "roots_total": len(roots),
                   "parallelism": "rank 0 only: the sequential oracle on one host core"},
        "cpu_baseline": {"value": round(v, 6), "unit": "GTEPS", "cores": 1, "kind": "oracle",
                         "sample": f"one root of the workload per step ({args.steps} steps)"},
        "e2e": {"value": round(v, 6), "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


if __name__ == "__main__":
    main()
