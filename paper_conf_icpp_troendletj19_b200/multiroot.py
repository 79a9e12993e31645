"""Batched multi-root BFS across ranks (BASELINE.json configs[4]).

Single-source BFS does not shard (one global FIFO), so the multi-GPU product
is a batch of independent roots: contiguous blocks of roots per rank, graph
replicated, no data-path collective, and one all-gather of per-rank stats at
the end (NCCL over NVLink on GPUs; gloo in the CPU tests). This module holds
only that host logic; each root is run by whatever `run_root` callable the
caller passes (the libtq plan on a GPU).
"""
from __future__ import annotations

from typing import Callable, Sequence

STAT_KEYS = ("ms", "traversed_edges", "reached", "ms_kernel", "launches", "runs", "edges_scanned")


def split_roots(roots: Sequence[int], rank: int, world: int) -> list[int]:
    """Contiguous block of `roots` for `rank` (sizes differ by at most one)."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank / world size")
    n = len(roots)
    return list(roots[rank * n // world:(rank + 1) * n // world])


def run_local(run_root: Callable[[int], dict], roots: Sequence[int], steps: int = 1) -> list[dict]:
    """Run this rank's roots `steps` times; returns the per-run stats."""
    out = []
    for _ in range(steps):
        for r in roots:
            out.append(run_root(int(r)))
    return out


def local_vector(stats: list[dict], ms_total: float, launches_per_run: int = 3):
    """Per-rank summary in STAT_KEYS order."""
    return [float(ms_total), float(sum(s["traversed_edges"] for s in stats)),
            float(sum(s["reached"] for s in stats)), float(sum(s.get("ms_kernel", 0.0) for s in stats)),
            float(launches_per_run * len(stats)), float(len(stats)),
            float(sum(s.get("edges_scanned", 0) for s in stats))]


def gather(vec, dist=None, device=None):
    """All-gather the per-rank summaries; returns a (world, len(STAT_KEYS)) list."""
    import torch
    t = torch.tensor(vec, dtype=torch.float64, device=device)
    if dist is None or not dist.is_initialized():
        return [t.tolist()]
    world = dist.get_world_size()
    out = torch.empty(world * t.numel(), dtype=torch.float64, device=device)
    dist.all_gather_into_tensor(out, t)
    return out.view(world, -1).tolist()


def aggregate(rows) -> dict:
    """Whole-job totals: time = max over ranks, counts = sums."""
    cols = list(zip(*rows))
    agg = {k: float(sum(c)) for k, c in zip(STAT_KEYS, cols)}
    agg["ms"] = float(max(cols[0]))
    agg["ms_kernel_sum"] = agg.pop("ms_kernel")
    agg["gteps"] = agg["traversed_edges"] / (agg["ms"] * 1e-3) / 1e9 if agg["ms"] > 0 else 0.0
    return agg
