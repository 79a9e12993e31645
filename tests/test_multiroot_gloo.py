"""N > 1 host path of the batched multi-root BFS, on CPU with gloo, world size 2.

Each rank runs its contiguous block of roots (here through the oracle, since
there is no GPU) and the per-rank stats are all-gathered; the aggregate must
equal a single-process run over all roots, every root exactly once.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icpp_troendletj19_b200 import multiroot


def test_split_roots_covers_each_root_once():
    roots = list(range(64))
    for world in (1, 2, 3, 4, 8, 64):
        parts = [multiroot.split_roots(roots, r, world) for r in range(world)]
        assert sum(parts, []) == roots
        assert max(map(len, parts)) - min(map(len, parts)) <= 1
    with pytest.raises(ValueError):
        multiroot.split_roots(roots, 2, 2)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_path):
    import oracle
    from inputs import kronecker_csr, sample_roots
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g = kronecker_csr(10, 16, 1)
    roots = [int(r) for r in sample_roots(g.row_ptr, 16, 2)]
    mine = multiroot.split_roots(roots, rank, world)

    def run_root(r):
        _, _, info = oracle.bfs(g.row_ptr, g.col, r, parents=False)
        return {"traversed_edges": info["traversed_edges"], "reached": info["reached"],
                "ms_kernel": 0.0}

    stats = multiroot.run_local(run_root, mine, steps=2)
    rows = multiroot.gather(multiroot.local_vector(stats, ms_total=10.0 + rank), dist)
    if rank == 0:
        agg = multiroot.aggregate(rows)
        np.save(out_path, np.array([agg["traversed_edges"], agg["reached"], agg["runs"], agg["ms"],
                                    agg["launches"]]))
    dist.barrier()
    dist.destroy_process_group()


def test_two_rank_gather_matches_single_process(tmp_path):
    import oracle
    from inputs import kronecker_csr, sample_roots
    out = str(tmp_path / "agg.npy")
    mp.spawn(_worker, args=(2, _free_port(), out), nprocs=2, join=True)
    te, reached, runs, ms, launches = np.load(out)
    g = kronecker_csr(10, 16, 1)
    roots = [int(r) for r in sample_roots(g.row_ptr, 16, 2)]
    exp_te = exp_re = 0
    for r in roots:
        _, _, info = oracle.bfs(g.row_ptr, g.col, r, parents=False)
        exp_te += info["traversed_edges"]
        exp_re += info["reached"]
    assert te == 2 * exp_te and reached == 2 * exp_re and runs == 2 * len(roots)
    assert ms == 11.0  # max over ranks, not the sum
    assert launches == 3 * runs
