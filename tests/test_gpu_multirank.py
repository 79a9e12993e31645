"""The N > 1 path of bench.py on one GPU: two ranks launched by torchrun share
the GPU (TQ_DIST_BACKEND=gloo, test-only host collectives; the product path
is NCCL), split the roots, and the all-gathered aggregate must cover every
root exactly once -- the same traversed-edge total as the one-rank run, which
itself goes through a one-rank NCCL process group."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
FLAGS = ["--workload", "kron20x16", "--steps", "2", "--warmup", "1", "--no-e2e", "--no-cpu", "--no-configs",
         "--no-queue"]


def _line(cmd, env):
    out = subprocess.run(cmd, capture_output=True, text=True, env=env, timeout=900, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    return json.loads(lines[0])


def test_two_ranks_cover_every_root_once():
    import __graft_entry__
    __graft_entry__.build()
    env = dict(os.environ)
    one = _line([sys.executable, "bench.py", *FLAGS], env)
    assert one["process_group"] == {"backend": "nccl", "world_size": 1}
    env2 = dict(env, TQ_DIST_BACKEND="gloo")
    two = _line([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
                 "--master-addr", "127.0.0.1", "--master-port", "29517", "bench.py", "--gpus", "2", *FLAGS],
                env2)
    assert two["n_gpus"] == 2 and two["process_group"]["world_size"] == 2
    assert two["runs_total"] == one["runs_total"] == 2 * 16
    assert two["traversed_edges_total"] == one["traversed_edges_total"]
    assert two["config"]["roots_per_rank"] == 8


def test_default_line_carries_every_config():
    """The bench line's contract keys on a quick workload, with configs 1, 3 and
    4 (the queue config is covered by test_gpu_queue.py): each carries parity,
    clocks and an oracle cpu_baseline with the host's core count."""
    import __graft_entry__
    __graft_entry__.build()
    d = _line([sys.executable, "bench.py", "--workload", "kron20x16", "--steps", "2", "--warmup", "3",
               "--no-e2e", "--no-queue", "--cpu-budget", "2"], dict(os.environ))
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "roofline", "roofline_l2_probe", "cpu_baseline", "clocks",
              "gpu_launches", "parity", "configs"):
        assert k in d, k
    assert d["parity"]["levels_identical"] and d["parity"]["parents_graph500_valid"]
    assert d["cpu_baseline"]["nproc"] >= 1 and d["cpu_baseline"]["kind"] == "oracle"
    assert 0 < d["roofline"]["frac"] < 1.5 and d["gpu_launches"] == 3 * 16 * 2
    for key in ("1_rmat10", "3_grid4096", "4_kron24"):
        c = d["configs"][key]
        assert "error" not in c, c
        assert all(v is True for k, v in c["parity"].items() if isinstance(v, bool)), c["parity"]
        assert c["cpu_baseline"]["nproc"] >= 1 and "clocks" in c
    assert d["configs"]["3_grid4096"]["levels"] == 8191
