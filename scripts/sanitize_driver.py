"""Small workloads for compute-sanitizer (P:281 queue-full path):
every BFS variant on an R-MAT scale-10 graph (both parent rules), a
queue-full abort (capacity 64) followed by a reset run, the chunk queue
(chunk = 32), the queue micro-benchmark of every variant, and the
device-API user kernel including its queue-full abort.  Exits non-zero on any
mismatch; compute-sanitizer reports memory / sync / race errors itself."""
import ctypes
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np
import torch

import oracle
import paper_conf_icpp_troendletj19_b200 as tq
from inputs import kronecker_csr, sample_roots
from paper_conf_icpp_troendletj19_b200 import _build

g = kronecker_csr(10, 16, 1)
rp, col = torch.from_numpy(g.row_ptr).cuda(), torch.from_numpy(g.col).cuda()
roots = [int(r) for r in sample_roots(g.row_ptr, 2, 2)]
lv = torch.empty(g.n_vertices, dtype=torch.int32, device="cuda")
pa = torch.empty_like(lv)
for v in ("rf_an", "per_thread_afa", "cas_retry", "an"):
    for parents in ("any", "min_id"):
        with tq.BfsPlan(rp, col, variant=v, parents=parents, threads=4096, timeout_s=60, chunk=32) as plan:
            for r in roots:
                plan.run(r, lv, pa)
                lo, _, _ = oracle.bfs(g.row_ptr, g.col, r, parents=False)
                assert np.array_equal(lv.cpu().numpy(), lo), (v, parents, r)
# round 2, session 3 paths: the shared-memory single-block BFS (and its
# queue-full abort), the persistent grid with level-carrying tokens, a
# relabelled plan with hub chunks, and a narrow level field (fenced tokens mixed in)
for sp in (1, -1):
    for parents in ("any", "min_id"):
        with tq.BfsPlan(rp, col, parents=parents, smem_path=sp, threads=4096, timeout_s=60) as plan:
            for r in roots:
                plan.run(r, lv, pa)
                lo, _, _ = oracle.bfs(g.row_ptr, g.col, r, parents=False)
                assert np.array_equal(lv.cpu().numpy(), lo), ("smem", sp, parents, r)
try:
    tq.bfs(rp, col, int(np.argmax(g.degrees())), capacity=64, smem_path=1)
    raise SystemExit("expected a queue-full abort on the shared-memory path")
except tq.TQError as e:
    assert e.status == -4
g2 = kronecker_csr(12, 16, 3)
rp2, col2 = torch.from_numpy(g2.row_ptr).cuda(), torch.from_numpy(g2.col).cuda()
lv2 = torch.empty(g2.n_vertices, dtype=torch.int32, device="cuda")
pa2 = torch.empty_like(lv2)
for kw in ({"relabel": 1, "chunk": 32}, {"relabel": 1, "level_bits": 2, "parents": "min_id"}):
    with tq.BfsPlan(rp2, col2, threads=4096, timeout_s=60, **kw) as plan:
        for r in [int(x) for x in sample_roots(g2.row_ptr, 2, 4)]:
            plan.run(r, lv2, pa2)
            lo, _, _ = oracle.bfs(g2.row_ptr, g2.col, r, parents=False)
            assert np.array_equal(lv2.cpu().numpy(), lo), (kw, r)
with tq.BfsPlan(rp, col, capacity=64, threads=4096, timeout_s=60, smem_path=-1) as plan:
    try:
        plan.run(int(np.argmax(g.degrees())), lv, pa)
        raise SystemExit("expected a queue-full abort")
    except tq.TQError as e:
        assert e.status == -4
for v in ("rf_an", "per_thread_afa", "cas_retry", "an", "rf_an_cta"):
    tq.queue_bench(v, warps=16, batch=8, items=1 << 12, capacity=1 << 10, timeout_s=60)
L = ctypes.CDLL(_build.build_user_kernel(os.path.join(ROOT, "tests", "csrc", "devapi_test.cu"),
                                         os.path.join(ROOT, "tests", "libtqdevapi.so")))
L.devapi_run.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_uint64,
                         ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_double,
                         ctypes.c_void_p, ctypes.c_void_p]
for cap, per_lane in ((1 << 12, 3), (64, 4)):  # second case: 128 items into C = 64 -> abort
    q = tq.Queue(cap)
    q.reset_at((1 << 32) - 50)
    torch.cuda.synchronize()
    v = q.view()
    nm = torch.full((1 * 2 * 32,), per_lane, dtype=torch.int32, device="cuda")
    logs = torch.zeros(4096, dtype=torch.int32, device="cuda"), torch.zeros(4096, dtype=torch.int32, device="cuda")
    out = torch.zeros(4, dtype=torch.int64, device="cuda")
    assert L.devapi_run(ctypes.byref(v), 1, 2, nm.data_ptr(), (1 << 32) - 50, logs[0].data_ptr(),
                        logs[1].data_ptr(), 4096, 1, 60.0, out.data_ptr(), None) == 0
    st = q.counters()["status"]
    assert st == (0 if cap > 64 else 2), st
    q.close()
print("sanitize driver ok")
