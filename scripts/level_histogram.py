"""Per-level dynamic parallelism (Fig 3 analogue; NEXT row 3):
vertices available at each BFS level for every config graph, from GPU BFS
levels (verified equal to the oracle's in the parity tests)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import inputs.gpu as gg
import paper_conf_icpp_troendletj19_b200 as tq
from inputs import sample_roots

out = {}
graphs = {
    "rmat10 (config 1)": lambda: gg.kronecker_csr_cuda(10, 16, 1),
    "grid4096 (config 3)": lambda: gg.grid_csr_cuda(4096),
    "kron24 (config 4)": lambda: gg.kronecker_csr_cuda(24, 16, 1),
    "kron26 (config 5)": lambda: gg.kronecker_csr_cuda(26, 16, 1),
    "tree4 10,485,760 (paper synthetic)": lambda: gg.tree4_csr_cuda(10485760),
}
for name, make in graphs.items():
    rp, col = make()
    root = 0 if ("grid" in name or "tree" in name) else int(sample_roots(rp.cpu().numpy(), 1, 2)[0])
    level, _, st = tq.bfs(rp, col, root)
    lv = level[level >= 0].long()
    h = torch.bincount(lv).cpu().tolist()
    out[name] = {"root": root, "levels": len(h), "reached": int(lv.numel()), "max_width": max(h),
                 "histogram": h if len(h) <= 64 else {"first": h[:8], "max_at": int(torch.tensor(h).argmax()),
                                                       "last": h[-8:]}}
    print(name, out[name]["levels"], out[name]["max_width"], h[:12] if len(h) <= 64 else "")
    del rp, col, level
    torch.cuda.empty_cache()
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/level_histograms.json", "w"), indent=1)
