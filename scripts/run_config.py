"""Run one of bench.py's config blocks alone (the same functions the default
bench line calls) and print its JSON: queue | rmat10 | grid | kron24."""
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
ap.add_argument("which", nargs="+")
ap.add_argument("--variant", default="rf_an")
args = ap.parse_args()
dev = torch.device("cuda", 0)
peak, src = bench.peaks()
for w in args.which:
    t = time.time()
    if w == "queue":
        r = bench.config_queue(tq, 0, args)
    elif w == "rmat10":
        r = bench.config_rmat10(tq, dev, 0, args)
    elif w == "grid":
        r = bench.config_grid(tq, dev, 0, args, peak, src)
    else:
        r = bench.config_kron24(tq, dev, 0, args, peak, src)
    r["wall_s"] = round(time.time() - t, 1)
    print(json.dumps({w: r}), flush=True)
