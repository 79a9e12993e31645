"""A/B two builds of libtq.so on the same box: alternates runs of
scripts/sweep_bfs.py with TQ_LIB pointing at each build and prints the mean
kernel ms per workload (interleaving cancels slow drift in clocks / L2 state).

  python scripts/ab_bfs.py build/libtq_A.so build/libtq_B.so --workloads kron24x8,kron26x64
"""
import argparse
import json
import os
import statistics
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ap = argparse.ArgumentParser()
ap.add_argument("libs", nargs="+")
ap.add_argument("--workloads", default="kron24x8,kron26x64,grid4096")
ap.add_argument("--roots", type=int, default=6)
ap.add_argument("--reps", type=int, default=2)
ap.add_argument("--extra", default="")
args = ap.parse_args()

res = {}
for wl in args.workloads.split(","):
    nr = 1 if wl.startswith("grid") else args.roots
    for rep in range(args.reps):
        for lib in args.libs:
            env = dict(os.environ, TQ_LIB=os.path.abspath(lib))
            out = subprocess.run([sys.executable, os.path.join(HERE, "sweep_bfs.py"), "--workload", wl,
                                  "--chunks", "512", "--roots", str(nr), *args.extra.split()],
                                 env=env, capture_output=True, text=True)
            if out.returncode != 0:
                print(f"{wl} {lib}: FAILED {out.stderr.strip().splitlines()[-1:]}", flush=True)
                continue
            for line in out.stdout.splitlines():
                if line.startswith("{"):
                    d = json.loads(line)
                    res.setdefault((wl, lib), []).append(d)
for (wl, lib), ds in res.items():
    ms = [d["ms"] for d in ds]
    print(json.dumps({"workload": wl, "lib": os.path.basename(lib), "n": len(ms),
                      "ms_mean": round(statistics.mean(ms), 3), "ms_min": min(ms),
                      "scan_x": round(statistics.mean(d["scan_x"] for d in ds), 3),
                      "tasks": round(statistics.mean(d["tasks"] for d in ds)),
                      "min_atomics": round(statistics.mean(d["min_atomics"] for d in ds))}), flush=True)
