"""Top source lines by warp-stall samples from `ncu --page source --csv --print-source cuda,sass`."""
import csv
import subprocess
import sys

raw = subprocess.check_output(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "cuda,sass"],
                              text=True, stderr=subprocess.DEVNULL)
f = None
out = []
tot = 0
for r in csv.reader(raw.splitlines()):
    if not r:
        continue
    if r[0] == "File Path":
        f = r[1].split("/")[-1]
        continue
    if not r[0].isdigit():
        continue
    try:
        k = next(i for i in range(1, len(r) - 1) if r[i] == "-" and r[i + 1] == "-")
        s_all = int(r[k + 2])
    except (StopIteration, ValueError):
        continue
    src = ",".join(r[1:k]).strip()
    tot += s_all
    out.append((s_all, f, int(r[0]), src))
out.sort(reverse=True)
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
for s, f, ln, src in out[:n]:
    print(f"{100.0 * s / tot:6.2f}%  {f}:{ln:<5d} {src[:110]}")
