"""Per source line: stall samples by reason, instructions executed, L2 sectors
(from `ncu --page source --csv --print-source cuda,sass`).  Top lines."""
import csv
import subprocess
import sys

raw = subprocess.check_output(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "cuda,sass"],
                              text=True, stderr=subprocess.DEVNULL)
hdr, f, rows = None, None, []
for r in csv.reader(raw.splitlines()):
    if not r:
        continue
    if r[0] == "File Path" or r[0] == "File Name":
        f = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or not r[0].isdigit():
        continue
    d = dict(zip(hdr, r))
    try:
        samp = int(d.get("Warp Stall Sampling (All Samples)", "0") or 0)
    except ValueError:
        continue
    reasons = {k[6:]: int(v) for k, v in d.items() if k.startswith("stall_") and "Not Issued" not in k
               and v.isdigit() and int(v) > 0}
    try:
        inst = int(d.get("Instructions Executed", "0") or 0)
    except ValueError:
        inst = 0
    rows.append((samp, f, int(r[0]), r[1].strip()[:70], reasons, inst))
tot = sum(x[0] for x in rows)
tinst = sum(x[5] for x in rows)
rows.sort(reverse=True)
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
print(f"total samples {tot}, warp instructions {tinst}")
for s, f, ln, src, rs, inst in rows[:n]:
    top = sorted(rs.items(), key=lambda kv: -kv[1])[:4]
    print(f"{100.0 * s / tot:5.2f}% inst {100.0 * inst / max(tinst, 1):5.2f}%  {f}:{ln:<5d} {src:<70s} " +
          " ".join(f"{k}={100.0 * v / max(s, 1):.0f}%" for k, v in top))
