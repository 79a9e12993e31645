"""Top source lines by executed warp instructions and stall samples, from
`ncu --page source --csv --print-source cuda,sass` (CUDA-source rows only)."""
import csv
import subprocess
import sys

raw = subprocess.check_output(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source",
                               "cuda,sass"], text=True, stderr=subprocess.DEVNULL)
f, hdr, rows = None, None, []
for r in csv.reader(raw.splitlines()):
    if not r:
        continue
    if r[0] == "File Path":
        f = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if not r[0].isdigit() or hdr is None:
        continue
    d = dict(zip(hdr[2:], r[2:]))  # Address/Source(sass) columns are "-" on CUDA rows
    try:
        inst = int(r[hdr.index("Instructions Executed")])
        samp = int(r[hdr.index("Warp Stall Sampling (All Samples)")])
    except ValueError:
        continue
    rows.append((inst, samp, f, int(r[0]), r[1].strip()))
ti = sum(x[0] for x in rows) or 1
ts = sum(x[1] for x in rows) or 1
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
print(f"total warp instructions {ti}")
for inst, samp, f, ln, src in sorted(rows, reverse=True)[:n]:
    print(f"{100.0 * inst / ti:6.2f}% inst {100.0 * samp / ts:6.2f}% stall  {f}:{ln:<5d} {src[:90]}")
