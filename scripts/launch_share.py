"""Per-kernel share of the GPU time in an `ncu --metrics gpu__time_duration.sum --csv`
launch list (cold-cache, serialised: shares, not absolutes)."""
import collections
import csv
import sys

path, cmd = sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else ""
rows = list(csv.reader(open(path)))
h, tot, cnt = None, collections.Counter(), collections.Counter()
for r in rows:
    if r and r[0] == "ID":
        h = r
        continue
    if h and len(r) == len(h):
        d = dict(zip(h, r))
        if d.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(d["Metric Value"].replace(",", ""))
        v *= {"ns": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0, "nsecond": 1e-6}.get(d["Metric Unit"], 1.0)
        k = d["Kernel Name"][:70]
        tot[k] += v
        cnt[k] += 1
s = sum(tot.values())
print(f"Launch list of `{cmd}` under `ncu --metrics gpu__time_duration.sum --clock-control none`\n"
      f"(cold-cache and serialised: shares, not absolutes). Source: {path}\n")
for k, v in tot.most_common():
    print(f"{100 * v / s:7.2f}%  {v:11.3f} ms  {cnt[k]:5d} launches  {k}")
