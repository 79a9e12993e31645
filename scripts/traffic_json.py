"""Write profiles/ncu_traffic_<workload>.json from one `ncu --set full` capture of
the persistent kernel: DRAM bytes read + written per launch (bench.py's
roofline.traffic)."""
import csv
import io
import json
import subprocess
import sys

rep, workload, rnd = sys.argv[1], sys.argv[2], sys.argv[3]
raw = subprocess.check_output(["ncu", "-i", rep, "--page", "raw", "--csv"], text=True, stderr=subprocess.DEVNULL)
rows = list(csv.reader(io.StringIO(raw)))
d = dict(zip(rows[0], zip(rows[2], rows[1])))
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}


def val(k):
    v, u = d[k]
    return float(v.replace(",", "")) * scale.get(u, 1.0)


out = {"workload": workload, "capture_round": rnd, "kernel": d["Kernel Name"][0] if "Kernel Name" in d else None,
       "capture": "ncu --set full --clock-control none, 1 launch (the second BFS of scripts/profile_bfs.py), "
                  "cold cache, serialised replay",
       "dram_bytes_read": val("dram__bytes_read.sum"), "dram_bytes_write": val("dram__bytes_write.sum"),
       "duration_ms_under_ncu": val("gpu__time_duration.sum") if d["gpu__time_duration.sum"][1] == "ms" else None,
       "report": rep + " (not committed); summary profiles/%s_ncu_full_%s.txt" % (rnd, workload)}
out["dram_bytes_per_launch"] = out["dram_bytes_read"] + out["dram_bytes_write"]
json.dump(out, open(f"profiles/ncu_traffic_{workload}.json", "w"), indent=1)
print(json.dumps(out))
