"""Per-launch L2 atomic / memory metrics of the queue micro-benchmark kernels
from an ncu report (one row per bench_kernel launch)."""
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "lts__t_sectors_op_atom.sum", "lts__t_sectors_op_red.sum",
        "lts__t_requests_srcunit_tex_op_atom_dot_alu.sum", "lts__d_atomic_input_cycles_active.max.pct_of_peak_sustained_elapsed",
        "lts__d_atomic_input_cycles_active.avg.pct_of_peak_sustained_elapsed", "lts__t_sectors.sum",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "launch__grid_size", "launch__block_size"]
raw = subprocess.check_output(["ncu", "-i", sys.argv[1], "--page", "raw", "--csv"], text=True)
rows = list(csv.reader(io.StringIO(raw)))
hdr = rows[0]
for r in rows[2:]:
    d = dict(zip(hdr, r))
    if "bench" not in d.get("Kernel Name", ""):
        continue
    print(d["Kernel Name"][:60])
    for k in KEYS:
        if k in d:
            print(f"  {k:75s} {d[k]}")
