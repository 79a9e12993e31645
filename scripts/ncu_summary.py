"""Summarise an ncu report: key throughput metrics and warp stall breakdown."""
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "launch__registers_per_thread", "launch__grid_size",
        "lts__t_sectors_op_atom.sum", "lts__t_sectors_op_red.sum", "lts__t_sectors_op_read.sum",
        "lts__t_sectors_op_write.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
        "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active"]


def main(path):
    raw = subprocess.check_output(["ncu", "-i", path, "--page", "raw", "--csv"], text=True)
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    d = dict(zip(hdr, zip(vals, units)))
    for k in KEYS:
        if k in d:
            print(f"{k:70s} {d[k][0]:>20s} {d[k][1]}")
    st = []
    pre = "smsp__pcsamp_warps_issue_stalled_"
    for h, (v, u) in d.items():
        if h.startswith(pre) and not h.endswith("_not_issued"):
            try:
                st.append((float(v.replace(",", "")), h[len(pre):]))
            except ValueError:
                pass
    tot = sum(v for v, _ in st) or 1.0
    print("--- warp stall reasons (share of PC samples) ---")
    for v, h in sorted(st, reverse=True)[:10]:
        print(f"{h:40s} {100.0 * v / tot:7.2f}%")


if __name__ == "__main__":
    main(sys.argv[1])
