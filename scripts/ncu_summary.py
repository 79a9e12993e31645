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

    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}

    def num(k):
        try:
            return float(d[k][0].replace(",", "")) * scale.get(d[k][1], 1)
        except (KeyError, ValueError):
            return 0.0
    # L2 sector lookups from the SMs by the eviction-policy tag ncu attributes
    # them to.  The col stream is the only evict_first load and the level-mirror
    # probes the only evict_last loads, but their createpolicy hints set the
    # *hit* priority only (the source view lists them as HIT_FIRST/MISS_NORMAL,
    # HIT_LAST/MISS_NORMAL), so part of their misses are counted under
    # evict_normal with the per-task loads (row_ptr, W, x8, slots); the per-line
    # source view (`--page source`, L2 theoretical sectors) is the per-buffer
    # attribution.  A miss is a 32-byte sector fetched from DRAM or from the
    # other die's L2.
    print("--- L2 sector lookups from the SMs, by policy tag (per launch; see comment) ---")
    cls = [("evict_first-tagged loads (col)", "lts__t_sectors_srcunit_tex_op_read_evict_first_lookup_hit.sum",
            "lts__t_sectors_srcunit_tex_op_read_evict_first_lookup_miss.sum"),
           ("evict_last-tagged loads (mirror probes)", "lts__t_sectors_srcunit_tex_op_read_evict_last_lookup_hit.sum",
            "lts__t_sectors_srcunit_tex_op_read_evict_last_lookup_miss.sum"),
           ("evict_normal-tagged loads (per-task; misses)", "lts__t_sectors_srcunit_tex_op_read_evict_normal_lookup_hit.sum",
            "lts__t_sectors_srcunit_tex_op_read_evict_normal_lookup_miss.sum"),
           ("atomics (W atomicMin, queue AFAs, nibble CAS)", "lts__t_sectors_srcunit_tex_op_atom_dot_alu_lookup_hit.sum",
            "lts__t_sectors_srcunit_tex_op_atom_dot_alu_lookup_miss.sum"),
           ("stores (slots, mirror, markers)", "lts__t_sectors_srcunit_tex_op_write_lookup_hit.sum",
            "lts__t_sectors_srcunit_tex_op_write_lookup_miss.sum")]
    tot_miss = 0.0
    for name, hk, mk in cls:
        h, m = num(hk), num(mk)
        tot_miss += m
        print(f"{name:48s} lookups {h + m:14.0f}  hits {h:14.0f}  misses {m:14.0f}  "
              f"miss bytes {m * 32 / 1e9:7.3f} GB")
    print(f"{'cross-die (ltcfabric) sector lookups':48s} {num('lts__t_sectors_srcunit_ltcfabric.sum'):14.0f}")
    print(f"{'DRAM read / write':48s} {num('dram__bytes_read.sum') / 1e9:8.3f} GB / "
          f"{num('dram__bytes_write.sum') / 1e9:8.3f} GB   (sum of SM-side miss sectors x 32 B: "
          f"{tot_miss * 32 / 1e9:.3f} GB)")


if __name__ == "__main__":
    main(sys.argv[1])
