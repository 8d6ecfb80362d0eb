#!/usr/bin/env python3
"""Summarise an ncu report (raw page) into the handful of numbers the roofline needs."""
import csv
import io
import subprocess
import sys

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
    "lts__t_sector_hit_rate.pct", "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "launch__occupancy_limit_registers", "sm__warps_active.avg.per_cycle_active",
    "smsp__issue_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
    "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "lts__t_sectors_srcunit_tex_op_read.sum",
]


def main(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, u = rows[0], rows[1]
    for v in rows[2:]:
        name = v[h.index("Kernel Name")] if "Kernel Name" in h else "?"
        print(f"kernel: {name[:90]}")
        for k in KEYS:
            if k in h:
                i = h.index(k)
                print(f"  {k:70s} {v[i]:>22s} {u[i]}")
        stalls = []
        for i, n in enumerate(h):
            if n.startswith("smsp__average_warp_latency_issue_stalled_") and n.endswith(".ratio") or \
               (n.startswith("smsp__warp_issue_stalled_") and n.endswith("_per_warp_active.pct")):
                try:
                    stalls.append((float(v[i].replace(",", "")), n))
                except ValueError:
                    pass
        for val, n in sorted(stalls, reverse=True)[:8]:
            print(f"  stall {n:64s} {val:10.2f}")


if __name__ == "__main__":
    main(sys.argv[1])
