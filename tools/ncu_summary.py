#!/usr/bin/env python
"""Summarise ncu reports: key throughput/latency metrics and top stall reasons."""
import csv
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "launch__registers_per_thread", "launch__occupancy_limit_shared_mem",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum",
        "lts__t_sectors_srcunit_tex_op_read.sum", "lts__t_sectors_srcunit_tex_op_write.sum",
        "l1tex__throughput.avg.pct_of_peak_sustained_active",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "launch__grid_size", "launch__block_size", "sm__cycles_elapsed.avg.per_second",
        "dram__cycles_elapsed.avg.per_second"]


def main():
    for f in sys.argv[1:]:
        out = subprocess.run(["ncu", "-i", f, "--page", "raw", "--csv"], capture_output=True,
                             text=True).stdout
        rows = list(csv.reader(out.splitlines()))
        hdr, units = rows[0], rows[1]
        for r in rows[2:]:
            d = dict(zip(hdr, r))
            print(f"== {f}: {d.get('Kernel Name', '')[:80]}")
            for k in KEYS:
                if k in d:
                    print(f"  {k:70s} {d[k]} {units[hdr.index(k)]}")
            for k in ("smsp__issue_active.avg.pct_of_peak_sustained_active",
                      "dram__throughput.avg.pct_of_peak_sustained_elapsed"):
                if k in d:
                    print(f"  {k:70s} {d[k]} {units[hdr.index(k)]}")
            # warps stalled per issued instruction, by reason (the top 8)
            stalls = []
            for k in hdr:
                if (k.startswith("smsp__average_warps_issue_stalled_")
                        and k.endswith("_per_issue_active.ratio")):
                    try:
                        stalls.append((float(d[k]), k[len("smsp__average_warps_issue_stalled_"):
                                                      -len("_per_issue_active.ratio")]))
                    except ValueError:
                        pass
            stalls.sort(reverse=True)
            for v, k in stalls[:8]:
                print(f"  stall {k:40s} {v:.2f} warps per issue")


if __name__ == "__main__":
    main()
