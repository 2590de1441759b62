#!/usr/bin/env python
"""Summarise an ncu report (--set full) into a small text file for profiles/.

    python scripts/ncu_summary.py gpurun_out/X.ncu-rep > profiles/X.txt

Prints, per profiled kernel: duration, registers, occupancy, issue/pipe
utilisation, L1/L2/DRAM counters of the surplus gathers and the top stall
reasons -- the numbers DESIGN.md's roofline discussion cites.
"""
import csv
import subprocess
import sys

KEYS = [
    "Kernel Name", "Block Size", "Grid Size", "launch__registers_per_thread", "gpu__time_duration.sum",
    "sm__cycles_elapsed.avg.per_second", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "smsp__inst_executed.sum", "sm__inst_executed.avg.per_cycle_active",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
    "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
    "l1tex__t_sector_pipe_lsu_mem_global_op_ld_hit_rate.pct", "l1tex__data_pipe_lsu_wavefronts_mem_lgds.sum",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
    "lts__t_sectors_srcunit_tex_op_read.sum", "lts__t_sector_hit_rate.pct", "dram__bytes_read.sum",
    "dram__bytes_write.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
]


def main(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr, units = rows[0], rows[1]
    for r in rows[2:]:
        rec = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        print("=" * 100)
        for k in KEYS:
            if k in rec:
                print(f"{k:70s} {rec[k]:>24s} {u.get(k, '')}")
        stalls = {k: float(v) for k, v in rec.items()
                  if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")
                  and v.replace(".", "").isdigit()}
        tot = sum(stalls.values()) or 1.0
        print("top stall reasons (pc sampling):")
        for k, v in sorted(stalls.items(), key=lambda kv: -kv[1])[:8]:
            print(f"  {k.replace('smsp__pcsamp_warps_issue_stalled_', ''):40s} {100 * v / tot:6.1f} %")


if __name__ == "__main__":
    main(sys.argv[1])
