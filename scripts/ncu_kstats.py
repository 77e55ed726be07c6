#!/usr/bin/env python
"""Per-kernel key counters of an ncu --set full report (issue, smem wavefronts, stalls).

  python scripts/ncu_kstats.py gpurun_out/prof.ncu-rep
"""
import csv
import io
import subprocess
import sys

WANT = ["gpu__time_duration.sum", "smsp__inst_executed.sum", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "smsp__thread_inst_executed_per_inst_executed.ratio",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "launch__registers_per_thread", "launch__occupancy_limit_shared_mem", "launch__grid_size", "launch__block_size"]


def main(rep):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, data = rows[0], rows[2:]
    ki = h.index("Kernel Name")
    for d in data:
        print("==", d[ki][:70])
        for w in WANT:
            if w in h:
                print(f"   {w:75s} {d[h.index(w)]}")
        st = {}
        for i, x in enumerate(h):
            if x.startswith("smsp__pcsamp_warps_issue_stalled_") and not x.endswith("not_issued"):
                try:
                    st[x[33:]] = float(d[i])
                except ValueError:
                    pass
        tot = sum(st.values()) or 1
        print("   stalls:", ", ".join(f"{k} {100 * v / tot:.0f}%" for k, v in sorted(st.items(), key=lambda x: -x[1])[:7]))


if __name__ == "__main__":
    main(sys.argv[1])
