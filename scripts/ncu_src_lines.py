#!/usr/bin/env python
"""Per-CUDA-line totals from an ncu report's mixed source+SASS page (ncu 2025 layout: CUDA line
rows "Line No","Source" followed by the SASS rows of that line): warp instructions, stall samples,
thread instructions (predicated-on), shared wavefronts.

  python scripts/ncu_src_lines.py gpurun_out/prof.ncu-rep <kernel-regex> [top] [launch-skip]
"""
import csv
import io
import subprocess
import sys


def main(rep, regex, top=40, skip=0):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                          "-k", f"regex:{regex}", "-s", str(skip), "-c", "1"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = None
    cur = None
    path = None
    agg = {}
    for r in rows:
        if not r:
            continue
        if r[0] == "File Path":
            path = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None:
            continue
        if r[0].isdigit():
            cur = (path, int(r[0]), r[1].strip())
            continue
        if len(r) > 4 and r[2].startswith("0x"):
            num = lambda i: int(r[i]) if r[i].strip().isdigit() else 0
            ii = hdr.index("Instructions Executed")
            wi = hdr.index("Warp Stall Sampling (All Samples)")
            ti = hdr.index("Predicated-On Thread Instructions Executed")
            a = agg.setdefault(cur, [0, 0, 0])
            a[0] += num(ii); a[1] += num(wi); a[2] += num(ti)
    tot_i = sum(v[0] for v in agg.values()) or 1
    tot_w = sum(v[1] for v in agg.values()) or 1
    tot_t = sum(v[2] for v in agg.values()) or 1
    print(f"warp instr {tot_i:.4g}  stall samples {tot_w}  thread instr {tot_t:.4g} (avg active {tot_t / tot_i:.1f})")
    for k, v in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
        if k is None:
            continue
        print(f"{100 * v[0] / tot_i:5.1f}% inst {100 * v[1] / tot_w:5.1f}% samp act {v[2] / max(v[0], 1):4.1f} "
              f"{k[0]}:{k[1]}  {k[2][:80]}")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], int(sys.argv[3]) if len(sys.argv) > 3 else 40,
         int(sys.argv[4]) if len(sys.argv) > 4 else 0)
