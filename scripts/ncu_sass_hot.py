#!/usr/bin/env python
"""Hot SASS of one kernel in an ncu report: instructions executed and stall samples per
instruction, printed in address order for the hottest regions.

  python scripts/ncu_sass_hot.py gpurun_out/prof.ncu-rep <kernel-regex>:<launch-index> [min_share]
"""
import csv
import io
import subprocess
import sys


def main(rep, regex, min_share=0.002):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass",
                          "--kernel-id", f"::regex:{regex}"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = rows[1]
    ai, si = hdr.index("Address"), hdr.index("Source")
    ii = hdr.index("Instructions Executed")
    wi = hdr.index("Warp Stall Sampling (All Samples)")
    num = lambda x: int(x) if x.strip().isdigit() else 0
    data = [(r[ai], r[si].strip(), num(r[ii]), num(r[wi])) for r in rows[2:] if len(r) > max(ii, wi)]
    ti = sum(d[2] for d in data) or 1
    tw = sum(d[3] for d in data) or 1
    print(f"total warp instr {ti}, stall samples {tw}")
    for q, (a, s, n, w) in enumerate(data):
        if n / ti >= min_share or w / tw >= min_share:
            print(f"{q:5d} {100 * n / ti:5.1f}% inst {100 * w / tw:5.1f}% samp  {s}")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], float(sys.argv[3]) if len(sys.argv) > 3 else 0.002)
