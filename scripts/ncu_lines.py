#!/usr/bin/env python
"""Per-source-line warp instructions and stall samples of one kernel in an ncu report (needs
-lineinfo): the hottest CUDA lines with their share of the kernel's instructions.

  python scripts/ncu_lines.py gpurun_out/prof.ncu-rep <kernel-regex>:<launch-index> [top]
"""
import csv
import io
import subprocess
import sys


def main(rep, kid, top=30):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                          "--kernel-id", f"::regex:{kid}"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    recs, path, hdr = [], None, None
    for r in rows:
        if not r:
            continue
        if r[0] == "File Path":
            path = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr and r[0].isdigit():
            ii = hdr.index("Instructions Executed")
            wi = hdr.index("Warp Stall Sampling (All Samples)")
            num = lambda x: int(x) if x.strip().isdigit() else 0
            n, w = num(r[ii]), num(r[wi])
            if n or w:
                recs.append((path, int(r[0]), r[1].strip(), n, w))
    ti = sum(x[3] for x in recs) or 1
    tw = sum(x[4] for x in recs) or 1
    print(f"warp instructions {ti}, stall samples {tw}")
    for p, ln, src, n, w in sorted(recs, key=lambda x: -x[3])[:top]:
        print(f"{100 * n / ti:5.1f}% inst {100 * w / tw:5.1f}% samp  {p}:{ln}  {src[:90]}")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], int(sys.argv[3]) if len(sys.argv) > 3 else 30)
