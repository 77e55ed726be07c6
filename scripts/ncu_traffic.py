#!/usr/bin/env python
"""DRAM traffic per kernel group of one bench step, from an `ncu --set full` report that captured
every expand / merge / compact launch of one step (scripts/gpu_prof.sh "k_merge|k_compact|k_expand").

  python scripts/ncu_traffic.py gpurun_out/prof_v8.ncu-rep C2 > profiles/r1_traffic_C2.json

bench.py reads profiles/r1_traffic_<config>.json and reports, for the dominant group, the DRAM
bytes (dram__bytes_read.sum + dram__bytes_write.sum, summed over the group's launches of the step)
as roofline.traffic -- the same per-step unit as roofline.achieved's algorithmic bytes.
"""
import csv
import io
import json
import subprocess
import sys

GROUPS = {"expand": ("k_expand",), "merge": ("k_merge", "k_copy_long"), "compact": ("k_compact",)}


def main(rep, config):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    ki = hdr.index("Kernel Name")
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "B": 1, "KB": 1e3, "MB": 1e6, "GB": 1e9}
    out = {"report": rep, "config": config, "groups": {}, "kernels": []}
    for d in data:
        name = d[ki].split("(")[0]
        b = 0.0
        for key in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            i = hdr.index(key)
            b += float(d[i]) * scale[units[i]]
        t = float(d[hdr.index("gpu__time_duration.sum")])
        tu = units[hdr.index("gpu__time_duration.sum")]
        ms = t * {"s": 1e3, "second": 1e3, "ms": 1.0, "msecond": 1.0, "us": 1e-3, "usecond": 1e-3}.get(tu, 1e-6)
        out["kernels"].append({"kernel": name, "dram_bytes": int(b), "ms": ms})
        for g, pre in GROUPS.items():
            if any(name.split("<")[0].split()[-1].startswith(p) for p in pre):
                e = out["groups"].setdefault(g, {"dram_bytes": 0, "ms": 0.0, "launches": 0})
                e["dram_bytes"] += int(b)
                e["ms"] += ms
                e["launches"] += 1
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
