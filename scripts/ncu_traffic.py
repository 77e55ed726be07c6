#!/usr/bin/env python
"""DRAM traffic per kernel group of one bench step, from an `ncu --set full` report that captured
every expand / merge / compact launch of one step (scripts/gpu_prof.sh "k_merge|k_compact|k_expand").

  python scripts/ncu_traffic.py gpurun_out/prof_r2_C5.ncu-rep C5 > profiles/r2_traffic_C5.json

bench.py reads profiles/r2_traffic_<config>.json and reports, for the dominant group, the DRAM
bytes (dram__bytes_read.sum + dram__bytes_write.sum, summed over the group's launches of the step)
as roofline.traffic -- the same per-step unit as roofline.achieved's algorithmic bytes.
"""
import csv
import io
import json
import subprocess
import sys

GROUPS = {"expand": ("k_expand",), "merge": ("k_merge", "k_copy_long", "k_long"), "compact": ("k_compact",)}
EXTRA = ["lts__t_bytes.sum", "lts__t_sectors_op_atom.sum", "lts__t_sectors_op_red.sum",
         "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum", "smsp__inst_executed.sum",
         "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum"]


def main(rep, config):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    ki = hdr.index("Kernel Name")
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "B": 1, "KB": 1e3, "MB": 1e6, "GB": 1e9}
    out = {"report": rep, "config": config, "groups": {}, "kernels": [],
           "step": "launches from the first k_pair_work up to (not including) the next one: one bench step"}
    names = [d[ki].split("(")[0] for d in data]
    starts = [q for q, nm in enumerate(names) if nm.split("::")[-1].startswith("k_pair_work")]
    if starts:
        data = data[starts[0]:starts[1]] if len(starts) > 1 else data[starts[0]:]
    for d in data:
        name = d[ki].split("(")[0]
        b = 0.0
        for key in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            i = hdr.index(key)
            b += float(d[i]) * scale[units[i]]
        t = float(d[hdr.index("gpu__time_duration.sum")])
        tu = units[hdr.index("gpu__time_duration.sum")]
        ms = t * {"s": 1e3, "second": 1e3, "ms": 1.0, "msecond": 1.0, "us": 1e-3, "usecond": 1e-3}.get(tu, 1e-6)
        rec = {"kernel": name, "dram_bytes": int(b), "ms": ms}
        for key in EXTRA:
            if key in hdr:
                i = hdr.index(key)
                try:
                    rec[key] = float(d[i].replace(",", "")) * scale.get(units[i], 1)
                except ValueError:
                    pass
        for key in ("sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread"):
            if key in hdr:
                try:
                    rec[key] = float(d[hdr.index(key)].replace(",", ""))
                except ValueError:
                    pass
        out["kernels"].append(rec)
        for g, pre in GROUPS.items():
            base = name.split("<")[0].split()[-1].split("::")[-1]
            if any(base.startswith(p) for p in pre):
                e = out["groups"].setdefault(g, {"dram_bytes": 0, "ms": 0.0, "launches": 0})
                e["dram_bytes"] += int(b)
                e["ms"] += ms
                e["launches"] += 1
                for key in EXTRA:
                    if key in rec:
                        e[key] = e.get(key, 0.0) + rec[key]
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
