#!/usr/bin/env python
"""Fig. 11 / Fig. 14 sweeps on B200 (PAPER.md L640-L687 L, L778-L790 L): for one config, the
expansion time and its load balancing index (LBI, Eq. (3), L564-L577 R) per B-Splitting factor
(options.reserved[7], 0 = the B200 default rule, 'off' = enable_split 0), and the B-Limited merge
time + LBI per limit_ctas_per_sm.  One JSON line per point (tooling; run under gpurun).

  python scripts/sweep_fig11.py C3 [--reps 3] > gpurun_out/fig11_C3.jsonl
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_icde_leekyjkp20_b200 as spg  # noqa: E402


def run(A, B, reps, **opts):
    res = list(opts.pop("reserved", (0,) * 16))
    res[8] = 1
    times, lbis = {}, []
    for _ in range(reps + 1):
        spg.set_timing(True)
        with spg.Plan(A, B, validate=0, reserved=tuple(res), **opts) as p:
            C = p.execute()
            torch.cuda.synchronize()
            lb = p.lbi()
            st = p.stats()
        tl = spg.last_timings()
        spg.set_timing(False)
        del C
        t = {}
        for nm, ms in tl:
            t[nm] = t.get(nm, 0.0) + ms
        for nm, ms in t.items():
            times.setdefault(nm, []).append(ms)
        lbis.append(lb)
    med = {nm: statistics.median(v[1:]) for nm, v in times.items()}
    lb = lbis[-1]
    return {"expand_ms": round(med.get("expand", 0.0) + med.get("expand_blocks", 0.0), 4),
            "long_partition_ms": round(med.get("merge_long_partition", 0.0), 4),
            "tiles_ms": round(med.get("merge_tiles", 0.0), 4),
            "merge_limited_ms": round(sum(v for k, v in med.items() if k.startswith("merge_limited")), 4),
            "step_kernels_ms": round(sum(med.values()), 4),
            "lbi_expand": lb["expand"] and round(lb["expand"]["lbi"], 4),
            "lbi_merge_limited": lb["merge_limited"] and round(lb["merge_limited"]["lbi"], 4),
            "n_dominator": st["n_dominator"], "n_pieces_split": st["n_pieces_split"]}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--only", choices=["split", "limit"], default=None)
    args = ap.parse_args()
    inp = synth.make_inputs(args.config)
    A, B = spg.from_inputs(inp, "cuda")
    for f in (["off", 0, 1, 2, 4, 8, 16, 32, 64] if args.only != "limit" else []):
        if f == "off":
            r = run(A, B, args.reps, enable_split=0)
        else:
            r = run(A, B, args.reps, reserved=(0,) * 7 + (f,) + (0,) * 8)
        print(json.dumps({"sweep": "splitting_factor", "config": args.config, "factor": f, **r}), flush=True)
    if args.only == "split":
        return
    for cap in [1, 2, 4]:   # B-Limiting: limited blocks of 1024 / 512 / 256 threads per SM (Fig. 14)
        r = run(A, B, args.reps, limit_ctas_per_sm=cap)
        print(json.dumps({"sweep": "limit_ctas_per_sm", "config": args.config, "cap": cap, **r}), flush=True)
    if args.only == "limit":
        return
    tiles = (0,) * 5 + (2,) + (0,) * 10   # tile merge: the long-row partition kernel's residency
    for cap in [1, 2]:
        r = run(A, B, args.reps, limit_ctas_per_sm=cap, reserved=tiles)
        print(json.dumps({"sweep": "limit_ctas_per_sm (tile merge)", "config": args.config, "cap": cap, **r}),
              flush=True)
    for beta in [10.0, 0.0]:
        r = run(A, B, args.reps, beta=beta)
        print(json.dumps({"sweep": "beta", "config": args.config, "beta": beta, **r}), flush=True)


if __name__ == "__main__":
    main()
