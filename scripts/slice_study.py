#!/usr/bin/env python
"""Multi-GPU readiness study on one B200 (the 8-GPU box is not reachable from the builder's
sandbox): for N = 1, 2, 4, 8, the balanced row partition of C (spgemm_row_partition, R8)
is computed once and EVERY rank's row block is run alone on this GPU (spgemm_plan_rows: the window
is cut on the GPU), device-timed plan + execute + destroy, median of --reps.  The projected N-GPU
step is the max over the ranks (no data-path collective: the row blocks are independent).

  python scripts/slice_study.py C5 [--reps 3] > gpurun_out/slices_C5.jsonl
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


def timed(A, B, rows, reps, flush, opts):
    ts = []
    st = None
    for q in range(reps + 1):
        flush.add_(1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        p = spg.Plan(A, B, rows=rows, validate=0, **opts)
        C = p.execute()
        st = p.stats()
        p.destroy()
        e1.record()
        e1.synchronize()
        if q:
            ts.append(e0.elapsed_time(e1))
        del C
    return statistics.median(ts), st


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--parts", default="1,2,4,8")
    ap.add_argument("--opt", action="append", default=[])
    args = ap.parse_args()
    opts = {}
    for kv in args.opt:
        k, v = kv.split("=")
        opts[k] = float(v) if k in ("alpha", "beta") else int(v)
    if os.environ.get("SPGEMM_RESERVED"):   # tuning knobs, as bench.py: "index=value,..."
        res = [0] * 16
        for kv in os.environ["SPGEMM_RESERVED"].split(","):
            q, v = kv.split("=")
            res[int(q)] = int(v)
        opts["reserved"] = tuple(res)
    inp = synth.make_inputs(args.config)
    A, B = spg.from_inputs(inp, "cuda")
    flush = torch.zeros(512 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    t1 = None
    for N in [int(x) for x in args.parts.split(",")]:
        bounds = spg.row_partition(A, B, N)
        per = []
        for r in range(N):
            ms, st = timed(A, B, (int(bounds[r]), int(bounds[r + 1])), args.reps, flush, opts)
            per.append({"rank": r, "rows": int(bounds[r + 1] - bounds[r]), "products": st["nnz_chat"],
                        "limited_rows": st["n_rows_bin"][5], "ms": round(ms, 3)})
            torch.cuda.empty_cache()
        mx = max(x["ms"] for x in per)
        mean = statistics.mean(x["ms"] for x in per)
        if N == 1:
            t1 = mx
        print(json.dumps({"config": args.config, "parts": N, "max_ms": round(mx, 3), "mean_ms": round(mean, 3),
                          "imbalance": round(mx / mean, 3), "speedup_vs_1": round(t1 / mx, 3) if t1 else None,
                          "ranks": per, "options": opts}), flush=True)


if __name__ == "__main__":
    main()
