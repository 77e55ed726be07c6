#!/usr/bin/env python
"""Benchmark: outer-product spGEMM C = A x A with the Block Reorganizer on B200.

One *step* = one pass of the whole hot path over the workload: spgemm_plan (workload
analysis + Block Reorganizer lists) + spgemm_execute (expansion, merge, C allocation and CSR
compaction) + spgemm_destroy, through the C-ABI.  Inputs are resident in HBM when the timed
region starts.  Metric (BASELINE.json): GFLOPS = 2 x intermediate products / s; the HBM
roofline fraction of the dominant kernel and of the whole step are reported beside it.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C5] [--impl ours|reference]
Default workload: C5 (BASELINE.json configs[4], the metric's 1/2/4/8-GPU config; it fits one B200).
Multi-GPU: one rank per GPU over NCCL (torch.distributed.run; `--gpus N` without WORLD_SIZE in the
environment re-launches itself that way).  Rank 0 generates the input, computes the balanced
row-block partition of C on its GPU, broadcasts B and sends every rank its row slice of A (NCCL,
dist.py); each rank runs the whole path on its block (strong scaling of one product).  value = all
products / max-over-ranks device time; the C row-block gather to rank 0 is timed on its own
(`c_gather`), outside the step.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "spGEMM GFLOPS (2*intermediate products/s), C=AxA"
UNIT = "GFLOPS"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C5")
    ap.add_argument("--seed", type=int, default=1)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--slice", default=None,
                    help="N:r -- run only rank r's row block of an N-way partition on this GPU (scaling study)")
    ap.add_argument("--opt", action="append", default=[],
                    help="spgemm option key=value (e.g. enable_split=0: the Fig. 10 ablations)")
    return ap.parse_args()


# ------------------------------------------------------------------ clocks -------------------
class ClockSampler:
    """SM clock, max clock and throttle reasons sampled DURING the timed region: NVML polled every
    ~2 ms from a thread (the timed region of a C2 run is ~60 ms); nvidia-smi as a fallback."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.nvml = None
        self.lines = []
        self.samples = []
        self.stop_flag = threading.Event()

    def start(self):
        try:
            import pynvml as nv
            nv.nvmlInit()
            h = nv.nvmlDeviceGetHandleByIndex(self.index)
            self.nvml = (nv, h)
            bits = [nv.nvmlClocksEventReasonHwSlowdown, nv.nvmlClocksEventReasonHwThermalSlowdown,
                    nv.nvmlClocksEventReasonSwThermalSlowdown, nv.nvmlClocksEventReasonSwPowerCap]
            mx = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)

            def poll():
                while not self.stop_flag.is_set():
                    try:
                        sm = nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)
                        r = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                        self.samples.append((sm, mx, [n for n, b in zip(self.NAMES, bits) if r & b]))
                    except Exception:
                        pass
                    time.sleep(0.002)
            self.t = threading.Thread(target=poll, daemon=True)
            self.t.start()
            return
        except Exception:
            self.nvml = None
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "10"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.nvml is not None:
            self.stop_flag.set()
            self.t.join(timeout=1)
            sm = [x[0] for x in self.samples]
            reasons = sorted({r for x in self.samples for r in x[2]})
            return {"sm_mhz": statistics.median(sm) if sm else None,
                    "sm_max_mhz": max(x[1] for x in self.samples) if self.samples else None,
                    "reasons": reasons, "samples": len(sm), "source": "nvml"}
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm, mx, reasons = [], [], set()
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 6:
                continue
            try:
                sm.append(float(f[0]))
                mx.append(float(f[1]))
            except ValueError:
                continue
            for nm, v in zip(self.NAMES, f[2:6]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm), "source": "nvidia-smi"}


# ------------------------------------------------------------------ CPU oracle timing ------
def time_oracle(inp, target_s: float, seed: int = 0):
    """The oracle as it stands (fp64 Gustavson, OpenMP) on a bounded random row sample."""
    import oracle
    from oracle import stages
    rowwork = stages.row_workload(inp)   # only to report products of the sample
    rng = np.random.default_rng(seed)
    perm = rng.permutation(inp.m).astype(np.int32)
    cores = oracle.max_threads()
    n = max(1, inp.m // 1000)
    while True:
        rows = np.sort(perm[:n])
        t0 = time.perf_counter()
        oracle.gustavson(inp, rows=rows)
        dt = time.perf_counter() - t0
        if dt >= target_s or n >= inp.m:
            break
        n = min(inp.m, int(n * min(8.0, max(1.5, 1.2 * target_s / max(dt, 1e-3)))))
    prods = int(rowwork[rows].sum())
    return {"value": 2.0 * prods / dt / 1e9, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"{rows.size} random rows of {inp.m} ({prods} products, {dt:.1f} s)"}, dt


# ------------------------------------------------------------------ helpers ----------------
def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def relaunch(args) -> int:
    """`bench.py --gpus N` outside torch.distributed: run N ranks (one per GPU) under
    torch.distributed.run on 127.0.0.1 with the same arguments; rank 0 prints the line."""
    import socket
    sck = socket.socket()
    sck.bind(("127.0.0.1", 0))
    port = sck.getsockname()[1]
    sck.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def flush_l2(buf):
    buf.add_(1)  # write 512 MiB (> 126 MB L2) between timed steps


def main():
    args = parse()
    if args.impl == "reference":
        ws, rank, _ = dist_env()
        return run_reference(args, ws, rank)
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        sys.exit(relaunch(args))
    ws, rank, local = dist_env()
    if "WORLD_SIZE" in os.environ and ws != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={ws} (launch one rank per GPU)")
    import torch
    import synth
    import paper_conf_icde_leekyjkp20_b200 as spg
    from paper_conf_icde_leekyjkp20_b200 import dist as pdist
    from paper_conf_icde_leekyjkp20_b200.build import build_library
    if rank == 0:
        build_library()
    share = bool(os.environ.get("SPGEMM_BENCH_SHARE_GPU"))   # test mode: N ranks share the visible GPUs (gloo)
    if share:
        local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist = None
    if ws > 1:
        import torch.distributed as dist
        if share:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)
        if rank == 0:
            build_library()
        dist.barrier()
    comm_dev = torch.device("cpu") if share else dev
    inp_full = None
    if rank == 0 or ws == 1:
        inp_full = synth.make_inputs(args.config, seed=args.seed)
    if ws > 1:
        # rank 0: input, partition; NCCL: B broadcast, A row-slice scatter (input movement, untimed)
        t_dist = time.perf_counter()
        if rank == 0:
            A_full, B_full = spg.from_inputs(inp_full, dev)
            bounds = torch.from_numpy(spg.row_partition(A_full, B_full, ws)).to(comm_dev)
            A_src = spg.CSC(A_full.nrows, A_full.ncols, A_full.colptr.to(comm_dev), A_full.rowidx.to(comm_dev),
                            A_full.val.to(comm_dev))
            B_src = spg.CSR(B_full.nrows, B_full.ncols, B_full.rowptr.to(comm_dev), B_full.colidx.to(comm_dev),
                            B_full.val.to(comm_dev))
        else:
            bounds = torch.zeros(ws + 1, dtype=torch.int64, device=comm_dev)
            A_src = B_src = None
        dist.broadcast(bounds, src=0)
        B = pdist.broadcast_csr(B_src, src=0, device=comm_dev)
        A = pdist.scatter_row_slices(A_src, bounds.tolist(), src=0, device=comm_dev)
        A = spg.CSC(A.nrows, A.ncols, A.colptr.to(dev), A.rowidx.to(dev), A.val.to(dev))
        B = spg.CSR(B.nrows, B.ncols, B.rowptr.to(dev), B.colidx.to(dev), B.val.to(dev))
        if rank == 0:
            del A_full, B_full, A_src, B_src
        torch.cuda.synchronize()
        dist.barrier()
        dist_s = time.perf_counter() - t_dist
        bounds = bounds.tolist()
        inp = synth.SparseInputs(f"{args.config}[{bounds[rank]}:{bounds[rank + 1]}]", A.nrows, A.ncols, B.ncols,
                                 A.colptr.cpu().numpy(), A.rowidx.cpu().numpy(), A.val.cpu().numpy(),
                                 B.rowptr.cpu().numpy(), B.colidx.cpu().numpy(), B.val.cpu().numpy())
    else:
        dist_s, bounds = 0.0, None
        A_full, B_full = spg.from_inputs(inp_full, dev)
        if args.slice:   # scaling study: rank r's row block of an N-way partition, alone on this GPU
            nparts, part = (int(x) for x in args.slice.split(":"))
            bounds = spg.row_partition(A_full, B_full, nparts)
            A = pdist.csc_row_slice(A_full, int(bounds[part]), int(bounds[part + 1]))
            B = B_full
            inp = synth.SparseInputs(f"{args.config}[{bounds[part]}:{bounds[part + 1]}]", A.nrows, A.ncols, B.ncols,
                                     A.colptr.cpu().numpy(), A.rowidx.cpu().numpy(), A.val.cpu().numpy(),
                                     inp_full.b_rowptr, inp_full.b_colidx, inp_full.b_val)
        else:
            inp, A, B = inp_full, A_full, B_full
    stream = torch.cuda.current_stream(dev)
    opts = dict(validate=0)
    for kv in args.opt:
        k, v = kv.split("=")
        opts[k] = float(v) if k in ("alpha", "beta") else int(v)
    if os.environ.get("SPGEMM_RESERVED"):   # tuning knobs: "index=value,..."
        res = [0] * 16
        for kv in os.environ["SPGEMM_RESERVED"].split(","):
            q, v = kv.split("=")
            res[int(q)] = int(v)
        opts["reserved"] = tuple(res)
    flush = torch.zeros(512 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)

    def step():
        with spg.Plan(A, B, stream=stream, **opts) as p:
            C = p.execute()
            return p, C

    # The headline steps run with per-launch event timing off (two event records per launch are
    # host time that would stretch host-bound steps); the kernel breakdown comes from as many
    # extra, untimed-for-the-headline steps with timing on.
    spg.set_timing(False)
    for _ in range(max(args.warmup, 0)):
        p, C = step()
        del C
    torch.cuda.synchronize()
    st = None
    # timed region
    sampler = ClockSampler(local)
    sampler.start()
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()
    step_ms, kern = [], {}
    launches = 0
    nnz_c = 0
    wall0 = time.perf_counter()
    for _ in range(args.steps):
        flush_l2(flush)
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        p = spg.Plan(A, B, stream=stream, **opts)
        C = p.execute()
        st = p.stats()
        if "1=2" in os.environ.get("SPGEMM_RESERVED", "") or "1=3" in os.environ.get("SPGEMM_RESERVED", ""):
            prof = p.inspect(spg.VIEW_UNIT_PROFILE, np.uint64)
            print("unit-profile", json.dumps([int(x) for x in prof]), file=sys.stderr)
        p.destroy()
        e1.record(stream)
        e1.synchronize()
        step_ms.append(e0.elapsed_time(e1))
        nnz_c = C.nnz
        del C
    torch.cuda.synchronize()
    if ws > 1:
        dist.barrier()
    wall = time.perf_counter() - wall0
    clocks = sampler.stop()
    # kernel breakdown (CUDA events around every launch, on the launch stream)
    spg.set_timing(True)
    for _ in range(args.steps):
        flush_l2(flush)
        p = spg.Plan(A, B, stream=stream, **opts)
        C = p.execute()
        p.destroy()
        torch.cuda.synchronize()
        tl = spg.last_timings()
        launches += len(tl)
        for nm, ms in tl:
            kern.setdefault(nm, []).append(ms)
        del C
    spg.set_timing(False)
    total_ms = float(sum(step_ms))
    products = st["nnz_chat"]
    # max over ranks of the device time; total products over ranks
    rank_ms = [round(total_ms / args.steps, 4)]
    if ws > 1:
        t = torch.tensor([total_ms, float(products), float(nnz_c), float(launches), float(inp.nnz_a)],
                         dtype=torch.float64, device=comm_dev)
        tmax = t.clone()
        dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
        tsum = t.clone()
        dist.all_reduce(tsum, op=dist.ReduceOp.SUM)
        total_ms_all = float(tmax[0])
        products_all = int(tsum[1])
        nnz_c_all = int(tsum[2])
        launches_all = int(tsum[3])
        nnz_a_all = int(tsum[4])
        every = [torch.zeros(1, dtype=torch.float64, device=comm_dev) for _ in range(ws)]
        dist.all_gather(every, t[:1].clone())
        rank_ms = [round(float(x) / args.steps, 4) for x in every]
        m_all = int(bounds[-1])
    else:
        total_ms_all, products_all, nnz_c_all, launches_all = total_ms, products, nnz_c, launches
        nnz_a_all, m_all = inp.nnz_a, inp.m
    ms_per_step = total_ms_all / args.steps
    value = 2.0 * products_all / (ms_per_step / 1e3) / 1e9

    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    hbm = peaks.get("hbm_gbs", 6650.0)
    peak_src = "measured" if "hbm_gbs" in peaks else "fallback"

    # per-kernel shares; algorithmic bytes
    k_ms = {nm: sum(v) / args.steps for nm, v in kern.items()}
    nnz_a, nnz_b = inp.nnz_a, inp.nnz_b
    bytes_step = 12 * nnz_a + 12 * nnz_b + 16 * (inp.m + 1 + inp.k + 1) // 2 + 16 * products + 12 * nnz_c + 8 * (inp.m + 1)
    groups = {
        "expand": ("expand_", 8 * products + 12 * nnz_a + 8 * nnz_b),
        "merge": ("merge_", 8 * products + 8 * nnz_c + 16 * inp.m),
        "compact": ("compact", 16 * nnz_c + 8 * inp.m),   # (legacy bin merge only)
    }
    gms = {g: sum(v for n, v in k_ms.items() if n.startswith(pre)) for g, (pre, _) in groups.items()}
    top = max(gms, key=lambda g: gms[g])
    top_bytes = groups[top][1]
    achieved = top_bytes / (gms[top] / 1e3) / 1e9 if gms[top] > 0 else 0.0
    # DRAM bytes of the same kernel group per step, from the committed ncu --set full capture
    # (scripts/ncu_traffic.py); null when no capture of this config exists
    traffic, traffic_src = None, None
    tpath = os.path.join(ROOT, "profiles", f"r2_traffic_{args.config}.json")
    if os.path.exists(tpath) and ws == 1 and not args.slice and not args.opt:
        try:
            tj = json.load(open(tpath))
            traffic = tj["groups"][top]["dram_bytes"]
            traffic_src = os.path.relpath(tpath, ROOT) + " <- " + tj["report"]
        except (KeyError, ValueError):
            pass
    roofline = {"bound": "hbm", "kernel": top, "achieved": round(achieved, 1), "peak": hbm, "unit": "GB/s",
                "frac": round(achieved / hbm, 4), "traffic": traffic, "traffic_src": traffic_src,
                "peak_source": peak_src, "ms": round(gms[top], 4), "algorithmic_bytes": int(top_bytes)}
    step_bw = bytes_step / (ms_per_step / 1e3) / 1e9
    breakdown = {nm: round(v, 4) for nm, v in sorted(k_ms.items(), key=lambda x: -x[1])}

    out = {
        "metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": ws, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(ms_per_step, 4), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f32 (fp64 merge accumulation)",
        "data": "synthetic (seeded generator, synth/)",
        "config": {"workload": f"{args.config}: " + synth.CONFIGS[args.config]["desc"], "m": m_all,
                   "nnz_a": nnz_a_all, "products": products_all, "nnz_c": nnz_c_all,
                   "parallelism": f"row-partition x{ws}" if ws > 1 else "single GPU",
                   "l2": "flushed between steps (512 MiB write); Ĉ >> L2", "seed": args.seed,
                   "step": "plan+execute+destroy via C-ABI, device-resident inputs",
                   **({"options": {k: v for k, v in opts.items() if k != "validate"}} if len(opts) > 1 else {})},
        "roofline": roofline,
        "step_roofline": {"achieved": round(step_bw, 1), "peak": hbm, "unit": "GB/s",
                          "frac": round(step_bw / hbm, 4), "bytes": int(bytes_step),
                          "def": "A + B + 2*Ĉ(8 B/product) + C, per step"},
        "kernel_ms": breakdown,
        "gpu_launches": launches_all,
        "rank_ms_per_step": rank_ms,
        "clocks": clocks,
        "wall_s": round(wall, 3),
    }
    if ws > 1:
        # C row-block gather to rank 0 (NCCL point-to-point into one CSR, no concatenation copy):
        # output movement, timed on its own
        p = spg.Plan(A, B, stream=stream, **opts)
        C = p.execute()
        p.destroy()
        Cc = C if not share else spg.CSR(C.nrows, C.ncols, C.rowptr.cpu(), C.colidx.cpu(), C.val.cpu())
        torch.cuda.synchronize()
        dist.barrier()
        g0 = time.perf_counter()
        G = pdist.gather_row_blocks(Cc, dst=0)
        torch.cuda.synchronize()
        g_s = time.perf_counter() - g0
        gb = torch.tensor([g_s], dtype=torch.float64, device=comm_dev)
        dist.all_reduce(gb, op=dist.ReduceOp.MAX)
        out["c_gather"] = {"ms": round(float(gb[0]) * 1e3, 3), "bytes": int(nnz_c_all * 8 + (m_all + 1) * 8),
                           "to": "rank 0", "how": "NCCL send/recv into one CSR; synchronised wall time, max over ranks",
                           "input_distribution_s": round(dist_s, 3)}
        if rank == 0:
            assert G.nnz == nnz_c_all and G.nrows == m_all
        del C, Cc, G
    # e2e through the C-ABI with host buffers (H2D of A, B and D2H of C inside the timed region)
    if not args.no_e2e:
        # (the device-output steps' C arrays and plan workspaces stay cached by torch / the plan pool:
        # a host-output product of C5 needs Ĉ plus a device staging copy of C, so release them first)
        torch.cuda.synchronize()
        torch.cuda.empty_cache()
        spg.trim_pool()
        Ah, Bh = spg.from_inputs(inp, "cpu")
        h2d = sum(t.numel() * t.element_size() for t in (Ah.colptr, Ah.rowidx, Ah.val, Bh.rowptr, Bh.colidx, Bh.val))
        es = []
        d2h = 0
        pool = spg.HostBufferPool()
        for it in range(1 + max(1, args.steps // 2)):
            flush_l2(flush)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            with spg.Plan(Ah, Bh, stream=stream, **opts) as p:
                Ch = p.execute(device="cpu", pool=pool)
            torch.cuda.synchronize()
            dt = time.perf_counter() - t0
            d2h = sum(t.numel() * t.element_size() for t in (Ch.rowptr, Ch.colidx, Ch.val))
            if it > 0:
                es.append(dt)
        e2e_t = sum(es) / len(es)
        if ws > 1:
            tt = torch.tensor([e2e_t], dtype=torch.float64, device=comm_dev)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            e2e_t = float(tt[0])
        out["e2e"] = {"value": round(2.0 * products_all / e2e_t / 1e9, 3), "unit": UNIT,
                      "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
                      "ms_per_step": round(e2e_t * 1e3, 3)}
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        cb, _ = time_oracle(inp_full, target_s=10.0)
        out["cpu_baseline"] = cb
    if rank == 0:
        print(json.dumps(out), flush=True)
    if ws > 1:
        dist.barrier()
        dist.destroy_process_group()


def run_reference(args, ws, rank):
    """--impl reference: the oracle (this tier's reference arm) on the host cores."""
    if ws > 1 and rank != 0:
        return
    if ws > 1:   # torchrun pins OMP_NUM_THREADS=1; rank 0 alone times the oracle on the host cores
        os.environ["OMP_NUM_THREADS"] = str(os.cpu_count() or 1)
    import synth
    import oracle
    inp = synth.make_inputs(args.config, seed=args.seed)
    oracle.build()
    for _ in range(max(args.warmup, 0)):
        time_oracle(inp, target_s=1.0, seed=99)
    vals = []
    cbs = []
    for s in range(args.steps):
        cb, dt = time_oracle(inp, target_s=8.0, seed=s)
        vals.append(cb["value"])
        cbs.append(cb)
    v = float(np.mean(vals))
    cb = dict(cbs[-1])
    cb["value"] = round(v, 4)
    out = {"metric": METRIC, "value": round(v, 4), "unit": UNIT, "n_gpus": ws, "steps": args.steps,
           "warmup": args.warmup, "higher_is_better": True, "impl": "reference", "dtype": "f64",
           "data": "synthetic (seeded generator, synth/)", "vs_baseline": None,
           "config": {"workload": f"{args.config}: " + synth.CONFIGS[args.config]["desc"]},
           "cpu_baseline": cb,
           "e2e": {"value": round(v, 4), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
