"""Two ranks sharing one B200 (gloo process group; NCCL needs one GPU per rank): the multi-GPU
row-block path end to end -- rank 0 builds the input and the balanced row partition on its GPU
(spgemm_row_partition), B is broadcast and A's row slices are scattered (dist.py), each rank runs
the CUDA path on its block, the C row blocks are gathered to rank 0 and the assembled C is
compared with the oracle's whole C (structure bit-exact, values within 1e-5)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, name, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import synth
        import paper_conf_icde_leekyjkp20_b200 as spg
        from paper_conf_icde_leekyjkp20_b200 import dist as pdist
        torch.cuda.set_device(0)
        cpu = torch.device("cpu")
        if rank == 0:
            inp = synth.make_inputs(name, seed=2)
            A, B = spg.from_inputs(inp, "cuda")
            bounds = torch.from_numpy(spg.row_partition(A, B, world))
            Ac = spg.CSC(A.nrows, A.ncols, A.colptr.cpu(), A.rowidx.cpu(), A.val.cpu())
            Bc = spg.CSR(B.nrows, B.ncols, B.rowptr.cpu(), B.colidx.cpu(), B.val.cpu())
        else:
            bounds = torch.zeros(world + 1, dtype=torch.int64)
            Ac = Bc = None
        dist.broadcast(bounds, src=0)
        Bl = pdist.broadcast_csr(Bc, src=0, device=cpu)
        Al = pdist.scatter_row_slices(Ac, bounds.tolist(), src=0, device=cpu)
        dev = torch.device("cuda", 0)
        Ag = spg.CSC(Al.nrows, Al.ncols, Al.colptr.to(dev), Al.rowidx.to(dev), Al.val.to(dev))
        Bg = spg.CSR(Bl.nrows, Bl.ncols, Bl.rowptr.to(dev), Bl.colidx.to(dev), Bl.val.to(dev))
        Cl = spg.matmul(Ag, Bg)                       # the CUDA path on this rank's row block
        torch.cuda.synchronize()
        Cc = spg.CSR(Cl.nrows, Cl.ncols, Cl.rowptr.cpu(), Cl.colidx[:Cl.nnz].cpu(), Cl.val[:Cl.nnz].cpu())
        C = pdist.gather_row_blocks(Cc, dst=0)
        if rank == 0:
            rowptr, col, val = oracle.gustavson(inp)
            ok = np.array_equal(C.rowptr.numpy(), rowptr) and np.array_equal(C.colidx.numpy(), col)
            ok = ok and bool(np.all(np.abs(C.val.numpy().astype(np.float64) - val) <= 1e-5 * np.abs(val)))
            q.put(("ok" if ok else "mismatch", [int(x) for x in bounds]))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put(("error", repr(e)))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("name", ["C1", "P3"])
def test_two_ranks_one_gpu_cuda_path(name):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, name, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=600)
    status, info = q.get(timeout=10)
    assert status == "ok", info
    assert info[0] == 0 and 0 < info[1] < info[2]


def test_bench_two_ranks_share_gpu():
    """bench.py --gpus 2 (re-launching itself under torch.distributed.run) with both ranks on this
    B200 (SPGEMM_BENCH_SHARE_GPU: gloo instead of NCCL): rank 0 prints one JSON line with n_gpus 2,
    the per-rank step times, the C gather timing and the e2e leg."""
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, SPGEMM_BENCH_SHARE_GPU="1")
    env.pop("WORLD_SIZE", None)
    out = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--gpus", "2", "--config", "C1",
                          "--steps", "2", "--warmup", "1", "--no-cpu-baseline"], capture_output=True, text=True,
                         timeout=900, cwd=root, env=env)
    assert out.returncode == 0, out.stderr[-3000:]
    line = [ln for ln in out.stdout.splitlines() if ln.startswith("{")][-1]
    d = json.loads(line)
    assert d["n_gpus"] == 2 and len(d["rank_ms_per_step"]) == 2 and d["value"] > 0
    assert d["c_gather"]["ms"] > 0 and d["e2e"]["value"] > 0
    assert d["config"]["products"] > 0 and d["config"]["m"] == 1024
