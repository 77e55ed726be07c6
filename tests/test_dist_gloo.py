"""Multi-process (world_size 2, gloo, CPU) test of the row-block partition layer in
paper_conf_icde_leekyjkp20_b200/dist.py: broadcast of B, scatter of A's row slices, per-rank
products, gather + concatenation of C's row blocks.  The per-rank compute here is the oracle
(this is a host-logic test; the CUDA path per block is covered by tests/test_gpu_parity.py)."""
import os
import socket

import numpy as np
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from oracle import stages
from paper_conf_icde_leekyjkp20_b200 import CSC, CSR
from paper_conf_icde_leekyjkp20_b200 import dist as pdist


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _to_inputs(A: CSC, B: CSR) -> synth.SparseInputs:
    return synth.SparseInputs("blk", A.nrows, A.ncols, B.ncols, A.colptr.numpy(), A.rowidx.numpy(), A.val.numpy(),
                              B.rowptr.numpy(), B.colidx.numpy(), B.val.numpy())


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        inp = synth.make_inputs("C1", seed=3)
        if rank == 0:
            A = CSC(inp.m, inp.k, torch.from_numpy(inp.a_colptr), torch.from_numpy(inp.a_rowidx),
                    torch.from_numpy(inp.a_val))
            B = CSR(inp.k, inp.n, torch.from_numpy(inp.b_rowptr), torch.from_numpy(inp.b_colidx),
                    torch.from_numpy(inp.b_val))
            bounds = torch.from_numpy(stages.balanced_row_partition(stages.row_workload(inp), world))
        else:
            A = B = None
            bounds = torch.zeros(world + 1, dtype=torch.int64)
        dist.broadcast(bounds, src=0)
        Bl = pdist.broadcast_csr(B, src=0)
        Al = pdist.scatter_row_slices(A, bounds.tolist(), src=0)
        assert Al.nrows == int(bounds[rank + 1] - bounds[rank])
        rp, col, val = oracle.gustavson(_to_inputs(Al, Bl))
        Cl = CSR(Al.nrows, Bl.ncols, torch.from_numpy(rp), torch.from_numpy(col),
                 torch.from_numpy(val.astype(np.float32)))
        C = pdist.gather_row_blocks(Cl, dst=0)
        if rank == 0:
            frp, fcol, fval = oracle.gustavson(inp)
            ok = (np.array_equal(C.rowptr.numpy(), frp) and np.array_equal(C.colidx.numpy(), fcol)
                  and np.array_equal(C.val.numpy(), fval.astype(np.float32)))
            q.put(("ok" if ok else "mismatch", [int(x) for x in bounds]))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put(("error", repr(e)))
        raise
    finally:
        dist.destroy_process_group()


def test_row_blocks_world2_gloo():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=300)
    status, info = q.get(timeout=10)
    assert status == "ok", info
    assert info[0] == 0 and info[-1] == 1024 and 0 < info[1] < 1024


def test_concat_row_blocks_identity():
    inp = synth.make_inputs("C1", seed=4)
    rp, col, val = oracle.gustavson(inp)
    C = CSR(inp.m, inp.n, torch.from_numpy(rp), torch.from_numpy(col), torch.from_numpy(val.astype(np.float32)))
    cut = [0, 100, 100, 700, inp.m]
    blocks = []
    for a, b in zip(cut[:-1], cut[1:]):
        brp = C.rowptr[a:b + 1] - C.rowptr[a]
        blocks.append(CSR(b - a, inp.n, brp, C.colidx[C.rowptr[a]:C.rowptr[b]], C.val[C.rowptr[a]:C.rowptr[b]]))
    D = pdist.concat_row_blocks(blocks)
    assert torch.equal(D.rowptr, C.rowptr) and torch.equal(D.colidx, C.colidx) and torch.equal(D.val, C.val)


def test_csc_row_slice_matches_generator():
    inp = synth.make_inputs("C1", seed=2)
    A = CSC(inp.m, inp.k, torch.from_numpy(inp.a_colptr), torch.from_numpy(inp.a_rowidx), torch.from_numpy(inp.a_val))
    s = pdist.csc_row_slice(A, 100, 300)
    ref = synth.row_slice_coo(inp, 100, 300)
    assert np.array_equal(s.colptr.numpy(), ref.a_colptr)
    assert np.array_equal(s.rowidx.numpy(), ref.a_rowidx)
    assert np.array_equal(s.val.numpy(), ref.a_val)
