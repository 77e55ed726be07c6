"""Multi-GPU row-block partition of C = A x B (BASELINE.json north_star, R8).

One process per GPU (torch.distributed; NCCL on B200 over NVLink/NVSwitch, gloo in the CPU
tests).  Rows of C are split into balanced blocks (equal shares of intermediate products,
computed on the GPU by ``spgemm_row_partition``); rank r owns rows [r_r, r_{r+1}) of A and a
full copy of B, runs the whole path on its block, and the CSR row blocks are concatenated.
The row blocks are independent: there is no data-path collective inside the product -- the
broadcast of B, the scatter of A's row slices and the gather of C are input / output movement.

All functions take and return plain tensors (``CSC`` / ``CSR`` of the package); the
per-rank compute is ``paper_conf_icde_leekyjkp20_b200.matmul`` (the caller's choice).
"""
from __future__ import annotations

from typing import List, Sequence

import torch
import torch.distributed as dist

from . import CSC, CSR


def _bcast(t: torch.Tensor, src: int) -> torch.Tensor:
    dist.broadcast(t, src=src)
    return t


def broadcast_csr(B: CSR | None, src: int = 0, device=None) -> CSR:
    """Replicate B (CSR) from rank ``src`` to every rank (one broadcast per array)."""
    rank = dist.get_rank()
    dev = torch.device(device) if device is not None else (B.rowptr.device if B is not None else torch.device("cpu"))
    meta = torch.tensor([B.nrows, B.ncols, B.nnz] if rank == src else [0, 0, 0], dtype=torch.int64, device=dev)
    _bcast(meta, src)
    nrows, ncols, nnz = (int(x) for x in meta.tolist())
    if rank == src:
        rowptr, colidx, val = B.rowptr.to(dev), B.colidx.to(dev), B.val.to(dev)
    else:
        rowptr = torch.empty(nrows + 1, dtype=torch.int64, device=dev)
        colidx = torch.empty(nnz, dtype=torch.int32, device=dev)
        val = torch.empty(nnz, dtype=torch.float32, device=dev)
    for t in (rowptr, colidx, val):
        if t.numel():
            _bcast(t, src)
    return CSR(nrows, ncols, rowptr, colidx, val)


def csc_row_slice(A: CSC, r0: int, r1: int) -> CSC:
    """Rows [r0, r1) of a CSC matrix (row indices renumbered from 0); a column keeps its order."""
    keep = (A.rowidx >= r0) & (A.rowidx < r1)
    col_of = torch.repeat_interleave(torch.arange(A.ncols, device=A.colptr.device),
                                     (A.colptr[1:] - A.colptr[:-1]))
    counts = torch.bincount(col_of[keep], minlength=A.ncols)
    colptr = torch.zeros(A.ncols + 1, dtype=torch.int64, device=A.colptr.device)
    colptr[1:] = torch.cumsum(counts, 0)
    return CSC(r1 - r0, A.ncols, colptr, (A.rowidx[keep] - r0).to(torch.int32).contiguous(),
               A.val[keep].contiguous())


def scatter_row_slices(A: CSC | None, bounds: Sequence[int], src: int = 0, device=None) -> CSC:
    """Rank ``src`` holds A; every rank receives its row block [bounds[r], bounds[r+1])."""
    rank, world = dist.get_rank(), dist.get_world_size()
    dev = torch.device(device) if device is not None else torch.device("cpu")
    if rank == src:
        mine = None
        for r in range(world):
            s = csc_row_slice(A, int(bounds[r]), int(bounds[r + 1]))
            if r == src:
                mine = CSC(s.nrows, s.ncols, s.colptr.to(dev), s.rowidx.to(dev), s.val.to(dev))
                continue
            meta = torch.tensor([s.nrows, s.ncols, s.rowidx.numel()], dtype=torch.int64, device=dev)
            dist.send(meta, dst=r)
            for t in (s.colptr, s.rowidx, s.val):
                if t.numel():
                    dist.send(t.to(dev).contiguous(), dst=r)
        return mine
    meta = torch.empty(3, dtype=torch.int64, device=dev)
    dist.recv(meta, src=src)
    nrows, ncols, nnz = (int(x) for x in meta.tolist())
    colptr = torch.empty(ncols + 1, dtype=torch.int64, device=dev)
    rowidx = torch.empty(nnz, dtype=torch.int32, device=dev)
    val = torch.empty(nnz, dtype=torch.float32, device=dev)
    for t in (colptr, rowidx, val):
        if t.numel():
            dist.recv(t, src=src)
    return CSC(nrows, ncols, colptr, rowidx, val)


def concat_row_blocks(blocks: List[CSR]) -> CSR:
    """Stack CSR row blocks vertically (row pointers shifted by the preceding nnz)."""
    ncols = blocks[0].ncols
    rowptrs, off = [], 0
    for q, b in enumerate(blocks):
        rp = b.rowptr + off
        rowptrs.append(rp if q == len(blocks) - 1 else rp[:-1])
        off += b.nnz
    return CSR(sum(b.nrows for b in blocks), ncols, torch.cat(rowptrs),
               torch.cat([b.colidx for b in blocks]), torch.cat([b.val for b in blocks]))


def gather_row_blocks(C: CSR, dst: int = 0) -> CSR | None:
    """Gather every rank's row block of C to rank ``dst`` (None on the other ranks).  Rank ``dst``
    allocates C once and receives every block straight into its slice (no concatenation copy);
    the received row pointers are shifted by the preceding blocks' nnz afterwards."""
    rank, world = dist.get_rank(), dist.get_world_size()
    dev = C.rowptr.device
    meta = torch.tensor([C.nrows, C.nnz], dtype=torch.int64, device=dev)
    metas = [torch.empty_like(meta) for _ in range(world)]
    dist.all_gather(metas, meta)
    if rank != dst:
        for t in (C.rowptr, C.colidx[:C.nnz], C.val[:C.nnz]):
            if t.numel():
                dist.send(t.contiguous(), dst=dst)
        return None
    sizes = [tuple(int(x) for x in m.tolist()) for m in metas]
    M = sum(s[0] for s in sizes)
    NNZ = sum(s[1] for s in sizes)
    rowptr = torch.empty(M + 1, dtype=torch.int64, device=dev)
    colidx = torch.empty(NNZ, dtype=torch.int32, device=dev)
    val = torch.empty(NNZ, dtype=torch.float32, device=dev)
    r0 = e0 = 0
    for r, (nrows, nnz) in enumerate(sizes):
        rp = rowptr[r0:r0 + nrows + 1]
        ci, vv = colidx[e0:e0 + nnz], val[e0:e0 + nnz]
        if r == rank:
            rp.copy_(C.rowptr)
            if nnz:
                ci.copy_(C.colidx[:nnz])
                vv.copy_(C.val[:nnz])
        else:
            for t in (rp, ci, vv):
                if t.numel():
                    buf = t if t.is_contiguous() else torch.empty_like(t)
                    dist.recv(buf, src=r)
        rp.add_(e0)   # block-local row pointers -> global (the next block overwrites rp[-1] with the same value)
        r0 += nrows
        e0 += nnz
    return CSR(M, C.ncols, rowptr, colidx, val)
