"""Whole-matrix parity of a GPU C against the oracle, row chunk by row chunk (test infrastructure).

The oracle (oracle.gustavson, fp64) computes C's rows [r0, r1) on the host cores; the GPU C's rows
[r0, r1) are compared with it: row pointers and column indices bit-exactly, values within the
north-star tolerance |got - want| <= 1e-5 |want| (signed inputs: + 2^-23 sum|a||b|).
Chunks hold ~`chunk_products` intermediate products so the oracle's output of one chunk stays a few
GB; the comparison itself runs on the GPU (torch ops on the copied oracle chunk)."""
import functools

import numpy as np
import torch

import oracle
import synth

RTOL = 1e-5


@functools.lru_cache(maxsize=1)
def cached_inputs(name, seed=1, values="real"):
    """The full-size generators take up to ~2.5 min (C5): one config is kept between tests."""
    return synth.make_inputs(name, seed=seed, values=values)


def row_products(inp):
    """Intermediate products per row (sum over stored a_ik of nnz(b_k*)), via bincount."""
    rb = np.diff(inp.b_rowptr).astype(np.float64)
    col_of = np.repeat(np.arange(inp.k, dtype=np.int64), np.diff(inp.a_colptr))
    return np.bincount(inp.a_rowidx, weights=rb[col_of], minlength=inp.m).astype(np.int64)


def abs_inputs(inp):
    return synth.SparseInputs(inp.name + "|abs|", inp.m, inp.k, inp.n, inp.a_colptr, inp.a_rowidx,
                              np.abs(inp.a_val), inp.b_rowptr, inp.b_colidx, np.abs(inp.b_val))


def whole_matrix_check(C, inp, chunk_products=600_000_000, signed=False, exact_values=False):
    """Every row of C against the oracle; returns (rows, entries, chunks) checked."""
    dev = C.colidx.device
    rowptr = C.rowptr.cpu().numpy()
    assert rowptr.shape == (inp.m + 1,) and rowptr[0] == 0 and rowptr[-1] == C.nnz
    pref = np.concatenate([[0], np.cumsum(row_products(inp))])
    r0, chunks, entries = 0, 0, 0
    while r0 < inp.m:
        r1 = int(np.searchsorted(pref, pref[r0] + chunk_products, side="right")) - 1
        r1 = min(inp.m, max(r1, r0 + 1))
        rows = np.arange(r0, r1, dtype=np.int32)
        orp, ocol, oval = oracle.gustavson(inp, rows=rows)
        np.testing.assert_array_equal(rowptr[r0:r1 + 1] - rowptr[r0], orp,
                                      err_msg=f"row pointers differ in rows [{r0}, {r1})")
        a, b = int(rowptr[r0]), int(rowptr[r1])
        gcol = C.colidx[a:b]
        ocol_t = torch.from_numpy(ocol).to(dev)
        if not torch.equal(gcol, ocol_t):
            bad = int(torch.nonzero(gcol != ocol_t)[0, 0])
            raise AssertionError(f"column index differs at entry {a + bad} (rows [{r0}, {r1})): "
                                 f"got {int(gcol[bad])} want {int(ocol_t[bad])}")
        gv = C.val[a:b].double()
        ov = torch.from_numpy(oval).to(dev)
        if exact_values:
            ok = gv == ov
        else:
            tol = RTOL * ov.abs()
            if signed:
                _, _, mag = oracle.gustavson(abs_inputs(inp), rows=rows)
                tol = tol + 2.0 ** -23 * torch.from_numpy(mag).to(dev)
            ok = (gv - ov).abs() <= tol
        if not bool(ok.all()):
            bad = int(torch.nonzero(~ok)[0, 0])
            raise AssertionError(f"value out of tolerance at entry {a + bad}: got {float(gv[bad])} "
                                 f"want {float(ov[bad])}")
        entries += b - a
        chunks += 1
        del gcol, ocol_t, gv, ov, orp, ocol, oval
        r0 = r1
    return inp.m, entries, chunks
