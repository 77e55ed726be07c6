"""ORACLE -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` leg may import this package.  It shares no code with the
CUDA path (``paper_conf_icde_leekyjkp20_b200``) and never imports it.

Contents
  * :func:`gustavson` -- plain C (OpenMP over rows) fp64 dense-accumulator
    row-product spGEMM, PAPER.md L199-L211 R / L476-L478 R (reconstructed
    Eq. (1)).  Pinned by tests/test_oracle_*.py against a hand-worked example,
    dense brute force, the transpose identity, exact integer runs and the
    invariants  sum_k nnzcol_A(k)*nnzrow_B(k) = #products  and  C*1 = A*(B*1).
  * :mod:`oracle.stages` -- the per-stage definitions of the Block Reorganizer
    (workload analysis, categorisation, B-Splitting, B-Gathering, B-Limiting
    bins, outer-product expansion of Eq. (2)), written out step by step.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "gustavson.c")
_lib = None


def build(force: bool = False) -> str:
    """Compile the C oracle with gcc (-O2 -fopenmp).  Building the checker is not using it."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11",
                               "-o", _SO, _SRC])
    return _SO


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        p = ctypes.c_void_p
        i64 = ctypes.c_int64
        lib.oracle_gustavson_count.argtypes = [i64, i64, i64, p, p, p, p, p, p, p, i64, p, ctypes.c_int]
        lib.oracle_gustavson_fill.argtypes = [i64, i64, i64, p, p, p, p, p, p, p, i64, p, p, p, ctypes.c_int]
        lib.oracle_gustavson_count.restype = ctypes.c_int
        lib.oracle_gustavson_fill.restype = ctypes.c_int
        lib.oracle_max_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p) if a is not None else None


def max_threads() -> int:
    return int(_load().oracle_max_threads())


def gustavson(inp, rows=None, threads: int = 0):
    """C = A x B by Gustavson's row product in fp64.

    ``inp`` is a :class:`synth.SparseInputs`.  Returns ``(rowptr int64, col int32,
    val float64)`` for all rows, or for the listed ``rows`` (in that order).
    """
    lib = _load()
    a_colptr = np.ascontiguousarray(inp.a_colptr, dtype=np.int64)
    a_rowidx = np.ascontiguousarray(inp.a_rowidx, dtype=np.int32)
    a_val = np.ascontiguousarray(inp.a_val, dtype=np.float32)
    b_rowptr = np.ascontiguousarray(inp.b_rowptr, dtype=np.int64)
    b_colidx = np.ascontiguousarray(inp.b_colidx, dtype=np.int32)
    b_val = np.ascontiguousarray(inp.b_val, dtype=np.float32)
    if rows is not None:
        rows = np.ascontiguousarray(rows, dtype=np.int32)
        nrows = rows.size
    else:
        nrows = inp.m
    count = np.zeros(max(nrows, 1), dtype=np.int64)
    args = (inp.m, inp.k, inp.n, _ptr(a_colptr), _ptr(a_rowidx), _ptr(a_val), _ptr(b_rowptr),
            _ptr(b_colidx), _ptr(b_val), _ptr(rows), nrows)
    if lib.oracle_gustavson_count(*args, _ptr(count), threads) != 0:
        raise MemoryError("oracle count failed")
    rowptr = np.zeros(nrows + 1, dtype=np.int64)
    np.cumsum(count[:nrows], out=rowptr[1:])
    nnz = int(rowptr[-1])
    col = np.zeros(max(nnz, 1), dtype=np.int32)
    val = np.zeros(max(nnz, 1), dtype=np.float64)
    if lib.oracle_gustavson_fill(*args, _ptr(rowptr), _ptr(col), _ptr(val), threads) != 0:
        raise MemoryError("oracle fill failed")
    return rowptr, col[:nnz], val[:nnz]
