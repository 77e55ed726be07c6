"""Python binding of the B200 outer-product spGEMM library (include/spgemm.h).

Argument marshalling only: every step of the path (workload analysis, Block
Reorganizer, expansion, merge, compaction) runs in the CUDA kernels of
``csrc/`` behind the C-ABI in ``libspgemm.so``.  There is no CPU fallback: if
the library is missing or no GPU is present the calls raise.

    C = matmul(A, B)                 # A: CSC, B: CSR (torch tensors, cuda or cpu)
    with Plan(A, B) as p:            # stage-by-stage access (tests, tooling)
        p.expand(); nnz = p.merge(); C = p.output()
"""
from __future__ import annotations

import ctypes
import dataclasses
import os
from typing import Optional

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SPGEMM_LIB") or os.path.join(_HERE, "libspgemm.so")   # (override: A/B builds)

SPGEMM_DEVICE, SPGEMM_HOST = 0, 1
VIEW_WORK, VIEW_ROWWORK, VIEW_ROWOFF, VIEW_PAIR_CLASS, VIEW_PIECES, VIEW_GATHER, VIEW_ROW_CLASS, \
    VIEW_CHAT_COL, VIEW_CHAT_VAL, VIEW_CROWPTR, VIEW_UNIT_PROFILE, VIEW_ROW_COLMIN, VIEW_ROW_COLMAX, VIEW_LBI = range(14)

EXPORTED = ["spgemm_abi_version", "spgemm_last_error", "spgemm_default_options", "spgemm_plan",
            "spgemm_expand", "spgemm_merge", "spgemm_output", "spgemm_execute", "spgemm_get_stats",
            "spgemm_inspect", "spgemm_destroy", "spgemm_set_timing", "spgemm_last_timings",
            "spgemm_row_partition", "spgemm_trim_pool", "spgemm_plan_rows"]


class SpgemmError(RuntimeError):
    pass


class _CSC(ctypes.Structure):
    _fields_ = [("nrows", ctypes.c_int64), ("ncols", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("colptr", ctypes.c_void_p), ("rowidx", ctypes.c_void_p), ("val", ctypes.c_void_p),
                ("where", ctypes.c_int32)]


class _CSR(ctypes.Structure):
    _fields_ = [("nrows", ctypes.c_int64), ("ncols", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("rowptr", ctypes.c_void_p), ("colidx", ctypes.c_void_p), ("val", ctypes.c_void_p),
                ("where", ctypes.c_int32)]


class Options(ctypes.Structure):
    _fields_ = [("alpha", ctypes.c_double), ("dom_waves", ctypes.c_int32), ("dom_min_work", ctypes.c_int64),
                ("split_ca_max", ctypes.c_int32), ("piece_work", ctypes.c_int64),
                ("split_b_tile", ctypes.c_int32), ("beta", ctypes.c_double),
                ("limit_ctas_per_sm", ctypes.c_int32), ("enable_split", ctypes.c_int32),
                ("enable_gather", ctypes.c_int32), ("enable_limit", ctypes.c_int32),
                ("validate", ctypes.c_int32), ("reserved", ctypes.c_int32 * 16)]


class Stats(ctypes.Structure):
    _fields_ = [(f, ctypes.c_int64) for f in (
        "m", "k", "n", "nnz_a", "nnz_b", "nnz_chat", "nnz_chat_rowwise", "nnz_c", "k_nonempty",
        "m_nonempty", "t_dom", "t_lim", "n_dominator", "n_normal", "n_low", "n_pieces_split")] + [
        ("n_gather_bin", ctypes.c_int64 * 6), ("n_rows_bin", ctypes.c_int64 * 6),
        ("bytes_workspace", ctypes.c_int64), ("n_units", ctypes.c_int64), ("n_units_fallback", ctypes.c_int64)]

    def as_dict(self):
        d = {f: getattr(self, f) for f, _ in self._fields_}
        d["n_gather_bin"] = list(self.n_gather_bin)
        d["n_rows_bin"] = list(self.n_rows_bin)
        return d


_ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int32, ctypes.c_void_p)
_lib_handle = None


def lib():
    """Load libspgemm.so; raises if it has not been built (no fallback path exists)."""
    global _lib_handle
    if _lib_handle is None:
        if not os.path.exists(LIB_PATH):
            raise SpgemmError(f"{LIB_PATH} missing: run __graft_entry__.build() (no CPU fallback)")
        L = ctypes.CDLL(LIB_PATH)
        vp, i32, i64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
        L.spgemm_abi_version.restype = ctypes.c_int
        L.spgemm_last_error.restype = ctypes.c_char_p
        L.spgemm_default_options.argtypes = [ctypes.POINTER(Options)]
        L.spgemm_plan.argtypes = [ctypes.POINTER(_CSC), ctypes.POINTER(_CSR), ctypes.POINTER(Options), vp,
                                  ctypes.POINTER(vp)]
        L.spgemm_plan_rows.argtypes = [ctypes.POINTER(_CSC), ctypes.POINTER(_CSR), i64, i64, ctypes.POINTER(Options),
                                       vp, ctypes.POINTER(vp)]
        L.spgemm_expand.argtypes = [vp, vp]
        L.spgemm_merge.argtypes = [vp, vp, ctypes.POINTER(i64)]
        L.spgemm_output.argtypes = [vp, ctypes.POINTER(_CSR), vp]
        L.spgemm_execute.argtypes = [vp, _ALLOC_FN, vp, i32, ctypes.POINTER(_CSR), vp]
        L.spgemm_get_stats.argtypes = [vp, ctypes.POINTER(Stats)]
        L.spgemm_inspect.argtypes = [vp, i32, vp, i64, ctypes.POINTER(i64)]
        L.spgemm_destroy.argtypes = [vp]
        L.spgemm_row_partition.argtypes = [ctypes.POINTER(_CSC), ctypes.POINTER(_CSR), i32, vp, vp]
        L.spgemm_set_timing.argtypes = [i32]
        L.spgemm_trim_pool.argtypes = []
        L.spgemm_last_timings.argtypes = [ctypes.POINTER(ctypes.c_char_p), ctypes.POINTER(ctypes.c_float), i32,
                                          ctypes.POINTER(i32)]
        for f in EXPORTED:
            if getattr(L, f).restype is None and f not in ("spgemm_default_options",):
                getattr(L, f).restype = ctypes.c_int
        if L.spgemm_abi_version() != 1:
            raise SpgemmError("ABI version mismatch")
        _lib_handle = L
    return _lib_handle


def _check(code: int):
    if code != 0:
        raise SpgemmError(f"spgemm error {code}: {lib().spgemm_last_error().decode(errors='replace')}")


@dataclasses.dataclass
class CSC:
    """A (nrows x ncols) by columns: colptr int64[ncols+1], rowidx int32[nnz], val float32[nnz]."""
    nrows: int
    ncols: int
    colptr: torch.Tensor
    rowidx: torch.Tensor
    val: torch.Tensor


@dataclasses.dataclass
class CSR:
    """(nrows x ncols) by rows: rowptr int64[nrows+1], colidx int32[nnz], val float32[nnz]."""
    nrows: int
    ncols: int
    rowptr: torch.Tensor
    colidx: torch.Tensor
    val: torch.Tensor

    @property
    def nnz(self) -> int:
        return int(self.colidx.numel())


def _where(t: torch.Tensor) -> int:
    return SPGEMM_DEVICE if t.is_cuda else SPGEMM_HOST


def _ptr(t: torch.Tensor):
    assert t.is_contiguous()
    return ctypes.c_void_p(t.data_ptr()) if t.numel() else ctypes.c_void_p(t.data_ptr() or 1)


def options(**kw) -> Options:
    o = Options()
    lib().spgemm_default_options(ctypes.byref(o))
    for k, v in kw.items():
        if not hasattr(o, k):
            raise KeyError(k)
        if k == "reserved":
            for q, x in enumerate(v):
                o.reserved[q] = x
            continue
        setattr(o, k, v)
    return o


def _stream(stream) -> ctypes.c_void_p:
    if stream is None:
        stream = torch.cuda.current_stream() if torch.cuda.is_available() else None
    return ctypes.c_void_p(stream.cuda_stream if stream is not None else 0)


class Plan:
    """One C = A x B problem: spgemm_plan (stages 1-2) on construction."""

    def __init__(self, A: CSC, B: CSR, stream=None, rows=None, **opts):
        """rows=(r0, r1): plan rows [r0, r1) of C only (spgemm_plan_rows; A is windowed on the GPU)."""
        self._keep = (A, B)
        self.stream = _stream(stream)
        r0, r1 = (0, A.nrows) if rows is None else (int(rows[0]), int(rows[1]))
        self.m, self.n = r1 - r0, B.ncols
        a = _CSC(A.nrows, A.ncols, A.rowidx.numel(), _ptr(A.colptr), _ptr(A.rowidx), _ptr(A.val), _where(A.colptr))
        b = _CSR(B.nrows, B.ncols, B.colidx.numel(), _ptr(B.rowptr), _ptr(B.colidx), _ptr(B.val), _where(B.rowptr))
        o = options(**opts)
        h = ctypes.c_void_p()
        _check(lib().spgemm_plan_rows(ctypes.byref(a), ctypes.byref(b), r0, r1, ctypes.byref(o), self.stream,
                                      ctypes.byref(h)))
        self.h = h

    def expand(self):
        _check(lib().spgemm_expand(self.h, self.stream))

    def merge(self) -> int:
        n = ctypes.c_int64()
        _check(lib().spgemm_merge(self.h, self.stream, ctypes.byref(n)))
        self.nnz_c = n.value
        return n.value

    def output(self, device: Optional[torch.device] = None, out: Optional[CSR] = None) -> CSR:
        """Compaction into new (or given) tensors on `device` (cuda default; 'cpu' = host)."""
        if out is None:
            dev = torch.device("cuda") if device is None else torch.device(device)
            pin = dev.type == "cpu"
            out = CSR(self.m, self.n, torch.empty(self.m + 1, dtype=torch.int64, device=dev, pin_memory=pin),
                      torch.empty(self.nnz_c, dtype=torch.int32, device=dev, pin_memory=pin),
                      torch.empty(self.nnz_c, dtype=torch.float32, device=dev, pin_memory=pin))
        c = _CSR(self.m, self.n, self.nnz_c, _ptr(out.rowptr), _ptr(out.colidx), _ptr(out.val), _where(out.rowptr))
        _check(lib().spgemm_output(self.h, ctypes.byref(c), self.stream))
        return out

    def execute(self, device=None, pool: "Optional[HostBufferPool]" = None) -> CSR:
        """spgemm_execute: expand + merge + allocate C through a callback + compaction.
        With device='cpu', C lands in pinned host memory (from `pool` when given)."""
        dev = torch.device("cuda") if device is None else torch.device(device)
        where = SPGEMM_HOST if dev.type == "cpu" else SPGEMM_DEVICE
        bufs = []

        def _alloc(nbytes, w, ctx):
            if pool is not None and w == SPGEMM_HOST:
                t = pool.get(len(bufs), max(int(nbytes), 1))
            else:
                t = torch.empty(max(int(nbytes), 1), dtype=torch.uint8, device=dev, pin_memory=(w == SPGEMM_HOST))
            bufs.append(t)
            return t.data_ptr()

        cb = _ALLOC_FN(_alloc)
        c = _CSR()
        _check(lib().spgemm_execute(self.h, cb, None, where, ctypes.byref(c), self.stream))
        nnz = int(c.nnz)
        self.nnz_c = nnz
        return CSR(self.m, self.n, bufs[0][: (self.m + 1) * 8].view(torch.int64),
                   bufs[1][: nnz * 4].view(torch.int32), bufs[2][: nnz * 4].view(torch.float32))

    def stats(self) -> dict:
        s = Stats()
        _check(lib().spgemm_get_stats(self.h, ctypes.byref(s)))
        return s.as_dict()

    def inspect(self, view: int, dtype, count: Optional[int] = None):
        import numpy as np
        size = ctypes.c_int64()
        lib().spgemm_inspect(self.h, view, None, 0, ctypes.byref(size))
        buf = np.empty(max(size.value, 1), dtype=np.uint8)
        _check(lib().spgemm_inspect(self.h, view, buf.ctypes.data_as(ctypes.c_void_p), buf.size, ctypes.byref(size)))
        return buf[: size.value].view(dtype)

    def lbi(self) -> dict:
        """Load balancing index (Eq. (3), L564-L577 R) of the expansion and of the B-Limited
        merge kernel of this plan (plan created with reserved[8] = 1, after merge): mean over the
        SMs of the SM's busy time T_i normalised by the longest, T_i = last CTA end on SM i - the
        kernel's first CTA start (SMs that ran nothing count as 0)."""
        import numpy as np
        raw = self.inspect(VIEW_LBI, np.uint64).reshape(2, -1).astype(np.int64)
        nsm = torch.cuda.get_device_properties(torch.cuda.current_device()).multi_processor_count
        out = {}
        for name, row in zip(("expand", "merge_limited"), raw):
            t0, ends = int(row[0]), row[1:1 + nsm]
            if t0 <= 0 or ends.max() <= 0:   # (0xff.. = never started: -1 as int64)
                out[name] = None
                continue
            busy = np.where(ends > 0, ends - t0, 0).astype(np.float64)
            out[name] = {"lbi": float(busy.mean() / busy.max()), "max_ms": float(busy.max() / 1e6),
                         "mean_ms": float(busy.mean() / 1e6)}
        return out

    def destroy(self):
        if getattr(self, "h", None):
            lib().spgemm_destroy(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.destroy()

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass


class HostBufferPool:
    """Reusable pinned host buffers for repeated host-output calls (C rowptr / colidx / val)."""

    def __init__(self):
        self.bufs = {}

    def get(self, slot: int, nbytes: int) -> torch.Tensor:
        b = self.bufs.get(slot)
        if b is None or b.numel() < nbytes:
            b = torch.empty(int(nbytes) + 4096, dtype=torch.uint8, pin_memory=True)
            self.bufs[slot] = b
        return b[:nbytes]


def matmul(A: CSC, B: CSR, device=None, stream=None, rows=None, **opts) -> CSR:
    """C = A x B (outer-product spGEMM with the Block Reorganizer); C is canonical CSR.
    rows=(r0, r1): only rows [r0, r1) of C (the row block, renumbered from 0)."""
    with Plan(A, B, stream=stream, rows=rows, **opts) as p:
        return p.execute(device=device)


def matmul_chunked(A: CSC, B: CSR, parts: int, device=None, stream=None, **opts) -> CSR:
    """C = A x B in `parts` balanced row blocks run one after another (north star C5: chunked
    expansion): the blocks' Ĉ are formed and merged in turn, so the peak intermediate storage is
    ~nnz(Ĉ)/parts.  Same boundaries as the multi-GPU row partition (R8)."""
    from . import dist as pdist
    if parts <= 1:
        return matmul(A, B, device=device, stream=stream, **opts)
    bounds = row_partition(A, B, parts, stream=stream)
    blocks = []
    for r in range(parts):   # (the row window is cut on the GPU by spgemm_plan_rows: no copy of A here)
        C = matmul(A, B, device=device, stream=stream, rows=(int(bounds[r]), int(bounds[r + 1])), **opts)
        if C.colidx.untyped_storage().nbytes() > C.colidx.numel() * 4 * 1.05:   # release capacity slack
            C = CSR(C.nrows, C.ncols, C.rowptr, C.colidx.clone(), C.val.clone())
        blocks.append(C)
    return pdist.concat_row_blocks(blocks)


def row_partition(A: CSC, B: CSR, parts: int, stream=None):
    """Balanced row-block boundaries (parts+1 int64) of C = A x B, computed on the GPU."""
    import numpy as np
    a = _CSC(A.nrows, A.ncols, A.rowidx.numel(), _ptr(A.colptr), _ptr(A.rowidx), _ptr(A.val), _where(A.colptr))
    b = _CSR(B.nrows, B.ncols, B.colidx.numel(), _ptr(B.rowptr), _ptr(B.colidx), _ptr(B.val), _where(B.rowptr))
    out = np.zeros(parts + 1, dtype=np.int64)
    _check(lib().spgemm_row_partition(ctypes.byref(a), ctypes.byref(b), parts,
                                      out.ctypes.data_as(ctypes.c_void_p), _stream(stream)))
    return out


def trim_pool():
    """Return the plans' cached device memory (stream-ordered pool) to the driver."""
    _check(lib().spgemm_trim_pool())


def set_timing(enable: bool):
    _check(lib().spgemm_set_timing(1 if enable else 0))


def last_timings():
    """[(kernel name, ms)] of the launches since the last spgemm_plan (timing enabled)."""
    cnt = ctypes.c_int32()
    _check(lib().spgemm_last_timings(None, None, 0, ctypes.byref(cnt)))
    names = (ctypes.c_char_p * cnt.value)()
    ms = (ctypes.c_float * cnt.value)()
    _check(lib().spgemm_last_timings(names, ms, cnt.value, ctypes.byref(cnt)))
    return [(names[q].decode(), float(ms[q])) for q in range(cnt.value)]


def from_inputs(inp, device="cuda"):
    """(CSC A, CSR B) tensors from a synth.SparseInputs (argument marshalling helper)."""
    dev = torch.device(device)
    pin = dev.type == "cpu" and torch.cuda.is_available()

    def t(x):
        x = torch.from_numpy(x)
        return x.pin_memory() if pin else x.to(dev)

    A = CSC(inp.m, inp.k, t(inp.a_colptr), t(inp.a_rowidx), t(inp.a_val))
    B = CSR(inp.k, inp.n, t(inp.b_rowptr), t(inp.b_colidx), t(inp.b_val))
    return A, B
