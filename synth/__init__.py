"""Seeded synthetic sparse-matrix generators shared by the oracle and the CUDA path.

This module holds NO arithmetic of the spGEMM method (no workload analysis, no
products, no merge).  It only draws graphs and edge weights and lays them out in
the two input formats the paper's outer-product formulation consumes: A by
columns (CSC, "a_*k") and B by rows (CSR, "b_k*") -- PAPER.md Fig. 5
(L333-L339: A'ptr/A'idx/A'val, B'ptr/B'idx/B'val).

Workload recipes (stated in DESIGN.md §3, "input recipe"):

* R-MAT (Chakrabarti et al. [29], PAPER.md L486-L491 R, Table III):
  ``edge_factor * 2**scale`` edges, each placed by ``scale`` recursive quadrant
  draws with probabilities (a, b, c, d); duplicate edges are dropped (Table III
  lists nnz below 16*2**scale).
* Chung-Lu power law: expected degrees ``w_i ∝ (i+i0)^(-1/(gamma-1))`` scaled to
  the edge count with ``i0`` chosen so the largest expected degree equals the
  target maximum degree; endpoints are drawn independently in proportion to
  the out / in weights; in-weight ranks are correlated with out-weight ranks by
  a log-normal rank perturbation ``sigma``; node labels are randomly permuted.
* Erdős–Rényi: ``per_row`` uniformly random columns per row.

Values are a counter-based hash of (row, col, seed) so any entry can be
recomputed independently; ``kind='real'`` gives values in [0.5, 1.5) on a
2**-23 grid (exactly representable in fp32), ``kind='int'`` gives {1,2,3,4},
``kind='pm1'`` gives +-1 (exact sums, many of them exactly zero).
"""
from __future__ import annotations

import dataclasses
import numpy as np

__all__ = [
    "CONFIGS", "SparseInputs", "rmat_edges", "chung_lu_edges", "er_edges",
    "edge_values", "coo_to_csr", "coo_to_csc", "make_inputs", "random_tiny",
    "row_slice_coo",
]

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def _splitmix64(x: np.ndarray) -> np.ndarray:
    """Counter-based 64-bit mixer (Steele et al. SplitMix64 finaliser), wrapping uint64."""
    with np.errstate(over="ignore"):
        z = (x + np.uint64(0x9E3779B97F4A7C15)) & _M64
        z = ((z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)) & _M64
        z = ((z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)) & _M64
        return z ^ (z >> np.uint64(31))


def edge_values(rows: np.ndarray, cols: np.ndarray, seed: int, kind: str = "real") -> np.ndarray:
    """Deterministic per-entry weights, a pure function of (row, col, seed)."""
    key = (rows.astype(np.uint64) << np.uint64(32)) | cols.astype(np.uint64)
    with np.errstate(over="ignore"):
        key = key ^ (np.uint64(seed & 0xFFFFFFFF) * np.uint64(0xD1B54A32D192ED03) & _M64)
    h = _splitmix64(key)
    if kind == "real":
        return (0.5 + (h >> np.uint64(41)).astype(np.float64) * 2.0 ** -23).astype(np.float32)
    if kind == "int":
        return (1 + (h >> np.uint64(62))).astype(np.float32)
    if kind == "pm1":   # +-1: exact integer sums with frequent exact cancellation (computed zeros)
        return np.where((h >> np.uint64(63)) == 1, -1.0, 1.0).astype(np.float32)
    if kind == "signed":
        v = (0.5 + (h >> np.uint64(41)).astype(np.float64) * 2.0 ** -23)
        sign = np.where((h & np.uint64(1)) == 1, -1.0, 1.0)
        return (v * sign).astype(np.float32)
    raise ValueError(kind)


def _dedupe(src: np.ndarray, dst: np.ndarray, ncols: int):
    key = np.sort(src.astype(np.int64) * np.int64(ncols) + dst.astype(np.int64))   # == np.unique, without
    if key.size > 1:                                                             # its slow hash path
        key = key[np.concatenate([[True], key[1:] != key[:-1]])]
    return (key // ncols).astype(np.int32), (key % ncols).astype(np.int32)


def rmat_edges(scale: int, edge_factor: int, a: float, b: float, c: float, seed: int):
    """R-MAT edge list (src, dst), duplicates dropped, sorted by (src, dst)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    m = edge_factor * (1 << scale)
    src = np.zeros(m, dtype=np.int64)
    dst = np.zeros(m, dtype=np.int64)
    ab, abc = a + b, a + b + c
    for _ in range(scale):
        u = rng.random(m)
        src = (src << 1) | (u >= ab)
        dst = (dst << 1) | (((u >= a) & (u < ab)) | (u >= abc))
    return _dedupe(src, dst, 1 << scale)


def rmat_n_edges(n: int, nedges: int, a: float, b: float, c: float, seed: int):
    """R-MAT over n nodes (any n): draws in the 2^ceil(log2 n) square, rejects endpoints >= n until
    nedges edges are drawn, then drops duplicates (Table III, R-MAT [29])."""
    rng = np.random.Generator(np.random.PCG64(seed))
    scale = max(1, int(np.ceil(np.log2(n))))
    ab, abc = a + b, a + b + c
    got_s, got_d, have = [], [], 0
    while have < nedges:
        m = int((nedges - have) * 1.3) + 1024
        src = np.zeros(m, dtype=np.int64)
        dst = np.zeros(m, dtype=np.int64)
        for _ in range(scale):
            u = rng.random(m)
            src = (src << 1) | (u >= ab)
            dst = (dst << 1) | (((u >= a) & (u < ab)) | (u >= abc))
        ok = (src < n) & (dst < n)
        src, dst = src[ok][: nedges - have], dst[ok][: nedges - have]
        got_s.append(src)
        got_d.append(dst)
        have += src.size
    return _dedupe(np.concatenate(got_s), np.concatenate(got_d), n)


def _powerlaw_weights(n: int, m: float, gamma: float, wmax: float) -> np.ndarray:
    p = 1.0 / (gamma - 1.0)
    i = np.arange(n, dtype=np.float64)
    lo, hi = 1e-6, 1e12
    for _ in range(200):
        mid = np.sqrt(lo * hi)
        if mid <= lo or mid >= hi:   # converged to adjacent doubles: later steps change nothing
            break
        w = (i + mid) ** (-p)
        w *= m / w.sum()
        if w[0] > wmax:
            lo = mid
        else:
            hi = mid
    w = (i + hi) ** (-p)
    return w * (m / w.sum())


def _inverse_cdf(cdf: np.ndarray, u: np.ndarray) -> np.ndarray:
    """np.searchsorted(cdf, u, side='right'), element for element; the draws are searched in sorted
    order (a cache-friendly sweep of the table) and put back in draw order."""
    order = np.argsort(u, kind="stable")
    out = np.empty(u.size, dtype=np.int64)
    out[order] = np.searchsorted(cdf, u[order], side="right")
    return out


def chung_lu_edges(n: int, m: int, gamma_out: float, gamma_in: float, max_out: float,
                   max_in: float, sigma: float, seed: int, symmetric: bool = False):
    """Directed (or symmetrised) Chung-Lu power-law graph; returns deduped (src, dst)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    w_out = _powerlaw_weights(n, m, gamma_out, max_out)
    w_in_sorted = _powerlaw_weights(n, m, gamma_in, max_in)
    if symmetric:
        w_in = w_out
    else:
        # in-rank of node i: sort log(i+1) + sigma*z  (sigma=0: identical ranks)
        key = np.log(np.arange(n, dtype=np.float64) + 1.0) + sigma * rng.standard_normal(n)
        order = np.argsort(key, kind="stable")
        w_in = np.empty(n)
        w_in[order] = w_in_sorted
    m_draw = m // 2 if symmetric else m
    cdf_o = np.cumsum(w_out)
    cdf_i = np.cumsum(w_in)
    src = _inverse_cdf(cdf_o, rng.random(m_draw) * cdf_o[-1])
    dst = _inverse_cdf(cdf_i, rng.random(m_draw) * cdf_i[-1])
    np.minimum(src, n - 1, out=src)
    np.minimum(dst, n - 1, out=dst)
    perm = rng.permutation(n)
    src, dst = perm[src], perm[dst]
    if symmetric:
        src, dst = np.concatenate([src, dst]), np.concatenate([dst, src])
    return _dedupe(src, dst, n)


def er_edges(n: int, per_row: int, seed: int):
    """Erdős–Rényi-style: per_row uniform columns for every row, deduped."""
    rng = np.random.Generator(np.random.PCG64(seed))
    src = np.repeat(np.arange(n, dtype=np.int64), per_row)
    dst = rng.integers(0, n, size=n * per_row, dtype=np.int64)
    return _dedupe(src, dst, n)


def _sorted_keys(major: np.ndarray, minor: np.ndarray, nminor: int) -> np.ndarray:
    key = major.astype(np.int64) * np.int64(nminor) + minor.astype(np.int64)
    key.sort(kind="stable")
    return key


def coo_to_csr(nrows: int, rows: np.ndarray, cols: np.ndarray, vals: np.ndarray, ncols: int | None = None):
    """(rowptr int64[nrows+1], colidx int32, val f32) with columns ascending per row."""
    ncols = int(cols.max()) + 1 if ncols is None and cols.size else (ncols or 1)
    key = rows.astype(np.int64) * np.int64(ncols) + cols.astype(np.int64)
    order = np.argsort(key, kind="stable")
    rowptr = np.zeros(nrows + 1, dtype=np.int64)
    np.cumsum(np.bincount(rows, minlength=nrows), out=rowptr[1:])
    return rowptr, cols[order].astype(np.int32), vals[order].astype(np.float32)


def coo_to_csc(ncols: int, rows: np.ndarray, cols: np.ndarray, vals: np.ndarray, nrows: int | None = None):
    """(colptr int64[ncols+1], rowidx int32, val f32) with rows ascending per column."""
    nrows = int(rows.max()) + 1 if nrows is None and rows.size else (nrows or 1)
    key = cols.astype(np.int64) * np.int64(nrows) + rows.astype(np.int64)
    order = np.argsort(key, kind="stable")
    colptr = np.zeros(ncols + 1, dtype=np.int64)
    np.cumsum(np.bincount(cols, minlength=ncols), out=colptr[1:])
    return colptr, rows[order].astype(np.int32), vals[order].astype(np.float32)


@dataclasses.dataclass
class SparseInputs:
    """C = A x B inputs: A (m x k) as CSC, B (k x n) as CSR, plus the COO they came from."""
    name: str
    m: int
    k: int
    n: int
    a_colptr: np.ndarray
    a_rowidx: np.ndarray
    a_val: np.ndarray
    b_rowptr: np.ndarray
    b_colidx: np.ndarray
    b_val: np.ndarray

    @property
    def nnz_a(self) -> int:
        return int(self.a_rowidx.size)

    @property
    def nnz_b(self) -> int:
        return int(self.b_colidx.size)


# Workloads of BASELINE.json "configs" (index -> recipe).  Shapes follow the paper's
# networks (Table II) and BASELINE.json; the power-law parameters are
# calibrated in DESIGN.md §3.
CONFIGS = {
    "C1": dict(kind="rmat", scale=10, edge_factor=16, a=0.57, b=0.19, c=0.19,
               desc="R-MAT scale-10 (1,024 nodes, edge factor 16, a=0.57) C=AxA fp32"),
    "C2": dict(kind="chunglu", n=916_428, m=5_105_039, gamma_out=2.6, gamma_in=2.0,
               max_out=456, max_in=6_326, sigma=1.5, symmetric=False,
               desc="power-law shaped like web-Google (916K nodes, 5.1M edges) C=AxA"),
    "C3": dict(kind="chunglu", n=1_696_415, m=22_190_596, gamma_out=2.5, gamma_in=2.5,
               max_out=42_000, max_in=42_000, sigma=0.0, symmetric=True,
               desc="hub-heavy power-law shaped like as-Skitter (1.7M nodes, 11M undirected edges, max degree 35K) C=AxA"),
    "C4": dict(kind="er", n=2_000_000, per_row=8,
               desc="low-skew Erdos-Renyi 2Mx2M, 8 nnz/row C=AxA"),
    "C5": dict(kind="chunglu", n=4_847_571, m=68_993_773, gamma_out=2.6, gamma_in=2.6,
               max_out=20_293, max_in=13_906, sigma=2.0, symmetric=False,
               desc="soc-LiveJournal-shaped power-law (4.8M nodes, 69M edges) C=AxA"),
}

# PAPER.md Table III synthetic sets (L739-L779): S (scalability), P (skewness), SP (sparsity) for
# C = A^2 and AB15-AB18 (distinct R-MAT operands A, B; scale 15-18, edge factor 16) for C = AB.
_S = (0.45, 0.15, 0.15)
_U = (0.25, 0.25, 0.25)
for _q, (_n, _m) in enumerate([(250_000, 62_500), (500_000, 250_000), (750_000, 562_500), (1_000_000, 1_000_000)]):
    CONFIGS[f"S{_q + 1}"] = dict(kind="rmat_n", n=_n, m=_m, a=_S[0], b=_S[1], c=_S[2],
                                 desc=f"Table III s{_q + 1}: R-MAT {_n} nodes, {_m} elements, (0.45,0.15,0.15,0.25) C=AxA")
for _q, _p in enumerate([(0.25, 0.25, 0.25), (0.45, 0.15, 0.15), (0.55, 0.15, 0.15), (0.57, 0.19, 0.19)]):
    CONFIGS[f"P{_q + 1}"] = dict(kind="rmat_n", n=1_000_000, m=1_000_000, a=_p[0], b=_p[1], c=_p[2],
                                 desc=f"Table III p{_q + 1}: R-MAT 1M nodes, 1M elements, {_p + (round(1 - sum(_p), 2),)} C=AxA")
for _q, _m in enumerate([4_000_000, 3_000_000, 2_000_000, 1_000_000]):
    CONFIGS[f"SP{_q + 1}"] = dict(kind="rmat_n", n=1_000_000, m=_m, a=_U[0], b=_U[1], c=_U[2],
                                  desc=f"Table III sp{_q + 1}: R-MAT 1M nodes, {_m} elements, uniform C=AxA")
for _sc in (15, 16, 17, 18):
    CONFIGS[f"AB{_sc}"] = dict(kind="rmat_ab", scale=_sc, edge_factor=16, a=0.57, b=0.19, c=0.19,
                               desc=f"Table III C=AB: distinct R-MAT A, B (scale {_sc}, edge factor 16)")


def make_inputs(name: str, seed: int = 1, values: str = "real", **override) -> SparseInputs:
    """Build the seeded C = A x A inputs of config ``name`` (A = B, both layouts)."""
    cfg = dict(CONFIGS[name])
    cfg.update(override)
    kind = cfg["kind"]
    if kind == "rmat":
        n = 1 << cfg["scale"]
        src, dst = rmat_edges(cfg["scale"], cfg["edge_factor"], cfg["a"], cfg["b"], cfg["c"], seed)
    elif kind == "chunglu":
        n = cfg["n"]
        src, dst = chung_lu_edges(n, cfg["m"], cfg["gamma_out"], cfg["gamma_in"], cfg["max_out"],
                                  cfg["max_in"], cfg["sigma"], seed, cfg.get("symmetric", False))
    elif kind == "rmat_n":
        n = cfg["n"]
        src, dst = rmat_n_edges(n, cfg["m"], cfg["a"], cfg["b"], cfg["c"], seed)
    elif kind == "rmat_ab":   # C = A B with two independent R-MAT operands
        n = 1 << cfg["scale"]
        ar, ac = rmat_edges(cfg["scale"], cfg["edge_factor"], cfg["a"], cfg["b"], cfg["c"], seed)
        br, bc = rmat_edges(cfg["scale"], cfg["edge_factor"], cfg["a"], cfg["b"], cfg["c"], seed + 1000)
        return _pack(name, n, n, n, ar.astype(np.int32), ac.astype(np.int32), edge_values(ar, ac, seed, values),
                     br.astype(np.int32), bc.astype(np.int32), edge_values(br, bc, seed + 1000, values))
    elif kind == "er":
        n = cfg["n"]
        src, dst = er_edges(n, cfg["per_row"], seed)
    else:
        raise ValueError(kind)
    return _pack_square(name, n, src, dst, seed, values)


def _pack_square(name, n, src, dst, seed, values) -> SparseInputs:
    """A = B = adjacency(src -> dst), values hashed from (row, col): no permutation needed."""
    # B (CSR): (src, dst) come back from _dedupe sorted by (src, dst)
    b_rowptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(src, minlength=n), out=b_rowptr[1:])
    b_colidx = dst.astype(np.int32)
    b_val = edge_values(src, dst, seed, values)
    # A (CSC): sort by (dst, src)
    key = _sorted_keys(dst, src, n)
    a_rowidx = (key % n).astype(np.int32)
    a_cols = (key // n).astype(np.int32)
    a_colptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(a_cols, minlength=n), out=a_colptr[1:])
    a_val = edge_values(a_rowidx, a_cols, seed, values)
    return SparseInputs(name, n, n, n, a_colptr, a_rowidx, a_val, b_rowptr, b_colidx, b_val)


def _pack(name, m, k, n, ar, ac, av, br, bc, bv) -> SparseInputs:
    a_colptr, a_rowidx, a_val = coo_to_csc(k, ar, ac, av, nrows=m)
    b_rowptr, b_colidx, b_val = coo_to_csr(k, br, bc, bv, ncols=n)
    return SparseInputs(name, m, k, n, a_colptr, a_rowidx, a_val, b_rowptr, b_colidx, b_val)


def random_tiny(m: int, k: int, n: int, density_a: float, density_b: float, seed: int,
                values: str = "real", skew: bool = False) -> SparseInputs:
    """Small random C = A x B (A != B) for brute-force tests; ``skew`` adds hub rows/cols."""
    rng = np.random.Generator(np.random.PCG64(seed))

    def draw(r, c, d):
        mask = rng.random((r, c)) < d
        if skew and r > 2 and c > 2:
            mask[rng.integers(0, r), :] |= rng.random(c) < 0.9
            mask[:, rng.integers(0, c)] |= rng.random(r) < 0.9
        rr, cc = np.nonzero(mask)
        return rr.astype(np.int32), cc.astype(np.int32)

    ar, ac = draw(m, k, density_a)
    br, bc = draw(k, n, density_b)
    av = edge_values(ar, ac, seed, values)
    bv = edge_values(br, bc, seed + 7919, values)
    return _pack(f"tiny{m}x{k}x{n}", m, k, n, ar, ac, av, br, bc, bv)


def from_coo(name, m, k, n, a_coo, b_coo) -> SparseInputs:
    """Inputs from explicit COO triples ((rows, cols, vals) for A and for B)."""
    ar, ac, av = (np.asarray(x) for x in a_coo)
    br, bc, bv = (np.asarray(x) for x in b_coo)
    return _pack(name, m, k, n, ar.astype(np.int32), ac.astype(np.int32), av.astype(np.float32),
                 br.astype(np.int32), bc.astype(np.int32), bv.astype(np.float32))


def row_slice_coo(inp: SparseInputs, r0: int, r1: int) -> SparseInputs:
    """Rows [r0, r1) of A (renumbered from 0) with the same B: one rank's / chunk's share."""
    cols = np.repeat(np.arange(inp.k, dtype=np.int32), np.diff(inp.a_colptr))
    keep = (inp.a_rowidx >= r0) & (inp.a_rowidx < r1)
    ar = (inp.a_rowidx[keep] - r0).astype(np.int32)
    ac = cols[keep]
    av = inp.a_val[keep]
    a_colptr, a_rowidx, a_val = coo_to_csc(inp.k, ar, ac, av, nrows=max(r1 - r0, 1))
    return SparseInputs(f"{inp.name}[{r0}:{r1}]", r1 - r0, inp.k, inp.n, a_colptr, a_rowidx, a_val,
                        inp.b_rowptr, inp.b_colidx, inp.b_val)
