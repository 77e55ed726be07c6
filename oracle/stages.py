"""ORACLE -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Step-by-step definitions of the Block Reorganizer stages, in the paper's order
and notation (§IV).  Plain numpy; no blocking, fusion or
reordering beyond what each definition states.  Where the paper is silent,
garbled or designed for a Titan Xp, the reading taken is the one listed in
DESIGN.md §2 ("Readings"), cited here as R<n>.

Notation: pair k = (a_*k, b_k*) = (column k of A, row k of B); its block has
nnz(b_k*) effective threads (L385-L386 R) and nnz(a_*k) computations per thread
(L411-L413 L); the intermediate matrix is Ĉ (L321-L323 L).
"""
from __future__ import annotations

import math

import numpy as np

WARP = 32                     # warp size (L127-L130 L; "32 (size of warps)" L317-L318 R)

# pair classes (L304-L318 R, Fig. 4)
EMPTY, DOMINATOR, NORMAL, LOW = 0, 1, 2, 3
# row classes of the merge (Fig. 4 "Limiting bin / Non-limiting bin", L474-L477 L; R6)
ROW_EMPTY, ROW_WARP, ROW_CTA, ROW_LIMITED = 0, 1, 2, 3


# --- (1) precalculation: block-wise and row-wise nnz(Ĉ)  (L326-L330 L, L289-L291 R) -----------

def pair_workload(inp):
    """ca[k] = nnz(a_*k), rb[k] = nnz(b_k*), work[k] = ca[k]*rb[k] (block-wise nnz of Ĉ)."""
    ca = np.diff(inp.a_colptr).astype(np.int64)
    rb = np.diff(inp.b_rowptr).astype(np.int64)
    return ca, rb, ca * rb


def row_workload(inp):
    """rowwork[i] = sum over stored a_ik of nnz(b_k*)  (row-wise nnz of Ĉ)."""
    ca, rb, _ = pair_workload(inp)
    rowwork = np.zeros(inp.m, dtype=np.int64)
    col_of_entry = np.repeat(np.arange(inp.k, dtype=np.int64), ca)
    np.add.at(rowwork, inp.a_rowidx.astype(np.int64), rb[col_of_entry])
    return rowwork


def chat_row_offsets(rowwork):
    """Exclusive scan of the row-wise nnz: where each row of Ĉ starts ("relocate the
    outer-product's elements with same row closer together", L289-L291 R)."""
    off = np.zeros(rowwork.size + 1, dtype=np.int64)
    np.cumsum(rowwork, out=off[1:])
    return off


# --- (2) categorisation (L304-L318 R) ------------------------------------------------------

def dominator_threshold(nnz_chat: int, k_nonempty: int, alpha: float, num_sms: int,
                        dom_waves: int, dom_min_work: int, piece_work: int) -> int:
    """threshold = nnz(Ĉ)/(#blocks × α)  (L309-L311 R) when α > 0, with #blocks the number
    of non-empty pair blocks (R1).  α = 0 selects the B200 re-derivation (R2): a block is
    overloaded when it exceeds the per-SM fair share ceil(nnz(Ĉ)/(#SMs × dom_waves)), clamped
    to [dom_min_work, piece_work] so that no unsplit block is larger than a split piece."""
    if alpha > 0:
        return int(math.floor(float(nnz_chat) / (float(max(k_nonempty, 1)) * alpha)))
    share = -(-int(nnz_chat) // int(num_sms * dom_waves))
    return int(min(piece_work, max(dom_min_work, share)))


def classify_pairs(ca, rb, work, t_dom: int, split_ca_max: int):
    """EMPTY if the block has no work; DOMINATOR if its block-wise nnz exceeds the
    threshold (L309-L311 R) or its per-thread computation count nnz(a_*k) exceeds
    split_ca_max (R3); LOW performer if it has < 32 effective threads (L317-L318 R);
    NORMAL otherwise."""
    cls = np.full(ca.size, NORMAL, dtype=np.int8)
    cls[rb < WARP] = LOW
    cls[(work > t_dom) | (ca > split_ca_max)] = DOMINATOR
    cls[work == 0] = EMPTY
    return cls


# --- (3) B-Splitting (L320-L415, Fig. 5) ----------------------------------------------------

def splitting_factor(ca: int, blen: int, piece_work: int, split_ca_max: int, fixed_f: int = 0) -> int:
    """Smallest power of two f (L410-L413 L: "splitting factor (2^n)") such that each
    greedy piece of the column, ceil(ca/f) entries, stays within piece_work products
    and split_ca_max computations per thread; f never exceeds the column length's
    next power of two (one entry per piece).  fixed_f > 0 (Fig. 11's sweep over the
    splitting factor, L640-L687 L) imposes the factor, with the same cap."""
    if fixed_f > 0:
        f = 1
        while f < fixed_f and f < ca:
            f *= 2
        return f
    f = 1
    while f < ca:
        chunk = -(-ca // f)
        if chunk * blen <= piece_work and chunk <= split_ca_max:
            break
        f *= 2
    return f


def split_pieces(inp, cls, piece_work: int, b_tile: int, split_ca_max: int, fixed_f: int = 0):
    """Pieces (k, a_lo, a_hi, b_lo, b_hi) (absolute entry ranges into A's rowidx and
    B's colidx) for every dominator, in order of ascending k, then B tile, then A piece.
    The A column is split greedily: piece p takes entries [p*chunk, (p+1)*chunk)
    ("several elements from each column vector are shifted to the next vector
    sequentially", L374-L376 L); empty trailing pieces are not emitted (Fig. 5: a
    25-computation block split into three blocks, L386-L388 L).  The B row is cut
    into tiles of b_tile entries (rounded up to a multiple of 8) only when it exceeds
    b_tile (R4, R16)."""
    b_tile = -(-b_tile // 8) * 8   # R4 / R16: a tile is whole 32-byte sectors (8 slots) of the run
    out = []
    for k in np.nonzero(cls == DOMINATOR)[0]:
        a0, a1 = int(inp.a_colptr[k]), int(inp.a_colptr[k + 1])
        b0, b1 = int(inp.b_rowptr[k]), int(inp.b_rowptr[k + 1])
        ca, rb = a1 - a0, b1 - b0
        blen = min(rb, b_tile)
        f = splitting_factor(ca, blen, piece_work, split_ca_max, fixed_f)
        chunk = -(-ca // f)
        for bs in range(b0, b1, b_tile):
            be = min(b1, bs + b_tile)
            for p in range(f):
                lo = p * chunk
                if lo >= ca:
                    break
                out.append((int(k), a0 + lo, a0 + min(ca, lo + chunk), bs, be))
    return np.array(out, dtype=np.int64).reshape(-1, 5)


def normal_pieces(inp, cls):
    """A normal pair is one block: piece (k, whole column, whole row), ascending k."""
    ks = np.nonzero(cls == NORMAL)[0]
    return np.stack([ks, inp.a_colptr[ks], inp.a_colptr[ks + 1], inp.b_rowptr[ks],
                     inp.b_rowptr[ks + 1]], axis=1).astype(np.int64).reshape(-1, 5)


# --- (4) B-Gathering (L369-L450, Fig. 6) ----------------------------------------------------

def gather_bin(t: int) -> int:
    """Bin n with 2^(n-1) < t <= 2^n (t = effective threads = nnz(b_k*) >= 1), L438-L439 L."""
    return int(math.ceil(math.log2(t))) if t > 1 else 0


def gathering_factor(t: int, block: int = WARP) -> int:
    """block / 2^n micro-blocks per combined block (L438-L441 L: t=2 -> 16 for block 32)."""
    return block // (1 << gather_bin(t))


def gather_lists(ca, rb, cls):
    """Per bin n (0..5), the low-performer pairs in the order they are packed into
    combined blocks: ascending (n, c, k) with c = min(15, floor(log2 nnz(a_*k))) so that
    the micro-blocks of one warp have similar per-thread loop lengths (R5)."""
    ks = np.nonzero(cls == LOW)[0]
    n = np.array([gather_bin(int(t)) for t in rb[ks]], dtype=np.int64)
    c = np.minimum(15, np.floor(np.log2(np.maximum(ca[ks], 1))).astype(np.int64))
    order = np.lexsort((ks, c, n))
    ks, n = ks[order], n[order]
    return {b: ks[n == b].astype(np.int64) for b in range(6)}


# --- (5) B-Limiting bins of the merge (L452-L477 L, Fig. 7) -------------------------------

def limiting_threshold(nnz_chat: int, m_nonempty: int, beta: float, cta_cap: int) -> int:
    """threshold = nnz(Ĉ)/(#blocks × β) (L475-L477 L) when β > 0, clamped to the
    non-limited merge block's capacity; β = 0 selects the B200 default = capacity (R6)."""
    if beta > 0:
        return int(min(cta_cap, math.floor(float(nnz_chat) / (float(max(m_nonempty, 1)) * beta))))
    return int(cta_cap)


def row_bins(rowwork, t_lim: int):
    b = np.full(rowwork.size, ROW_CTA, dtype=np.int8)
    b[rowwork <= WARP] = ROW_WARP
    b[rowwork > t_lim] = ROW_LIMITED
    b[rowwork == 0] = ROW_EMPTY
    return b


# --- (6) expansion: Ĉ by the outer product (reconstructed Eq. (2)) --------------

def expand_outer(inp):
    """All products (i, j, a_ik*b_kj) of C = sum_k a_*k ⊗ b_k*, pair by pair (k ascending),
    values in fp64 (the product of two fp32 values is exact in fp64)."""
    ca, rb, work = pair_workload(inp)
    rows, cols, vals = [], [], []
    for k in np.nonzero(work)[0]:
        a0, a1 = inp.a_colptr[k], inp.a_colptr[k + 1]
        b0, b1 = inp.b_rowptr[k], inp.b_rowptr[k + 1]
        ai = inp.a_rowidx[a0:a1].astype(np.int64)
        av = inp.a_val[a0:a1].astype(np.float64)
        bj = inp.b_colidx[b0:b1].astype(np.int64)
        bv = inp.b_val[b0:b1].astype(np.float64)
        rows.append(np.repeat(ai, bj.size))
        cols.append(np.tile(bj, ai.size))
        vals.append(np.outer(av, bv).ravel())
    if not rows:
        z = np.zeros(0, dtype=np.int64)
        return z, z.copy(), np.zeros(0)
    return np.concatenate(rows), np.concatenate(cols), np.concatenate(vals)


# --- (7) merge: sort + segmented reduce (L452-L455 L) ---------------------------------------

def merge(m: int, rows, cols, vals):
    """Elements of Ĉ with the same (row, col) are merged into one (L453-L455 L):
    sort by (row, col), then sum each equal-key segment in fp64.  Returns CSR."""
    order = np.lexsort((cols, rows))
    r, c, v = rows[order], cols[order], vals[order]
    if r.size == 0:
        return np.zeros(m + 1, dtype=np.int64), np.zeros(0, np.int32), np.zeros(0)
    head = np.ones(r.size, dtype=bool)
    head[1:] = (r[1:] != r[:-1]) | (c[1:] != c[:-1])
    seg = np.cumsum(head) - 1
    out_v = np.zeros(int(seg[-1]) + 1)
    np.add.at(out_v, seg, v)
    out_r, out_c = r[head], c[head]
    rowptr = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(np.bincount(out_r, minlength=m), out=rowptr[1:])
    return rowptr, out_c.astype(np.int32), out_v


# --- row partition for chunked expansion and multi-GPU (R8) ---------------------------------

def balanced_row_partition(rowwork, parts: int):
    """Boundaries r_0 = 0 <= ... <= r_P = m with r_p the first row whose Ĉ prefix reaches
    floor(p * nnz(Ĉ) / P): equal shares of intermediate products per part."""
    prefix = np.zeros(rowwork.size + 1, dtype=np.int64)
    np.cumsum(rowwork, out=prefix[1:])
    total = int(prefix[-1])
    b = [0]
    for p in range(1, parts):
        target = (p * total) // parts
        b.append(max(b[-1], int(np.searchsorted(prefix, target, side="left"))))
    b.append(rowwork.size)
    return np.array(b, dtype=np.int64)

