"""CPU pins of the oracle (oracle/) against things other than itself:
hand-worked examples and the paper's printed figures (tests/golden/), dense brute
force, an independent library product (scipy.sparse), closed forms, invariants and
special cases.  Each pin is chosen so that a plausible slip in the oracle (dropped
term, wrong index, transposed operand, lost computed zero) fails at least one."""
import numpy as np
import pytest
import scipy.sparse as sp

import oracle
import synth
from oracle import stages
from golden_io import read_kv, read_triples


def _inputs_from_golden(name):
    sec, sc = read_triples(name)
    ar, ac, av = sec["A"]
    br, bc, bv = sec["B"]
    m = int(max(ar.max(), sec["C"][0].max() if "C" in sec else 0)) + 1
    m = max(m, len(sc.get("rowwork", [])))
    k = len(sc["work"])
    n = int(max(bc.max(), sec["C"][1].max())) + 1
    return synth.from_coo(name, m, k, n, (ar, ac, av), (br, bc, bv)), sec, sc


def _dense(inp):
    A = np.zeros((inp.m, inp.k))
    cols = np.repeat(np.arange(inp.k), np.diff(inp.a_colptr))
    A[inp.a_rowidx, cols] = inp.a_val
    B = np.zeros((inp.k, inp.n))
    rows = np.repeat(np.arange(inp.k), np.diff(inp.b_rowptr))
    B[rows, inp.b_colidx] = inp.b_val
    Ap = np.zeros((inp.m, inp.k), dtype=np.int64)
    Ap[inp.a_rowidx, cols] = 1
    Bp = np.zeros((inp.k, inp.n), dtype=np.int64)
    Bp[rows, inp.b_colidx] = 1
    return A, B, Ap, Bp


def _to_dense_c(m, n, rowptr, col, val):
    C = np.zeros((m, n))
    S = np.zeros((m, n), dtype=bool)
    r = np.repeat(np.arange(m), np.diff(rowptr))
    C[r, col] = val
    S[r, col] = True
    return C, S


# ---------------------------------------------------------------- golden (hand / paper) ---

@pytest.mark.parametrize("name", ["hand_example_4x4.txt", "cancellation_1x2x1.txt"])
def test_hand_examples(name):
    inp, sec, sc = _inputs_from_golden(name)
    rowptr, col, val = oracle.gustavson(inp)
    cr, cc, cv = sec["C"]
    exp_rowptr = np.zeros(inp.m + 1, dtype=np.int64)
    np.cumsum(np.bincount(cr, minlength=inp.m), out=exp_rowptr[1:])
    np.testing.assert_array_equal(rowptr, exp_rowptr)
    np.testing.assert_array_equal(col, cc)
    np.testing.assert_array_equal(val, cv)          # exact: small integers
    ca, rb, work = stages.pair_workload(inp)
    np.testing.assert_array_equal(work, sc["work"])
    np.testing.assert_array_equal(stages.row_workload(inp), sc["rowwork"])
    assert int(work.sum()) == sc["products"][0]
    r, c, v = stages.expand_outer(inp)
    assert r.size == sc["products"][0]
    m_rowptr, m_col, m_val = stages.merge(inp.m, r, c, v)
    np.testing.assert_array_equal(m_rowptr, exp_rowptr)
    np.testing.assert_array_equal(m_col, cc)
    np.testing.assert_array_equal(m_val, cv)


def test_fig4_merge():
    kv = {r[0]: [float(x) for x in r[1:]] for r in read_kv("fig4_merge.txt")}
    cols = np.array(kv["cols"], dtype=np.int64)
    vals = np.array(kv["vals"])
    rowptr, mc, mv = stages.merge(1, np.zeros(cols.size, np.int64), cols, vals)
    np.testing.assert_array_equal(mc, kv["merged_cols"])
    np.testing.assert_array_equal(mv, kv["merged_vals"])
    assert rowptr.tolist() == [0, 4]


def test_fig4_classification():
    rows = read_kv("fig4_classification.txt")
    pairs = [tuple(int(x) for x in r[1:]) for r in rows if r[0] == "pair"]
    kv = {r[0]: [int(x) for x in r[1:]] for r in rows if r[0] != "pair" and r[0] != "rowwork"}
    thr = kv["threshold"][0]
    idx = np.array([p[0] for p in pairs])
    ca = np.array([p[1] for p in pairs], dtype=np.int64)
    rb = np.array([p[2] for p in pairs], dtype=np.int64)
    work = ca * rb
    assert dict(zip(idx.tolist(), work.tolist())) == {0: 27, 2: 18863, 3: 22751, 7: 19, 11: 371, 13: 9}
    cls = stages.classify_pairs(ca, rb, work, t_dom=thr, split_ca_max=1 << 30)
    assert sorted(idx[cls == stages.DOMINATOR].tolist()) == kv["dominators"]
    assert sorted(idx[cls == stages.NORMAL].tolist()) == kv["normal"]
    assert sorted(idx[cls == stages.LOW].tolist()) == kv["low"]
    rw = {int(r[1]): int(r[2]) for r in rows if r[0] == "rowwork"}
    ridx = np.array(sorted(rw))
    bins = stages.row_bins(np.array([rw[i] for i in ridx], dtype=np.int64), t_lim=thr)
    assert ridx[bins == stages.ROW_LIMITED].tolist() == kv["limiting"]
    assert ridx[bins != stages.ROW_LIMITED].tolist() == kv["nonlimiting"]


def test_fig5_split_and_fig6_gather():
    rows = read_kv("fig5_fig6_reorganizer.txt")
    for r in rows:
        kv = dict(x.split("=") for x in r[1:])
        if r[0] == "split":
            ca, rb, f = int(kv["ca"]), int(kv["rb"]), int(kv["factor"])
            inp = synth.from_coo("fig5", ca, 1, rb,
                                 (np.arange(ca), np.zeros(ca, int), np.ones(ca)),
                                 (np.zeros(rb, int), np.arange(rb), np.ones(rb)))
            _, _, work = stages.pair_workload(inp)
            comps = [int(x) for x in kv["computations"].split(",")]
            # piece budget = the largest piece in the figure; factor must come out as 2^2
            assert stages.splitting_factor(ca, rb, piece_work=max(comps), split_ca_max=1 << 30) == f
            cls = np.array([stages.DOMINATOR], dtype=np.int8)
            pieces = stages.split_pieces(inp, cls, piece_work=max(comps), b_tile=1 << 30,
                                         split_ca_max=1 << 30)
            sizes = (pieces[:, 2] - pieces[:, 1]).tolist()
            assert sizes == [int(x) for x in kv["pieces"].split(",")]
            assert ((pieces[:, 2] - pieces[:, 1]) * (pieces[:, 4] - pieces[:, 3])).tolist() == comps
            assert sum(comps) == int(work[0]) == 25
        elif r[0] == "gather":
            assert stages.gathering_factor(int(kv["t"]), int(kv["block"])) == int(kv["factor"])


# ---------------------------------------------------------------- brute force ------------

@pytest.mark.parametrize("shape,dens,seed,skew,values", [
    ((1, 1, 1), (1.0, 1.0), 1, False, "real"),
    ((7, 5, 9), (0.3, 0.4), 2, False, "real"),
    ((16, 16, 16), (0.2, 0.2), 3, True, "real"),
    ((33, 20, 41), (0.1, 0.15), 4, True, "signed"),
    ((40, 64, 40), (0.05, 0.5), 5, False, "int"),
    ((20, 3, 30), (0.0, 0.5), 6, False, "real"),      # A empty
    ((25, 30, 12), (0.3, 0.0), 7, False, "real"),     # B empty
    ((64, 1, 64), (0.5, 0.5), 8, False, "real"),      # rank-1 outer product
])
def test_bruteforce_dense(shape, dens, seed, skew, values):
    m, k, n = shape
    inp = synth.random_tiny(m, k, n, dens[0], dens[1], seed, values=values, skew=skew)
    A, B, Ap, Bp = _dense(inp)
    rowptr, col, val = oracle.gustavson(inp)
    C, S = _to_dense_c(m, n, rowptr, col, val)
    np.testing.assert_array_equal(S, (Ap @ Bp) > 0)       # structure incl. computed zeros
    np.testing.assert_allclose(C, A @ B, rtol=1e-12, atol=1e-12)
    for i in range(m):                                     # canonical: ascending columns
        assert np.all(np.diff(col[rowptr[i]:rowptr[i + 1]]) > 0)
    # workload definitions against the dense pattern product
    ca, rb, work = stages.pair_workload(inp)
    np.testing.assert_array_equal(stages.row_workload(inp), (Ap @ Bp).sum(axis=1))
    assert int(work.sum()) == int((Ap @ Bp).sum())
    np.testing.assert_array_equal(work, Ap.sum(axis=0) * Bp.sum(axis=1))
    # Eq. (2) expansion + merge reaches the same C as Eq. (1)
    r, c, v = stages.expand_outer(inp)
    mr, mc, mv = stages.merge(m, r, c, v)
    np.testing.assert_array_equal(mr, rowptr)
    np.testing.assert_array_equal(mc, col)
    np.testing.assert_allclose(mv, val, rtol=1e-12, atol=1e-12)


def test_subset_rows_match_full():
    inp = synth.make_inputs("C1", seed=3)
    rowptr, col, val = oracle.gustavson(inp)
    rows = np.array([5, 0, 1023, 17, 17, 400], dtype=np.int32)
    sr, sc, sv = oracle.gustavson(inp, rows=rows)
    for t, i in enumerate(rows):
        np.testing.assert_array_equal(sc[sr[t]:sr[t + 1]], col[rowptr[i]:rowptr[i + 1]])
        np.testing.assert_array_equal(sv[sr[t]:sr[t + 1]], val[rowptr[i]:rowptr[i + 1]])


# ---------------------------------------------------------------- library / invariants ----

def _scipy(inp):
    cols = np.repeat(np.arange(inp.k), np.diff(inp.a_colptr))
    A = sp.csr_matrix((inp.a_val.astype(np.float64), (inp.a_rowidx, cols)), shape=(inp.m, inp.k))
    B = sp.csr_matrix((inp.b_val.astype(np.float64), (np.repeat(np.arange(inp.k), np.diff(inp.b_rowptr)),
                                                      inp.b_colidx)), shape=(inp.k, inp.n))
    return A, B


@pytest.mark.parametrize("seed", [1, 2])
def test_c1_against_scipy_and_invariants(seed):
    inp = synth.make_inputs("C1", seed=seed)
    rowptr, col, val = oracle.gustavson(inp)
    A, B = _scipy(inp)
    C = (A @ B).tocsr()
    C.sort_indices()
    # values are positive, so scipy dropping exact zeros cannot hide a structural difference
    np.testing.assert_array_equal(rowptr, C.indptr)
    np.testing.assert_array_equal(col, C.indices)
    np.testing.assert_allclose(val, C.data, rtol=1e-13)
    # C 1 = A (B 1)
    ones = np.ones(inp.n)
    lhs = np.bincount(np.repeat(np.arange(inp.m), np.diff(rowptr)), weights=val, minlength=inp.m)
    rhs = A @ (B @ ones)
    np.testing.assert_allclose(lhs, rhs, rtol=1e-12)
    # #products two ways
    ca, rb, work = stages.pair_workload(inp)
    assert int(work.sum()) == int(stages.row_workload(inp).sum())


def test_transpose_identity():
    """(A B)^T = B^T A^T: the oracle run on the transposed operands gives C^T."""
    inp = synth.random_tiny(37, 23, 29, 0.2, 0.25, seed=11, skew=True)
    rowptr, col, val = oracle.gustavson(inp)
    # B^T (n x k) as CSC == B as CSR; A^T (k x m) as CSR == A as CSC
    t = synth.SparseInputs("T", inp.n, inp.k, inp.m, inp.b_rowptr, inp.b_colidx, inp.b_val,
                           inp.a_colptr, inp.a_rowidx, inp.a_val)
    tr, tc, tv = oracle.gustavson(t)
    C, S = _to_dense_c(inp.m, inp.n, rowptr, col, val)
    CT, ST = _to_dense_c(inp.n, inp.m, tr, tc, tv)
    np.testing.assert_array_equal(S, ST.T)
    np.testing.assert_allclose(C, CT.T, rtol=1e-12)


def test_integer_values_exact():
    inp = synth.make_inputs("C1", seed=5, values="int")
    rowptr, col, val = oracle.gustavson(inp)
    A, B = _scipy(inp)
    C = (A @ B).tocsr()
    C.sort_indices()
    np.testing.assert_array_equal(col, C.indices)
    np.testing.assert_array_equal(val, C.data)              # integer sums are exact
    assert np.all(val == np.round(val))


def test_identity_special_case():
    inp0 = synth.make_inputs("C1", seed=2)
    n = inp0.n
    eye = (np.arange(n), np.arange(n), np.ones(n))
    cols = np.repeat(np.arange(n), np.diff(inp0.a_colptr))
    inp = synth.from_coo("AI", n, n, n, (inp0.a_rowidx, cols, inp0.a_val), eye)
    rowptr, col, val = oracle.gustavson(inp)
    A, _ = _scipy(inp)
    A = A.tocsr()
    A.sort_indices()
    np.testing.assert_array_equal(rowptr, A.indptr)
    np.testing.assert_array_equal(col, A.indices)
    np.testing.assert_array_equal(val, A.data)


# ---------------------------------------------------------------- reorganizer definitions -

@pytest.mark.parametrize("piece_work,b_tile,ca_max", [(64, 1 << 30, 1 << 30), (500, 37, 8), (1, 1, 1)])
def test_pieces_tile_dominators_exactly(piece_work, b_tile, ca_max):
    inp = synth.make_inputs("C1", seed=4)
    ca, rb, work = stages.pair_workload(inp)
    t = stages.dominator_threshold(int(work.sum()), int((work > 0).sum()), 0.0, 148, 4, 2000, 16384)
    cls = stages.classify_pairs(ca, rb, work, t, ca_max)
    pieces = stages.split_pieces(inp, cls, piece_work, b_tile, ca_max)
    doms = np.nonzero(cls == stages.DOMINATOR)[0]
    assert doms.size > 0
    for k in doms:
        pk = pieces[pieces[:, 0] == k]
        cover = np.zeros((ca[k], rb[k]), dtype=np.int64)
        for _, a0, a1, b0, b1 in pk:
            cover[a0 - inp.a_colptr[k]:a1 - inp.a_colptr[k], b0 - inp.b_rowptr[k]:b1 - inp.b_rowptr[k]] += 1
            assert (a1 - a0) <= ca_max or (a1 - a0) == 1
        assert np.all(cover == 1)
        f = stages.splitting_factor(int(ca[k]), int(min(rb[k], b_tile)), piece_work, ca_max)
        assert f & (f - 1) == 0                               # 2^n (L410-L413 L)
    # order: ascending k, then B tile, then A piece
    keys = pieces[:, [0, 3, 1]]
    assert np.all(np.lexsort(keys[:, ::-1].T) == np.arange(len(keys)))


def test_gather_lists_partition_low_performers():
    inp = synth.make_inputs("C1", seed=4)
    ca, rb, work = stages.pair_workload(inp)
    cls = stages.classify_pairs(ca, rb, work, 10 ** 9, 10 ** 9)
    lists = stages.gather_lists(ca, rb, cls)
    allk = np.concatenate([lists[b] for b in range(6)])
    assert sorted(allk.tolist()) == np.nonzero(cls == stages.LOW)[0].tolist()
    for b, ks in lists.items():
        assert np.all((rb[ks] > (1 << b) // 2) & (rb[ks] <= (1 << b)))
        assert all(stages.gathering_factor(int(t)) == 32 >> b for t in rb[ks])


def test_balanced_row_partition():
    inp = synth.make_inputs("C1", seed=1)
    rw = stages.row_workload(inp)
    for parts in (1, 2, 3, 8):
        b = stages.balanced_row_partition(rw, parts)
        assert b[0] == 0 and b[-1] == inp.m and np.all(np.diff(b) >= 0) and b.size == parts + 1
        shares = np.array([rw[b[p]:b[p + 1]].sum() for p in range(parts)])
        assert shares.sum() == rw.sum()
        assert shares.max() - shares.min() <= 2 * rw.max()


def test_thresholds_formulas():
    # paper form: nnz(Ĉ)/(#blocks × α)  (L309-L311 R),  nnz(Ĉ)/(#blocks × β) with β = 10 (L475-L477 L)
    assert stages.dominator_threshold(1000, 10, 2.0, 148, 4, 0, 16384) == 50
    assert stages.dominator_threshold(10 ** 7, 10, 0.0, 148, 4, 0, 10 ** 9) == -(-10 ** 7 // 592)
    assert stages.dominator_threshold(10 ** 9, 10, 0.0, 148, 4, 0, 16384) == 16384      # clamped to a piece
    assert stages.dominator_threshold(10 ** 3, 10, 0.0, 148, 4, 4096, 16384) == 4096    # floor
    assert stages.limiting_threshold(100000, 100, 10.0, 4096) == 100
    assert stages.limiting_threshold(10 ** 9, 100, 10.0, 4096) == 4096
    assert stages.limiting_threshold(10 ** 9, 100, 0.0, 4096) == 4096


def test_chat_row_offsets_hand_example():
    """Ĉ row offsets = exclusive scan of the row-wise nnz (L289-L291 R), pinned by the hand example's
    rowwork 4 2 3 0 -> offsets 0 4 6 9 9 (tests/golden/hand_example_4x4.txt)."""
    inp, sec, sc = _inputs_from_golden("hand_example_4x4.txt")
    np.testing.assert_array_equal(stages.chat_row_offsets(stages.row_workload(inp)), sc["rowoff"])
    np.testing.assert_array_equal(stages.chat_row_offsets(np.zeros(0, np.int64)), [0])


def test_gather_order_hand_list():
    """R5 packing order of the B-Gathering lists against a hand-derived list
    (tests/golden/r5_gather_order.txt): bins by 2^(n-1) < t <= 2^n, inside a bin by
    floor(log2 nnz(a_*k)) then k -- a plain k order or a swapped key fails it."""
    kv = {r[0]: [int(x) for x in r[1:]] for r in read_kv("r5_gather_order.txt")}
    ca = np.array(kv["ca"], dtype=np.int64)
    rb = np.array(kv["rb"], dtype=np.int64)
    work = ca * rb
    cls = stages.classify_pairs(ca, rb, work, t_dom=10 ** 9, split_ca_max=10 ** 9)
    assert list(np.nonzero(cls == stages.LOW)[0]) == [0, 1, 2, 3, 4, 6, 8, 9, 10]
    assert cls[5] == stages.NORMAL and cls[7] == stages.EMPTY
    lists = stages.gather_lists(ca, rb, cls)
    for b in range(6):
        np.testing.assert_array_equal(lists[b], kv[f"bin{b}"])


@pytest.mark.parametrize("fixed_f,chunks", [(1, [5]), (2, [3, 2]), (4, [2, 2, 1]), (64, [1, 1, 1, 1, 1])])
def test_fixed_splitting_factor_fig5_block(fixed_f, chunks):
    """Fig. 11's sweep imposes the splitting factor 2^n (L640-L687 L): the Fig. 5 block (5 column
    entries x 5 row entries, L386-L388 L) split by f gives greedy chunks of ceil(5/f) entries; f is
    capped at the column's next power of two (8 -> one entry per piece)."""
    inp = synth.from_coo("fig5", 5, 1, 5, (np.arange(5), np.zeros(5, int), np.ones(5, np.float32)),
                         (np.zeros(5, int), np.arange(5), np.ones(5, np.float32)))
    ca, rb, work = stages.pair_workload(inp)
    cls = np.array([stages.DOMINATOR], dtype=np.int8)
    pcs = stages.split_pieces(inp, cls, piece_work=10 ** 9, b_tile=4096, split_ca_max=10 ** 9, fixed_f=fixed_f)
    assert [int(p[2] - p[1]) for p in pcs] == chunks
    assert int(sum((p[2] - p[1]) * (p[4] - p[3]) for p in pcs)) == 25
