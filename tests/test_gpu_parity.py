"""GPU parity: every stage of the CUDA path, called through the C-ABI, against the oracle on
the same seeded inputs.  Integer / index work is compared bit-exactly; C values within the
north-star tolerance (relative 1e-5 per entry vs the fp64 oracle; for signed inputs the
rounding bound 2^-23 * sum|a_ik b_kj| is added)."""
import numpy as np
import pytest
import torch

import oracle
import synth
from oracle import stages
import paper_conf_icde_leekyjkp20_b200 as spg

pytestmark = pytest.mark.gpu

RTOL = 1e-5


def _sms():
    return torch.cuda.get_device_properties(0).multi_processor_count


def _plan(inp, **opts):
    A, B = spg.from_inputs(inp, "cuda")
    return spg.Plan(A, B, **opts), (A, B)


def _abs_inputs(inp):
    return synth.SparseInputs(inp.name + "|abs|", inp.m, inp.k, inp.n, inp.a_colptr, inp.a_rowidx,
                              np.abs(inp.a_val), inp.b_rowptr, inp.b_colidx, np.abs(inp.b_val))


def assert_c_matches(C, inp, signed=False):
    rowptr, col, val = oracle.gustavson(inp)
    got_rowptr = C.rowptr.cpu().numpy()
    got_col = C.colidx.cpu().numpy()
    got_val = C.val.cpu().numpy().astype(np.float64)
    np.testing.assert_array_equal(got_rowptr, rowptr)       # structure bit-exact
    np.testing.assert_array_equal(got_col, col)
    tol = RTOL * np.abs(val)
    if signed:
        _, _, mag = oracle.gustavson(_abs_inputs(inp))
        tol = tol + 2.0 ** -23 * mag
    bad = np.abs(got_val - val) > tol
    assert not bad.any(), f"{bad.sum()} values out of tolerance, e.g. got {got_val[bad][:4]} want {val[bad][:4]}"


PAD_KEY = 0x7FFFFFFF


def _caps(inp):
    """Padded Ĉ bucket length of every row: runs rounded up to 8 slots (32-byte sectors, DESIGN.md
    §4, R16); not method arithmetic, the layout of the buffer."""
    ca, rb, _ = stages.pair_workload(inp)
    col_of = np.repeat(np.arange(inp.k), ca)
    cap = np.zeros(inp.m, dtype=np.int64)
    np.add.at(cap, inp.a_rowidx.astype(np.int64), (rb[col_of] + 7) // 8 * 8)
    return cap


def _deg(inp):
    ca, rb, _ = stages.pair_workload(inp)
    col_of = np.repeat(np.arange(inp.k), ca)
    d = np.zeros(inp.m, dtype=np.int64)
    np.add.at(d, inp.a_rowidx.astype(np.int64), (rb[col_of] > 0).astype(np.int64))
    return d


TILES = dict(reserved=(0, 0, 0, 0, 0, 2) + (0,) * 10)   # tile merge (merge_tiles.cuh, merge_long.cuh)
TILES_INPLACE = dict(reserved=(0, 0, 0, 0, 0, 2, 1) + (0,) * 9)   # tile merge, legacy long rows

CASES = [
    ("C1", dict()),
    ("C1", dict(reserved=(0, 0, 0, 1) + (0,) * 12)),   # row-product expansion (comparison order)
    ("C1", dict(reserved=(0, 0, 1) + (0,) * 13)),      # per-row compaction kernels
    ("C1", dict(reserved=(0, 0, 0, 0, 1) + (0,) * 11)),   # no per-row column range from the plan
    ("C1", dict(enable_gather=0)),
    ("C1", dict(enable_split=0)),
    ("C1", dict(piece_work=300, split_b_tile=37, split_ca_max=5)),
    ("C1", dict(alpha=2.0)),
    ("C1", dict(beta=10.0)),
    ("C1", dict(beta=10.0, enable_limit=0)),
    ("C1", dict(reserved=(0,) * 9 + (1,) + (0,) * 6)),   # expansion: every block through the flat kernel
    ("C1", dict(reserved=(0,) * 9 + (2,) + (0,) * 6)),   # expansion: Low performers a vector per thread
    ("C1", dict(reserved=(0,) * 11 + (1,) + (0,) * 4)),   # rows of <= 256 slots: warp merge path (round 1)
    ("C1", dict(reserved=(0,) * 7 + (4,) + (0,) * 8)),   # fixed splitting factor 4 (Fig. 11 sweep)
    ("C1", dict(reserved=(0,) * 7 + (64,) + (0,) * 8)),
    ("C1", TILES),
    ("C1", dict(beta=10.0, **TILES)),                # the paper's β: many long rows -> column groups
    ("C1", dict(beta=10.0, **TILES_INPLACE)),        # ... or merged in place and moved
]


def _inp(name, seed=1, **kw):
    if name == "C1":
        return synth.make_inputs("C1", seed=seed, **kw)
    raise KeyError(name)


# ------------------------------------------------------------------ stage (1) -------------
@pytest.mark.parametrize("seed", [1, 2])
def test_stage1_workload(seed):
    inp = _inp("C1", seed)
    p, keep = _plan(inp)
    ca, rb, work = stages.pair_workload(inp)
    rowwork = stages.row_workload(inp)
    np.testing.assert_array_equal(p.inspect(spg.VIEW_WORK, np.int64), work)
    np.testing.assert_array_equal(p.inspect(spg.VIEW_ROWWORK, np.int64), rowwork)
    np.testing.assert_array_equal(p.inspect(spg.VIEW_ROWOFF, np.int64), stages.chat_row_offsets(_caps(inp)))
    st = p.stats()
    assert st["nnz_chat"] == st["nnz_chat_rowwise"] == int(work.sum())
    assert st["k_nonempty"] == int((work > 0).sum()) and st["m_nonempty"] == int((rowwork > 0).sum())
    p.destroy()


@pytest.mark.parametrize("name", ["C1", "tiny"])
def test_stage1_row_column_range(name):
    """The plan's per-row column range (the merge's bucket mapping, R12) is exactly the
    first / last column of each row of the oracle's C; empty rows keep min > max."""
    inp = _inp("C1") if name == "C1" else synth.random_tiny(300, 700, 500, 0.03, 0.05, 9, skew=True)
    p, keep = _plan(inp)
    mn = p.inspect(spg.VIEW_ROW_COLMIN, np.int32)
    mx = p.inspect(spg.VIEW_ROW_COLMAX, np.int32)
    rowptr, col, _ = oracle.gustavson(inp)
    ne = np.diff(rowptr) > 0
    # the range is computed for the bucket-sorted rows (padded Ĉ bucket > 256 slots), the others
    # stay "unknown" (min > max)
    big = ne & (np.diff(stages.chat_row_offsets(_caps(inp))) > 256)
    assert big.sum() > 0
    np.testing.assert_array_equal(mn[big], col[rowptr[:-1][big]])
    np.testing.assert_array_equal(mx[big], col[rowptr[1:][big] - 1])
    assert np.all(mn[~big] > mx[~big])
    p.destroy()


# ------------------------------------------------------------------ stage (2) -------------
@pytest.mark.parametrize("name,opts", CASES)
def test_stage2_reorganizer(name, opts):
    inp = _inp(name)
    p, keep = _plan(inp, **opts)
    o = spg.options(**opts)
    st = p.stats()
    ca, rb, work = stages.pair_workload(inp)
    t_dom = stages.dominator_threshold(int(work.sum()), int((work > 0).sum()), o.alpha, _sms(), o.dom_waves,
                                       o.dom_min_work, o.piece_work)
    assert st["t_dom"] == t_dom
    cls = stages.classify_pairs(ca, rb, work, t_dom, o.split_ca_max)
    np.testing.assert_array_equal(p.inspect(spg.VIEW_PAIR_CLASS, np.int8), cls)
    if o.enable_split:
        want = stages.split_pieces(inp, cls, o.piece_work, o.split_b_tile, o.split_ca_max, fixed_f=o.reserved[7])
        got = p.inspect(spg.VIEW_PIECES, np.int64).reshape(-1, 5)
        np.testing.assert_array_equal(got, want)
        assert st["n_pieces_split"] == len(want)
    if o.enable_gather:
        lists = stages.gather_lists(ca, rb, cls)
        np.testing.assert_array_equal(p.inspect(spg.VIEW_GATHER, np.int32),
                                      np.concatenate([lists[b] for b in range(6)]))
        assert st["n_gather_bin"] == [len(lists[b]) for b in range(6)]
    rowwork = stages.row_workload(inp)
    # enable_limit = 0 (Fig. 10 ablation): no Limiting rows by the β threshold
    t_lim = stages.limiting_threshold(int(work.sum()), int((rowwork > 0).sum()), o.beta if o.enable_limit else 0.0,
                                      4096)
    assert st["t_lim"] == t_lim
    want_rows = stages.row_bins(rowwork, t_lim)
    got_rows = p.inspect(spg.VIEW_ROW_CLASS, np.int8)
    cap = _caps(inp)
    # single-run rows are already merged; short ones (padded bucket <= 2048, the unit kernel's
    # row bound) are classed apart, long ones go through the long-row bins
    single = (_deg(inp) == 1) & (rowwork > 0) & (cap <= 2048)
    # processing bins: the paper's limiting rows (B-Limiting) plus rows whose padded bucket
    # exceeds the non-limited kernels' capacity; the others by padded length
    lim = ((want_rows == stages.ROW_LIMITED) | (cap > 4096)) & ~single & (rowwork > 0)
    np.testing.assert_array_equal(got_rows == 0, want_rows == stages.ROW_EMPTY)
    np.testing.assert_array_equal(got_rows == 1, single)
    np.testing.assert_array_equal(got_rows == 5, lim)
    rest = (rowwork > 0) & ~single & ~lim
    np.testing.assert_array_equal(got_rows == 2, rest & (cap <= 32))
    np.testing.assert_array_equal((got_rows == 3) | (got_rows == 4), rest & (cap > 32))
    p.destroy()


# ------------------------------------------------------------------ stage (3) -------------
def _rows_sorted(m, rowoff, cols, vals):
    out = []
    for i in range(m):
        c = cols[rowoff[i]:rowoff[i + 1]]
        v = vals[rowoff[i]:rowoff[i + 1]]
        o = np.lexsort((v, c))
        out.append((c[o], v[o]))
    return out


EXPAND_CASES = [c for c in CASES if not c[1] or {"enable_gather", "enable_split", "piece_work"} & set(c[1])
                or c[1].get("reserved", (0,) * 16)[3] == 1 or c[1].get("reserved", (0,) * 16)[9] != 0]


@pytest.mark.parametrize("name,opts", EXPAND_CASES)
def test_stage3_expansion_is_eq2(name, opts):
    inp = _inp(name)
    p, keep = _plan(inp, **opts)
    p.expand()
    cols = p.inspect(spg.VIEW_CHAT_COL, np.int32)
    vals = p.inspect(spg.VIEW_CHAT_VAL, np.float32)
    rowoff_pad = p.inspect(spg.VIEW_ROWOFF, np.int64)
    # drop the sentinel padding slots (col = INT32_MAX, val = 0), then compare per row
    real = cols != PAD_KEY
    assert np.all(vals[~real] == 0)
    row_of = np.repeat(np.arange(inp.m), np.diff(rowoff_pad))
    cols, vals = cols[real], vals[real]
    rowoff = np.zeros(inp.m + 1, dtype=np.int64)
    np.cumsum(np.bincount(row_of[real], minlength=inp.m), out=rowoff[1:])
    r, c, v = stages.expand_outer(inp)
    # each oracle product a*b (exact in fp64) rounded once to fp32 = the kernel's fp32 multiply
    v32 = v.astype(np.float32)
    order = np.lexsort((v32, c, r))
    r, c, v32 = r[order], c[order], v32[order]
    o_rowoff = np.zeros(inp.m + 1, dtype=np.int64)
    np.cumsum(np.bincount(r, minlength=inp.m), out=o_rowoff[1:])
    np.testing.assert_array_equal(rowoff, o_rowoff)
    got = _rows_sorted(inp.m, rowoff, cols, vals)
    gc = np.concatenate([g[0] for g in got])
    gv = np.concatenate([g[1] for g in got])
    np.testing.assert_array_equal(gc, c)
    np.testing.assert_array_equal(gv.view(np.uint32), v32.view(np.uint32))   # bit-exact
    p.destroy()


# ------------------------------------------------------------------ stage (4) + output ----
@pytest.mark.parametrize("name,opts", CASES)
def test_c_matches_oracle(name, opts):
    inp = _inp(name)
    A, B = spg.from_inputs(inp, "cuda")
    C = spg.matmul(A, B, **opts)
    assert_c_matches(C, inp)


@pytest.mark.parametrize("shape,dens,seed,skew,values", [
    ((1, 1, 1), (1.0, 1.0), 1, False, "real"),
    ((7, 5, 9), (0.3, 0.4), 2, False, "real"),
    ((33, 20, 41), (0.1, 0.15), 4, True, "signed"),
    ((40, 64, 40), (0.05, 0.5), 5, False, "int"),
    ((20, 3, 30), (0.0, 0.5), 6, False, "real"),
    ((25, 30, 12), (0.3, 0.0), 7, False, "real"),
    ((64, 1, 64), (0.5, 0.5), 8, False, "real"),
    ((300, 700, 500), (0.03, 0.05), 9, True, "signed"),
])
def test_random_tiny(shape, dens, seed, skew, values):
    inp = synth.random_tiny(*shape, dens[0], dens[1], seed, values=values, skew=skew)
    A, B = spg.from_inputs(inp, "cuda")
    for opts in (dict(), dict(beta=1000.0, piece_work=64, split_ca_max=3), dict(reserved=(0, 0, 1) + (0,) * 13),
                 TILES, dict(beta=1000.0, **TILES), dict(beta=1000.0, piece_work=64, split_ca_max=3, **TILES)):
        C = spg.matmul(A, B, **opts)
        assert_c_matches(C, inp, signed=(values == "signed"))


def test_integer_values_exact():
    inp = synth.make_inputs("C1", seed=5, values="int")
    A, B = spg.from_inputs(inp, "cuda")
    C = spg.matmul(A, B)
    rowptr, col, val = oracle.gustavson(inp)
    np.testing.assert_array_equal(C.colidx.cpu().numpy(), col)
    np.testing.assert_array_equal(C.val.cpu().numpy().astype(np.float64), val)   # exact


def _wide_inputs(m, k, n, a_density, run_len, seed, hub_col=False, narrow=False, kind="real"):
    rng = np.random.default_rng(seed)
    ar, ac = np.nonzero(rng.random((m, k)) < a_density)
    br = np.repeat(np.arange(k), run_len)
    cols = []
    for q in range(k):
        c = rng.choice(np.arange(1, n) if hub_col else n, run_len - (1 if hub_col else 0), replace=False)
        if hub_col:
            c = np.concatenate([[0], c])
        cols.append(np.sort(c))
    bc = np.concatenate(cols)
    if narrow:
        bc[:run_len] = np.arange(run_len) * 3
    return synth.from_coo("wide", m, k, n, (ar, ac, synth.edge_values(ar, ac, seed, kind)),
                          (br, bc, synth.edge_values(br, bc, seed + 1, kind)))


@pytest.mark.parametrize("m,k,n,dens,run_len,hub,narrow", [
    (40, 120, 70000, 0.25, 300, False, True),     # limited rows ~9K: in-smem path and sparse windows
    (24, 200, 400000, 0.5, 200, False, False),     # sparse long rows: several smem windows
    (16, 100, 30000, 0.3, 2000, False, False),     # dense rows: fp64 column windows
    (2, 10000, 1000000, 1.0, 21, True, False),     # column 0 in 10000 runs: single-column overflow
])
@pytest.mark.parametrize("fused", [False, "lim2", "lim4", "tiles", "tiles_inplace"])
def test_limited_paths(m, k, n, dens, run_len, hub, narrow, fused):
    """B-Limited merge: rows longer than the non-limited capacity, through every sub-path."""
    inp = _wide_inputs(m, k, n, dens, run_len, 3, hub_col=hub, narrow=narrow)
    A, B = spg.from_inputs(inp, "cuda")
    opts = {False: {}, "lim2": dict(limit_ctas_per_sm=2), "lim4": dict(limit_ctas_per_sm=4),   # B-Limiting 2 / 4 per SM
            "tiles": TILES, "tiles_inplace": TILES_INPLACE}[fused]
    with spg.Plan(A, B, **opts) as p:
        st = p.stats()
        assert st["n_rows_bin"][5] > 0
        p.expand()
        p.merge()
        C = p.output()
    assert_c_matches(C, inp)
    with spg.Plan(A, B, **opts) as p:   # staged path with host output
        p.expand()
        p.merge()
        C = p.output(device="cpu")
    assert_c_matches(C, inp)


@pytest.mark.parametrize("k,cluster,spread", [(10, 20, 10), (40, 40, 60), (60, 100, 2)])
def test_clustered_columns_fallback(k, cluster, spread):
    """Rows whose columns cluster in a narrow range of a wide span overflow the bucket sort's
    buckets; the natural merge sort fallback (and the limited kernel's inline fallback) take them;
    the tile merge ranks the crowded buckets."""
    rng = np.random.default_rng(5)
    m, n = 6, 1_000_000
    ar, ac = np.nonzero(np.ones((m, k), dtype=bool))
    br, bc = [], []
    for q in range(k):
        c = np.concatenate([np.arange(q * cluster, (q + 1) * cluster),
                            rng.choice(np.arange(10 ** 5, n), spread, replace=False)])
        c = np.unique(c)
        br.append(np.full(c.size, q))
        bc.append(c)
    br, bc = np.concatenate(br), np.concatenate(bc)
    inp = synth.from_coo("clustered", m, k, n, (ar, ac, synth.edge_values(ar, ac, 1)),
                         (br, bc, synth.edge_values(br, bc, 2)))
    A, B = spg.from_inputs(inp, "cuda")
    C = spg.matmul(A, B)
    assert_c_matches(C, inp)
    assert_c_matches(spg.matmul(A, B, **TILES), inp)


def test_row_partition_and_row_blocks():
    """spgemm_row_partition equals the oracle's balanced partition (R8), and C assembled from
    independently computed row blocks (the multi-GPU decomposition) equals the oracle's C."""
    from paper_conf_icde_leekyjkp20_b200 import dist as pdist
    inp = synth.make_inputs("C1", seed=3)
    A, B = spg.from_inputs(inp, "cuda")
    rw = stages.row_workload(inp)
    for parts in (1, 2, 3, 8):
        np.testing.assert_array_equal(spg.row_partition(A, B, parts), stages.balanced_row_partition(rw, parts))
    bounds = spg.row_partition(A, B, 4)
    blocks = [spg.matmul(pdist.csc_row_slice(A, int(bounds[r]), int(bounds[r + 1])), B) for r in range(4)]
    C = pdist.concat_row_blocks(blocks)
    assert_c_matches(C, inp)


@pytest.mark.parametrize("name", ["S1", "S2", "S3", "P1", "P2", "P3", "P4", "SP1", "SP2", "SP3", "SP4",
                                  "AB15", "AB16"])
def test_table3_synthetic(name):
    """PAPER.md Table III synthetic sets (S / P / SP for C = A^2, AB for C = AB) against the
    oracle's whole C."""
    inp = synth.make_inputs(name, seed=1)
    A, B = spg.from_inputs(inp, "cuda")
    assert_c_matches(spg.matmul(A, B), inp)


@pytest.mark.parametrize("parts", [1, 3, 8])
def test_chunked_execution(parts):
    """Chunked expansion (row blocks one after another on one GPU) gives the oracle's C."""
    inp = synth.make_inputs("C1", seed=4)
    A, B = spg.from_inputs(inp, "cuda")
    assert_c_matches(spg.matmul_chunked(A, B, parts), inp)


def test_repeated_plans_and_concurrent_streams():
    """Plans are single-use and independent: 20 products in a row keep the same workspace size, and
    two host threads running products on two streams at once both match the oracle."""
    import threading
    inp = synth.make_inputs("C1", seed=6)
    A, B = spg.from_inputs(inp, "cuda")
    sizes = []
    for _ in range(20):
        with spg.Plan(A, B) as p:
            C = p.execute()
            sizes.append(p.stats()["bytes_workspace"])
    assert len(set(sizes)) == 1
    assert_c_matches(C, inp)
    out = [None, None]

    def run(q):
        st = torch.cuda.Stream()
        with torch.cuda.stream(st):
            out[q] = spg.matmul(A, B, stream=st)
        st.synchronize()

    ts = [threading.Thread(target=run, args=(q,)) for q in range(2)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    for q in range(2):
        assert_c_matches(out[q], inp)
    spg.trim_pool()


def test_empty_and_degenerate():
    for shape in [(5, 0, 7), (0, 4, 3), (3, 4, 0)]:
        m, k, n = shape
        inp = synth.random_tiny(max(m, 1), max(k, 1), max(n, 1), 0.0, 0.0, 1)
        inp = synth.SparseInputs("e", m, k, n, np.zeros(k + 1, np.int64), np.zeros(0, np.int32),
                                 np.zeros(0, np.float32), np.zeros(k + 1, np.int64), np.zeros(0, np.int32),
                                 np.zeros(0, np.float32))
        A, B = spg.from_inputs(inp, "cuda")
        C = spg.matmul(A, B)
        assert C.nnz == 0 and C.rowptr.cpu().tolist() == [0] * (m + 1)


def test_host_inputs_and_outputs():
    inp = synth.make_inputs("C1", seed=7)
    A, B = spg.from_inputs(inp, "cpu")
    C = spg.matmul(A, B, device="cpu")
    assert not C.val.is_cuda
    assert_c_matches(C, inp)


def test_validation_rejects_malformed():
    inp = synth.make_inputs("C1", seed=1)
    bad = inp.a_rowidx.copy()
    s = int(inp.a_colptr[10])
    if inp.a_colptr[11] - s >= 2:
        bad[s], bad[s + 1] = bad[s + 1], bad[s]
    else:
        bad[s] = inp.m + 5
    inp2 = synth.SparseInputs("bad", inp.m, inp.k, inp.n, inp.a_colptr, bad, inp.a_val, inp.b_rowptr,
                              inp.b_colidx, inp.b_val)
    A, B = spg.from_inputs(inp2, "cuda")
    with pytest.raises(spg.SpgemmError, match="malformed"):
        spg.Plan(A, B)


# ------------------------------------------------------------------ computed zeros ----------
def _assert_exact(C, inp):
    rowptr, col, val = oracle.gustavson(inp)
    np.testing.assert_array_equal(C.rowptr.cpu().numpy(), rowptr)
    np.testing.assert_array_equal(C.colidx.cpu().numpy(), col)
    np.testing.assert_array_equal(C.val.cpu().numpy().astype(np.float64), val)   # +-1 sums: exact
    return val


def test_computed_zeros_hand():
    """c_0j = (+1)(b_0j) + (-1)(b_1j) with b_0* = b_1*: every entry of row 0 cancels exactly and is
    still stored (R7: "merged into unique elements", PAPER.md L453-L455 L)."""
    cols = np.array([3, 17, 40, 41], dtype=np.int32)
    br = np.repeat(np.array([0, 1], dtype=np.int32), cols.size)
    bc = np.tile(cols, 2)
    bv = np.tile(np.array([0.5, 1.25, 2.0, 3.0], dtype=np.float32), 2)
    inp = synth.from_coo("cancel", 2, 2, 64, (np.array([0, 0, 1]), np.array([0, 1, 1]),
                                              np.array([1.0, -1.0, 2.0], dtype=np.float32)), (br, bc, bv))
    A, B = spg.from_inputs(inp, "cuda")
    for opts in ({}, TILES):
        C = spg.matmul(A, B, **opts)
        val = _assert_exact(C, inp)
        assert C.rowptr.cpu().tolist() == [0, 4, 8]
        assert np.all(val[:4] == 0) and np.all(C.val[:4].cpu().numpy() == 0)


@pytest.mark.parametrize("opts", [{}, dict(beta=10.0), TILES])
def test_computed_zeros_pm1(opts):
    """+-1 values (synth kind 'pm1'): thousands of entries cancel exactly; the structure keeps them and
    the values are exact (short rows, the paper's β-Limiting rows, and the legacy bins)."""
    inp = synth.make_inputs("C1", seed=2, values="pm1")
    A, B = spg.from_inputs(inp, "cuda")
    val = _assert_exact(spg.matmul(A, B, **opts), inp)
    assert (val == 0).sum() > 1000


def test_computed_zeros_long_rows():
    """Exact cancellation inside B-Limited rows (padded bucket > 4096 slots)."""
    inp = _wide_inputs(40, 120, 70000, 0.25, 300, 3, narrow=True, kind="pm1")
    A, B = spg.from_inputs(inp, "cuda")
    with spg.Plan(A, B) as p:
        assert p.stats()["n_rows_bin"][5] > 0
        C = p.execute()
    val = _assert_exact(C, inp)
    assert (val == 0).sum() > 0


# ------------------------------------------------------------------ overflow regression -----
@pytest.mark.parametrize("k,run", [(69, 130), (140, 60)])
def test_limited_bucket_overflow_many_heavy_buckets(k, run):
    """one limited row made of k runs of the same `run` columns spread
    over ~130K columns: `run` buckets of k equal keys.  (69, 130): 130 heavy buckets below the
    overflow threshold (kBucketMax = 127), ranked by their sort codes; (140, 60): 60 buckets above it
    -- the overflow flag of the bucket scan must not wrap and the row takes the fallback.  Both match
    the oracle."""
    cols = np.sort(np.random.default_rng(4).choice(130_000, run, replace=False)).astype(np.int32)
    br = np.repeat(np.arange(k, dtype=np.int32), run)
    bc = np.tile(cols, k)
    ar = np.zeros(k, dtype=np.int32)
    ac = np.arange(k, dtype=np.int32)
    inp = synth.from_coo("heavy", 1, k, 130_000, (ar, ac, synth.edge_values(ar, ac, 1)),
                         (br, bc, synth.edge_values(br, bc, 2)))
    A, B = spg.from_inputs(inp, "cuda")
    for opts in ({}, TILES):
        with spg.Plan(A, B, **opts) as p:
            assert p.stats()["n_rows_bin"][5] == 1   # the row is B-Limited (9384 / 8960 padded slots)
            C = p.execute()
        assert_c_matches(C, inp)


@pytest.mark.parametrize("lim", [1, 2, 4])
def test_limited_huge_row_every_blocks_per_sm(lim):
    """B-Limiting at 1 / 2 / 4 limited blocks per SM (PAPER.md L463-L469 L, Fig. 14) on two rows of
    ~1.1M products each spread over 20M columns: more column groups than the coarse tables hold for
    the smaller sorters, so those rows are deferred to the 1-per-SM launch; C matches the oracle."""
    rng = np.random.default_rng(7)
    k, run, n = 1100, 1000, 20_000_000
    bc = np.concatenate([np.sort(rng.choice(n, run, replace=False)) for _ in range(k)]).astype(np.int32)
    br = np.repeat(np.arange(k, dtype=np.int32), run)
    ar = np.repeat(np.arange(2, dtype=np.int32), k)
    ac = np.tile(np.arange(k, dtype=np.int32), 2)
    inp = synth.from_coo("huge", 2, k, n, (ar, ac, synth.edge_values(ar, ac, 1)),
                         (br, bc, synth.edge_values(br, bc, 2)))
    A, B = spg.from_inputs(inp, "cuda")
    with spg.Plan(A, B, limit_ctas_per_sm=lim) as p:
        assert p.stats()["n_rows_bin"][5] == 2
        C = p.execute()
    assert_c_matches(C, inp)


# ------------------------------------------------------------------ LBI (Eq. 3) ---------------
def test_lbi_recording():
    """PAPER.md Eq. (3): LBI = mean_i T_i / max_i T_i over the SMs, from per-SM busy times the
    kernels record with options.reserved[8] = 1 (0 < LBI <= 1); recording does not change C."""
    inp = _wide_inputs(40, 120, 70000, 0.25, 300, 3, narrow=True)
    A, B = spg.from_inputs(inp, "cuda")
    opts = dict(reserved=(0,) * 8 + (1,) + (0,) * 7)
    with spg.Plan(A, B, **opts) as p:
        C = p.execute()
        lb = p.lbi()
    assert_c_matches(C, inp)
    for name in ("expand", "merge_limited"):
        assert lb[name] is not None, name
        assert 0.0 < lb[name]["lbi"] <= 1.0 and lb[name]["max_ms"] > 0


@pytest.mark.parametrize("ca,rb", [(1, 6000), (3, 6000), (2, 4097), (40, 1)])
def test_expansion_block_shapes(ca, rb):
    """The block-path expansion (TMA-staged B' tiles): a Normal block whose B row exceeds one
    shared-memory buffer (1 x 6000: sub-tiles), a split Dominator with B tiles, a row one past a
    tile, and thin blocks -- Ĉ against Eq. (2) through the full C."""
    rng = np.random.default_rng(ca * 7 + rb)
    ar = np.arange(ca, dtype=np.int32)
    ac = np.zeros(ca, dtype=np.int32)
    bc = np.sort(rng.choice(10 * rb + 10, rb, replace=False)).astype(np.int32)
    br = np.zeros(rb, dtype=np.int32)
    inp = synth.from_coo("blk", ca, 1, 10 * rb + 10, (ar, ac, synth.edge_values(ar, ac, 1)),
                         (br, bc, synth.edge_values(br, bc, 2)))
    A, B = spg.from_inputs(inp, "cuda")
    for opts in ({}, dict(reserved=(0,) * 9 + (1,) + (0,) * 6), dict(split_b_tile=1000)):
        assert_c_matches(spg.matmul(A, B, **opts), inp)


@pytest.mark.parametrize("r0,r1", [(0, 1024), (0, 1), (100, 300), (512, 512), (1000, 1024), (7, 1021)])
def test_row_window_plan(r0, r1):
    """spgemm_plan_rows: rows [r0, r1) of C (A windowed on the GPU, no copy by the caller) equal the
    oracle's rows [r0, r1) -- the chunked expansion and multi-GPU row blocks (R8)."""
    inp = synth.make_inputs("C1", seed=3)
    A, B = spg.from_inputs(inp, "cuda")
    C = spg.matmul(A, B, rows=(r0, r1))
    rows = np.arange(r0, r1, dtype=np.int32)
    orp, ocol, oval = oracle.gustavson(inp, rows=rows) if r1 > r0 else (np.zeros(1, np.int64), [], np.zeros(0))
    np.testing.assert_array_equal(C.rowptr.cpu().numpy(), orp)
    np.testing.assert_array_equal(C.colidx.cpu().numpy(), ocol)
    got = C.val.cpu().numpy().astype(np.float64)
    assert np.all(np.abs(got - oval) <= RTOL * np.abs(oval))
