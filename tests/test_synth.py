"""Generators: seeded determinism, layout invariants, and the R-MAT / Table III shape."""
import numpy as np

import synth


def test_deterministic_and_consistent_layouts():
    a = synth.make_inputs("C1", seed=9)
    b = synth.make_inputs("C1", seed=9)
    for f in ("a_colptr", "a_rowidx", "a_val", "b_rowptr", "b_colidx", "b_val"):
        np.testing.assert_array_equal(getattr(a, f), getattr(b, f))
    # A (CSC) and B (CSR) hold the same matrix for C = A x A
    cols = np.repeat(np.arange(a.k), np.diff(a.a_colptr))
    rows = np.repeat(np.arange(a.k), np.diff(a.b_rowptr))
    ka = np.sort(a.a_rowidx.astype(np.int64) * a.n + cols)
    kb = np.sort(rows.astype(np.int64) * a.n + a.b_colidx)
    np.testing.assert_array_equal(ka, kb)
    # sorted within column / row, values a pure function of (row, col)
    for p in range(a.k):
        assert np.all(np.diff(a.a_rowidx[a.a_colptr[p]:a.a_colptr[p + 1]]) > 0)
        assert np.all(np.diff(a.b_colidx[a.b_rowptr[p]:a.b_rowptr[p + 1]]) > 0)
    np.testing.assert_array_equal(a.a_val, synth.edge_values(a.a_rowidx, cols, 9))
    assert a.a_val.min() >= 0.5 and a.a_val.max() < 1.5


def test_rmat_shape_like_table_iii():
    # Table III (L765-L777): scale 15, edge-factor 16 R-MAT has ~440K entries (< 16*2^15 = 524288)
    src, dst = synth.rmat_edges(15, 16, 0.57, 0.19, 0.19, seed=1)
    assert 380_000 < src.size < 524_288
    assert src.max() < 1 << 15 and dst.max() < 1 << 15


def test_row_slice():
    a = synth.make_inputs("C1", seed=2)
    s = synth.row_slice_coo(a, 100, 300)
    assert s.m == 200 and s.nnz_a == int(((a.a_rowidx >= 100) & (a.a_rowidx < 300)).sum())


def test_table3_shapes():
    """PAPER.md Table III: node counts and element counts (duplicates dropped) of the S / P / SP sets,
    distinct operands for the C = AB sets."""
    import numpy as np
    for name in ["S1", "S2", "S3", "S4", "P1", "P2", "P3", "P4", "SP1", "SP2", "SP3", "SP4"]:
        cfg = synth.CONFIGS[name]
        inp = synth.make_inputs(name, seed=1)
        assert inp.m == inp.k == inp.n == cfg["n"]
        assert 0.99 * cfg["m"] <= inp.nnz_a <= cfg["m"]
        np.testing.assert_array_equal(np.diff(inp.a_colptr).sum(), inp.nnz_b)   # A = B
    inp = synth.make_inputs("AB15", seed=1)
    assert inp.m == inp.k == inp.n == 1 << 15
    assert inp.nnz_a != inp.nnz_b or not np.array_equal(inp.a_rowidx, inp.b_colidx)
