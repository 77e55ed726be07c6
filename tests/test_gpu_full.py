"""Whole-matrix parity at BASELINE.json's full sizes, in the bench's launch configuration
(spgemm_plan + spgemm_execute through the C-ABI, device-resident inputs): EVERY row of C compared
with the oracle -- row pointers and column indices bit-exactly, values within relative 1e-5
(tests/parity_util.py) -- for C2, C3, C4, C5 (whole and in 4 chunks) and the Table III C = AB sets
AB17 / AB18.  Plus the full-size stage arrays of the hub-heavy C3 (pair classes and B-Splitting
pieces, PAPER.md L304-L318 R, L320-L415) against the oracle's stage definitions."""
import numpy as np
import pytest
import torch

import paper_conf_icde_leekyjkp20_b200 as spg
from oracle import stages
from parity_util import cached_inputs, whole_matrix_check

pytestmark = pytest.mark.gpu

TILES = dict(reserved=(0, 0, 0, 0, 0, 2) + (0,) * 10)   # tile merge: look-back placement, no compaction


def _fresh():
    torch.cuda.synchronize()
    torch.cuda.empty_cache()
    spg.trim_pool()


@pytest.mark.parametrize("name,opts", [("C2", {}), ("C2", TILES), ("C4", {}), ("C3", {}), ("C3", TILES), ("C5", {}),
                                       ("C5", {"chunks": 4}), ("AB17", {}), ("AB18", {})])
def test_whole_matrix(name, opts):
    inp = cached_inputs(name)
    _fresh()
    A, B = spg.from_inputs(inp, "cuda")
    if "chunks" in opts:     # north star C5: chunked expansion (row blocks in turn)
        C = spg.matmul_chunked(A, B, opts["chunks"])
    else:
        with spg.Plan(A, B, **opts) as p:
            st = p.stats()
            C = p.execute()
        ca, rb, work = stages.pair_workload(inp)
        assert st["nnz_chat"] == int(work.sum())
    del A, B
    rows, entries, chunks = whole_matrix_check(C, inp)
    assert rows == inp.m and entries == C.nnz
    del C
    _fresh()


def test_c3_stage_arrays_full_size():
    """Pair classes and every B-Splitting piece of the hub-heavy C3 (35K-degree hubs: B tiles and
    A sub-columns) equal the oracle's definitions, bit-exactly."""
    inp = cached_inputs("C3")
    _fresh()
    A, B = spg.from_inputs(inp, "cuda")
    with spg.Plan(A, B) as p:
        o = spg.options()
        st = p.stats()
        ca, rb, work = stages.pair_workload(inp)
        sms = torch.cuda.get_device_properties(0).multi_processor_count
        t_dom = stages.dominator_threshold(int(work.sum()), int((work > 0).sum()), o.alpha, sms, o.dom_waves,
                                           o.dom_min_work, o.piece_work)
        assert st["t_dom"] == t_dom
        cls = stages.classify_pairs(ca, rb, work, t_dom, o.split_ca_max)
        np.testing.assert_array_equal(p.inspect(spg.VIEW_PAIR_CLASS, np.int8), cls)
        want = stages.split_pieces(inp, cls, o.piece_work, o.split_b_tile, o.split_ca_max)
        got = p.inspect(spg.VIEW_PIECES, np.int64).reshape(-1, 5)
        assert len(want) > 10000   # the hubs really are split
        np.testing.assert_array_equal(got, want)
        lists = stages.gather_lists(ca, rb, cls)
        np.testing.assert_array_equal(p.inspect(spg.VIEW_GATHER, np.int32),
                                      np.concatenate([lists[b] for b in range(6)]))
    _fresh()
