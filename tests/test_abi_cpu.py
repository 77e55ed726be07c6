"""CPU-only checks of the boundary: the C-ABI library loads and exports every symbol that
include/spgemm.h declares, options defaults are sane, and calls fail loudly (never fall back)
without a GPU or with bad arguments."""
import ctypes
import os
import re

import pytest
import torch

import paper_conf_icde_leekyjkp20_b200 as spg
from paper_conf_icde_leekyjkp20_b200.build import build_library

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    text = open(os.path.join(ROOT, "include", "spgemm.h")).read()
    return sorted(set(re.findall(r"^\s*(?:int|void|const char \*)\s*(spgemm_\w+)\s*\(", text, re.M)))


def test_library_exports_every_declared_symbol():
    build_library()
    L = ctypes.CDLL(spg.LIB_PATH)
    names = _declared()
    assert len(names) >= 12
    for nm in names:
        assert hasattr(L, nm), nm
    assert sorted(spg.EXPORTED) == names


def test_struct_layouts_match_header():
    # natural C layout of spgemm_options_t / spgemm_stats_t (x86-64 SysV, as the header declares)
    assert ctypes.sizeof(spg.Options) == 144
    assert spg.Options.piece_work.offset == 32 and spg.Options.beta.offset == 48
    assert spg.Options.reserved.offset == 76
    assert ctypes.sizeof(spg.Stats) == 31 * 8
    o = spg.options()
    assert o.dom_waves == 16 and o.split_ca_max == 256 and o.piece_work == 16384
    assert o.split_b_tile == 4096 and o.limit_ctas_per_sm == 1 and o.validate == 1
    assert o.enable_split == o.enable_gather == o.enable_limit == 1
    assert spg.lib().spgemm_abi_version() == 1


def test_bad_arguments_are_rejected():
    L = spg.lib()
    h = ctypes.c_void_p()
    assert L.spgemm_plan(None, None, None, None, ctypes.byref(h)) == 1
    assert b"NULL" in L.spgemm_last_error()
    assert L.spgemm_expand(None, None) == 1
    assert L.spgemm_destroy(None) == 0


@pytest.mark.skipif(torch.cuda.is_available(), reason="checks the no-GPU error path")
def test_no_gpu_fails_loudly():
    import synth
    inp = synth.make_inputs("C1", seed=1)
    A, B = spg.from_inputs(inp, "cpu")
    with pytest.raises(spg.SpgemmError):
        spg.matmul(A, B, device="cpu")
