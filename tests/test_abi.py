"""CPU-side checks of the C-ABI boundary: the library loads, exports every entry point
include/tc.h declares, and fails loudly (no CPU fallback) when no GPU is present."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_sigmod_hu0l21_b200 as tc
from tests.conftest import ROOT


def declared_functions():
    src = open(os.path.join(ROOT, "include", "tc.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(tc_[a-z_]+)\s*\(", src)))


def test_header_declares_the_survey_boundary():
    names = declared_functions()
    for f in ("tc_graph_from_edges", "tc_direct", "tc_reorder", "tc_count", "tc_count_dist",
              "tc_export", "tc_graph_free", "tc_last_error", "tc_get_stats"):
        assert f in names


def test_library_exports_every_declared_symbol():
    L = ctypes.CDLL(tc.LIB_PATH)
    missing = [f for f in declared_functions() if not hasattr(L, f)]
    assert not missing, missing


def test_binding_mirrors_abi_names():
    for f in declared_functions():
        assert hasattr(tc, f), f


def test_struct_layouts():
    assert ctypes.sizeof(tc.AOrderParams) == 3 * 8 + 8 + 4 + 4 + 4 + 4  # padded to 8
    assert ctypes.sizeof(tc.Stats) == 8 * 7 + 8 + 4 * 6 + 8 * 3 + 8 * 5 + 8 + 8 + 8 + 8


def test_version_string():
    assert "sm_100a" in tc.tc_version()


@pytest.mark.skipif(os.environ.get("CUDA_VISIBLE_DEVICES", None) != "" and
                    __import__("torch").cuda.is_available(), reason="a GPU is present")
def test_no_cpu_fallback_without_gpu():
    z = np.array([0, 1], np.uint32)
    with pytest.raises(tc.TCError) as e:
        tc.Graph(z, z[::-1].copy(), 2)
    assert e.value.status == tc.TC_ERR_CUDA
    assert "no CUDA device" in str(e.value)


# (key, default, an accepted value, a rejected value or None): the options tc.h documents
OPTIONS = [("cuckoo", 64, 0, 2000), ("otiles", 1, 7, 300), ("otile_mb", 48, 16, 0), ("otile_min", 4, 0, -1),
           ("e2sort", -1, 1, None), ("aorder_device", 1, 0, None), ("peel_red", -1, 1, None),
           ("owner_span", 128, 32, None), ("owner_lspan", 2048, 64, 4), ("small_cap", 256, 512, 100),
           ("extra_compute", -1, 8, 2000), ("shorter", 1, 0, None), ("vtiles", 1, 2, 0)]


@pytest.mark.parametrize("key,default,good,bad", OPTIONS, ids=[o[0] for o in OPTIONS])
def test_options_validate_and_restore(key, default, good, bad):
    """tc_set_option accepts the documented range, rejects values outside it with
    TC_ERR_INVALID (no partial state), and unknown keys; runs without a GPU."""
    try:
        tc.tc_set_option(key, good)
        if bad is not None:
            with pytest.raises(tc.TCError) as e:
                tc.tc_set_option(key, bad)
            assert e.value.status == tc.TC_ERR_INVALID
    finally:
        tc.tc_set_option(key, default)


def test_unknown_option_rejected():
    with pytest.raises(tc.TCError) as e:
        tc.tc_set_option("no_such_option", 1)
    assert e.value.status == tc.TC_ERR_INVALID
