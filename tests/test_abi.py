"""CPU-side checks of the C-ABI library: it loads, exports every symbol that
include/nulpa.h declares, and rejects bad arguments without touching a GPU."""
import ctypes
import os
import re

import pytest

import paper_conf_ipps_sahunk25_b200 as nl
from paper_conf_ipps_sahunk25_b200 import build as nlbuild

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "nulpa.h")


@pytest.fixture(scope="module")
def lib():
    nlbuild.build()
    return nl.load_library()


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(nulpa_[a-z_]+)\s*\(", src)))


def test_header_declares_the_boundary():
    names = declared_functions()
    for required in ["nulpa_create", "nulpa_run", "nulpa_labels", "nulpa_modularity", "nulpa_sweep",
                     "nulpa_destroy", "nulpa_last_error"]:
        assert required in names


def test_every_declared_symbol_is_exported(lib):
    for name in declared_functions():
        assert hasattr(lib, name), name
    # the python binding carries the same names
    for name in declared_functions():
        if name in ("nulpa_last_error", "nulpa_state_pointers"):
            continue
        assert hasattr(nl, name), name


def test_struct_layout_matches_header(lib):
    # nulpa_default_params fills the paper's constants
    p = nl.nulpa_default_params()
    assert p.tolerance == 0.05 and p.max_iterations == 20 and p.pickless_period == 4
    assert p.mode == nl.ASYNC and p.reset == 1
    assert 1 <= p.switch_degree <= p.block_degree <= p.giant_degree
    assert ctypes.sizeof(nl.Params) == 8 + 13 * 4 + 4   # 13 int32 fields, padded to 8
    assert 1 <= p.wide_degree <= 512
    assert nl.nulpa_version().startswith("nulpa")


def test_invalid_arguments_fail_loudly(lib):
    h = ctypes.c_void_p()
    rc = lib.nulpa_create(None, None, None, 0, 0, 0, 0, None, ctypes.byref(h))
    assert rc == 1 and b"offsets" in lib.nulpa_last_error()
    rc = lib.nulpa_create(None, None, None, 0, 0, 0, 0, None, None)
    assert rc == 1
    assert lib.nulpa_run(None, None, None) == 1
    assert lib.nulpa_sweep(None, 0, None, None) == 1
    assert lib.nulpa_labels(None, None, 0) == 1
    q = ctypes.c_double()
    assert lib.nulpa_modularity(None, None, 0, ctypes.byref(q)) == 1
    assert lib.nulpa_destroy(None) == 0


def test_no_cpu_fallback():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    import synth
    g = synth.karate()
    with pytest.raises(nl.NulpaError):
        nl.Graph(g.offsets, g.indices)


def test_build_flags_target_sm100a():
    assert "arch=compute_100a,code=sm_100a" in " ".join(nlbuild.NVCC_FLAGS)
    assert "-lineinfo" in nlbuild.NVCC_FLAGS
