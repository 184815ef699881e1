"""The C-ABI library loads on a GPU-less box and exports every symbol include/npp.h declares."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "npp.h")
LIB = os.path.join(ROOT, "paper_conf_micro_leebsro14_b200", "libnpp.so")


def declared_symbols():
    text = open(HEADER).read()
    return sorted(set(re.findall(r"NPP_API\s+[\w\s\*]+?\b(npp_\w+)\s*\(", text)))


def test_header_declares_the_boundary():
    syms = declared_symbols()
    for s in ("npp_plan", "npp_execute", "npp_select", "npp_limits_query", "npp_plan_with_mapping",
              "npp_plan_workspace_bytes", "npp_plan_destroy", "npp_last_error", "npp_execute_host"):
        assert s in syms


def test_library_exports_every_declared_symbol():
    assert os.path.exists(LIB), "run python -m paper_conf_micro_leebsro14_b200.build"
    lib = ctypes.CDLL(LIB)
    for s in declared_symbols():
        assert hasattr(lib, s), s


def test_struct_layout_matches_binding():
    from paper_conf_micro_leebsro14_b200 import npp
    assert ctypes.sizeof(npp.Level) == 40
    assert ctypes.sizeof(npp.Mapping) == 16 + 4 * 40 + 32 + 12 + 4 + 8 + 8
    assert ctypes.sizeof(npp.Limits) == 4 * 12 + 8
    assert npp.lib().npp_version() == 1
    assert set(npp.EXPORTS) == set(declared_symbols())


def test_no_gpu_calls_fail_cleanly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    from paper_conf_micro_leebsro14_b200 import npp
    with pytest.raises(npp.NppError) as e:
        npp.limits_query(0)
    assert e.value.status == npp.ERR_CUDA
