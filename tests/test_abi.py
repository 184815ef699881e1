"""The C-ABI library loads on a GPU-less box and exports every symbol include/npp.h declares."""
import ctypes
import os
import re
import shutil
import subprocess

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


def _c_layout(tmp_path, struct, fields):
    """sizeof/offsetof of a struct of include/npp.h as the C compiler lays it out."""
    src = tmp_path / "layout.c"
    body = "".join(f'  printf("%zu\\n", offsetof({struct}, {f}));\n' for f in fields)
    src.write_text(f'#include <stddef.h>\n#include <stdio.h>\n#include "npp.h"\n'
                   f'int main(void) {{\n  printf("%zu\\n", sizeof({struct}));\n{body}  return 0;\n}}\n')
    exe = tmp_path / "layout"
    subprocess.run(["gcc", "-std=c99", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)], check=True)
    vals = [int(v) for v in subprocess.run([str(exe)], capture_output=True, text=True, check=True).stdout.split()]
    return vals[0], vals[1:]


@pytest.mark.skipif(shutil.which("gcc") is None, reason="gcc not available")
def test_struct_layout_matches_binding(tmp_path):
    # the ctypes mirrors of npp_level / npp_mapping / npp_limits have the C compiler's layout
    from paper_conf_micro_leebsro14_b200 import npp
    for struct, cls in (("npp_level", npp.Level), ("npp_mapping", npp.Mapping), ("npp_limits", npp.Limits)):
        names = [f[0] for f in cls._fields_]
        size, offs = _c_layout(tmp_path, struct, names)
        assert ctypes.sizeof(cls) == size, struct
        assert [getattr(cls, n).offset for n in names] == offs, struct
    assert npp.lib().npp_version() == 4
    assert set(npp.EXPORTS) == set(declared_symbols())


def test_no_gpu_calls_fail_cleanly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    from paper_conf_micro_leebsro14_b200 import npp
    with pytest.raises(npp.NppError) as e:
        npp.limits_query(0)
    assert e.value.status == npp.ERR_CUDA


@pytest.mark.skipif(shutil.which("gcc") is None, reason="gcc not available")
def test_enum_values_match_binding(tmp_path):
    # every pattern / kernel-class / strategy constant of the binding equals the header's enum value
    from paper_conf_micro_leebsro14_b200 import npp
    names = ([f"NPP_{k}" for k in npp.PATTERNS] +
             ["NPP_CLASS_RX", "NPP_CLASS_MX", "NPP_CLASS_KMEANS", "NPP_CLASS_LOGREG", "NPP_CLASS_EMPTY",
              "NPP_CLASS_RC", "NPP_CLASS_KMUPDATE", "NPP_CLASS_PAGERANK"] +
             ["NPP_MAP_AUTO", "NPP_MAP_LITERAL", "NPP_MAP_1D", "NPP_MAP_TB_THREAD", "NPP_MAP_WARP"])
    src = tmp_path / "enums.c"
    body = "".join(f'  printf("%d\\n", (int){n});\n' for n in names)
    src.write_text(f'#include <stdio.h>\n#include "npp.h"\nint main(void) {{\n{body}  return 0;\n}}\n')
    exe = tmp_path / "enums"
    subprocess.run(["gcc", "-std=c99", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)], check=True)
    vals = [int(v) for v in subprocess.run([str(exe)], capture_output=True, text=True, check=True).stdout.split()]
    want = (list(npp.PATTERNS.values()) +
            [npp.CLASS_RX, npp.CLASS_MX, npp.CLASS_KMEANS, npp.CLASS_LOGREG, npp.CLASS_EMPTY, npp.CLASS_RC,
             npp.CLASS_KMUPDATE, npp.CLASS_PAGERANK] +
            [npp.STRATEGIES[k] for k in ("AUTO", "LITERAL", "1D", "TB_T", "WARP")])
    assert vals == want
