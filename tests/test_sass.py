"""The built sm_100a code uses the instructions the design depends on (checked here, without a GPU,
from `cuobjdump -sass` of the in-tree library): a compiler heuristic that silently picks a slower
instruction form would otherwise only show up as a lower bench number.

- staged sums / logreg / k-means move their tiles with TMA (UTMALDG) — DESIGN.md §6;
- k-means reads centroids on the uniform datapath (LDCU into uniform registers feeding FFMA2), not
  per-thread LDC, which measured ~5x slower in tools/micro_const.cu;
- the ALU-bound x·c products run on the packed FP32 pipe (FFMA2).
"""
import collections
import os
import re
import shutil
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_micro_leebsro14_b200", "libnpp.so")
CUOBJDUMP = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"

pytestmark = pytest.mark.skipif(not os.path.exists(CUOBJDUMP), reason="cuobjdump not available")


@pytest.fixture(scope="module")
def sass():
    assert os.path.exists(LIB), "run python -m paper_conf_micro_leebsro14_b200.build"
    out = subprocess.run([CUOBJDUMP, "-sass", LIB], capture_output=True, text=True, check=True).stdout
    funcs, name = collections.defaultdict(collections.Counter), None
    for line in out.splitlines():
        m = re.search(r"Function : (\S+)", line)
        if m:
            name = m.group(1)
            continue
        m = re.match(r"\s+/\*[0-9a-f]+\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_.]*)", line)
        if m and name:
            funcs[name][m.group(1)] += 1
            if m.group(1).startswith("LDC") and "c[0x3]" in line:  # user __constant__ bank (not params)
                funcs[name][m.group(1) + "@bank3"] += 1
    return funcs


def _find(sass, *parts):
    names = [n for n in sass if all(p in n for p in parts)]
    assert names, parts
    return names


def test_all_kernels_built_for_sm100a():
    out = subprocess.run([CUOBJDUMP, "-lelf", LIB], capture_output=True, text=True, check=True).stdout
    archs = set(re.findall(r"sm_\d+a?", out))
    assert archs == {"sm_100a"}, archs


def test_staged_kernels_use_tma(sass):
    for parts in (("npp_sum_tma_kernel",), ("npp_logreg_tma_kernel",), ("npp_kmeans_tma_kernel",)):
        for n in _find(sass, *parts):
            assert sum(sass[n][f"UTMALDG.{d}D"] for d in (1, 2, 3)) + sass[n]["UBLKCP.S.G"] > 0, n


def test_kmeans_centroids_on_uniform_datapath(sass):
    for n in _find(sass, "npp_kmeans_tma_kernel"):
        c = sass[n]
        ffma2 = c["FFMA2"]
        assert ffma2 >= 64, (n, ffma2)
        # centroid operand pairs come from uniform registers (at least one LDCU.64 per 8 FFMA2; the D > 64
        # kernel takes some pairs from a broadcast shared-memory copy) and never from per-thread constant
        # loads
        assert c["LDCU.64"] + 2 * c["LDCU.128"] >= ffma2 // 8, (n, dict(c))
        assert c["LDC.64@bank3"] + c["LDC@bank3"] + c["LDC.128@bank3"] == 0, (n, dict(c))


def test_packed_fma_in_kmeans(sass):
    for n in _find(sass, "npp_kmeans_tma_kernel"):
        assert sass[n]["FFMA2"] >= 2 * sass[n]["FFMA"], (n, sass[n]["FFMA2"], sass[n]["FFMA"])


def test_new_staged_families_use_tma(sass):
    # the one-pass rows+cols (staged variant) and the k-means update stream their tiles with TMA; the
    # rows+cols direct variant (ragged row pitch) has no tensor map and loads with LDG instead
    for n in _find(sass, "npp_rowscols_kernel"):
        tma = sum(sass[n][f"UTMALDG.{d}D"] for d in (1, 2, 3))
        if "Lb1E" in n:   # STAGED = true
            assert tma > 0, n
        else:
            assert tma == 0 and sum(v for k, v in sass[n].items() if k.startswith("LDG")) > 0, n
    for n in _find(sass, "npp_kmupdate_kernel"):
        assert sass[n]["UTMALDG.2D"] > 0 and sass[n]["UTMALDG.1D"] > 0, n


def test_slot_tags_use_native_shared_atomics(sass):
    # the staged sums hand slot tags over with 32-bit shared atomics (racecheck-visible); a 64-bit form
    # compiles to a CAS loop (ATOMS.CAST.SPIN), which the design avoids
    for n in _find(sass, "npp_sum_tma_kernel"):
        assert sass[n]["ATOMS.CAST.SPIN.64"] == 0 and sass[n]["ATOMS.EXCH"] > 0, (n, dict(sass[n]))
