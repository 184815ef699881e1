"""GPU tests of library robustness: per-device kernel attributes, launch flags, explicit-mapping limits
and the per-stream plan cache of the Python front-ends."""
import numpy as np
import pytest
import torch

from oracle import sums
from synth import gen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def npp(cuda_device):
    from paper_conf_micro_leebsro14_b200 import npp as _npp
    return _npp


def _close(got, want, scale):
    return np.all(np.abs(got.astype(np.float64) - want) <= 1e-5 * scale)


def test_rx_explicit_block_must_suit_the_shuffle(npp, cuda_device):
    # class RX reduces a row with xor-shuffles over min(b_x, 32) lanes: b_x = 48 or 3 would mix rows
    shape = (64, 4096)
    m = gen.uniform_f32(3, shape, device=cuda_device)
    base = npp.Plan("SUM_ROWS", shape, "f32", "TB_T").mapping
    for bx in (48, 3, 24):
        bad = dict(base, levels=[dict(base["levels"][0], block=1), dict(base["levels"][1], block=bx)])
        with pytest.raises(npp.NppError) as e:
            npp.Plan("SUM_ROWS", shape, "f32", mapping=bad)
        assert e.value.status == npp.ERR_UNSUPPORTED
    for bx in (1, 2, 16, 32, 96, 160):
        ok = dict(base, levels=[dict(base["levels"][0], block=2), dict(base["levels"][1], block=bx)])
        p = npp.Plan("SUM_ROWS", shape, "f32", mapping=ok)
        out = p.execute([m], p.new_out())
        torch.cuda.synchronize()
        mn = m.cpu().numpy()
        assert _close(out.cpu().numpy(), sums.sum_rows(mn), sums.sum_abs_rows(mn)), bx


def test_launch_flags(npp, cuda_device):
    shape = (8192, 8192)
    m = gen.uniform_f32(5, shape, device=cuda_device)
    mn = m.cpu().numpy()
    for pattern in ("SUM_ROWS", "SUM_COLS", "SUM_ROWS_COLS"):
        p = npp.Plan(pattern, shape, "f32", "AUTO")
        for kw in (dict(pdl=False), dict(overlap=True), dict()):
            out = p.execute([m], p.new_out(), **kw)
            torch.cuda.synchronize()
            if pattern == "SUM_ROWS_COLS":
                want = np.concatenate([sums.sum_rows(mn), sums.sum_cols(mn)])
                scale = np.concatenate([sums.sum_abs_rows(mn), sums.sum_abs_cols(mn)])
            elif pattern == "SUM_ROWS":
                want, scale = sums.sum_rows(mn), sums.sum_abs_rows(mn)
            else:
                want, scale = sums.sum_cols(mn), sums.sum_abs_cols(mn)
            assert _close(out.cpu().numpy(), want, scale), (pattern, kw)
        with pytest.raises(npp.NppError) as e:
            p.execute([m], p.new_out(), overlap=True, pdl=False)
        assert e.value.status == npp.ERR_INVALID_ARG


def test_front_end_plan_per_stream(npp, cuda_device):
    # two streams running the same shape concurrently must not share one workspace
    shape = (8192, 8192)
    a = gen.uniform_f32(6, shape, device=cuda_device)
    b = gen.uniform_f32(7, shape, device=cuda_device)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    torch.cuda.synchronize()
    outs = []
    for _ in range(20):
        outs.append((npp.sum_cols(a, stream=s1), npp.sum_cols(b, stream=s2)))
    torch.cuda.synchronize()
    wa, wb = sums.sum_cols(a.cpu().numpy()), sums.sum_cols(b.cpu().numpy())
    for oa, ob in outs:
        assert _close(oa.cpu().numpy(), wa, wa) and _close(ob.cpu().numpy(), wb, wb)


@pytest.mark.skipif(not torch.cuda.is_available() or torch.cuda.device_count() < 2, reason="needs 2 GPUs")
def test_two_devices_one_process(npp):
    # kernel attributes (dynamic shared memory) are per device: plan and execute on both from one process
    for dev in (0, 1):
        d = torch.device("cuda", dev)
        with torch.cuda.device(d):
            for pattern, shape in [("SUM_COLS", (8192, 8192)), ("SUM_ROWS", (1024, 65536))]:
                m = gen.uniform_f32(8, shape, device=d)
                p = npp.Plan(pattern, shape, "f32", "AUTO", device=d)
                out = p.execute([m], p.new_out())
                torch.cuda.synchronize(d)
                mn = m.cpu().numpy()
                want = sums.sum_cols(mn) if pattern == "SUM_COLS" else sums.sum_rows(mn)
                assert _close(out.cpu().numpy(), want, want)
