"""Per-block timelines of the staged sums launched back to back (no PDL) from a CUDA graph — needs the
measurement build `python -m paper_conf_micro_leebsro14_b200.build -DNPP_SUM_STAMPS --out=LIB` loaded
through NPP_LIB_PATH=LIB. For three consecutive launches it prints, in us after the launch's first block
start: the gap from the previous launch's last block end, the first tile's arrival (min..max over
blocks), the consumers' stream end (p10 / p50 / max) and the combiner's end (max)."""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_micro_leebsro14_b200 import npp  # noqa: E402
from synth import gen  # noqa: E402

SHAPES = [(65536, 1024), (8192, 8192), (1024, 65536)]
NL, NBUF = 20, 8


def read_stamps():
    buf = (ctypes.c_ulonglong * (32 * 256 * 4))()
    rc = npp._lib.npp_debug_sum_stamps(buf)
    assert rc == 0, rc
    return np.frombuffer(buf, dtype=np.uint64).reshape(32, 256, 4).astype(np.int64)


def main():
    npp._lib.npp_debug_sum_stamps.argtypes = [ctypes.c_void_p]
    dev = torch.device("cuda:0")
    launches = 0
    for R, C in SHAPES:
        bufs = [gen.uniform_f32(70 + i, (R, C), device=dev) for i in range(NBUF)]
        for pattern in ("SUM_ROWS", "SUM_COLS"):
            p = npp.Plan(pattern, (R, C), "f32", "AUTO")
            G = p.mapping["grid"]
            assert G == 148
            out = p.new_out()
            for i in range(3):
                p.execute([bufs[i]], out, pdl=False)
                launches += 1
            s = torch.cuda.Stream()
            s.wait_stream(torch.cuda.current_stream())
            g = torch.cuda.CUDAGraph()
            with torch.cuda.stream(s):
                with torch.cuda.graph(g, stream=s):
                    for i in range(NL):
                        p.execute([bufs[i % NBUF]], out, stream=s, pdl=False)
            for _ in range(3):
                g.replay()
                launches += NL
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            g.replay()
            b.record()
            launches += NL
            torch.cuda.synchronize()
            us = a.elapsed_time(b) * 1e3 / NL
            st = read_stamps()
            print(f"{pattern} [{R},{C}] graph b2b {us:.2f} us  {R * C * 4 / us / 1e3:.1f} GB/s", flush=True)
            for L in (launches - 10, launches - 9, launches - 8):
                cur, prv = st[L % 32, :G], st[(L - 1) % 32, :G]
                s0 = cur[:, 0].min()
                prev_end = np.maximum(prv[:, 2], prv[:, 3]).max()
                ends = np.sort(cur[:, 2])
                print(f"   gap {(s0 - prev_end) / 1e3:5.2f} | start spread {(cur[:, 0].max() - s0) / 1e3:4.2f} | "
                      f"first tile {(cur[:, 1].min() - s0) / 1e3:5.2f}..{(cur[:, 1].max() - s0) / 1e3:5.2f} | "
                      f"stream end p10 {(ends[G // 10] - s0) / 1e3:6.2f} p50 {(ends[G // 2] - s0) / 1e3:6.2f} "
                      f"max {(ends[-1] - s0) / 1e3:6.2f} | combiner end max {(cur[:, 3].max() - s0) / 1e3:6.2f}",
                      flush=True)
        del bufs


if __name__ == "__main__":
    main()
