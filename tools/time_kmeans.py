"""Time KMEANS_ASSIGN over several (N, D, K) shapes (CUDA events, graph-free, warm):
    python tools/time_kmeans.py            -> one line per shape: us, TFLOP/s (2·N·K·D), GB/s of x"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_micro_leebsro14_b200 import npp  # noqa: E402
from synth import gen  # noqa: E402

SHAPES = [(1 << 22, 64, 32), (1 << 22, 32, 32), (1 << 22, 64, 256), (1 << 21, 128, 128), (1 << 22, 16, 64),
          (1 << 21, 96, 32)]


def main():
    dev = torch.device("cuda:0")
    for N, D, K in SHAPES:
        x, c = gen.kmeans_inputs(N, D, K, device=dev)
        p = npp.Plan("KMEANS_ASSIGN", (N, D, K), "f32", "AUTO")
        out = p.new_out()
        for _ in range(3):
            p.execute([x, c], out)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        reps = 10
        e0.record()
        for _ in range(reps):
            p.execute([x, c], out)
        e1.record()
        torch.cuda.synchronize()
        us = e0.elapsed_time(e1) * 1e3 / reps
        neg = int((out < 0).sum())  # NPP_KM_MARK_FLAGS builds: points the fp32 bound could not settle
        print(f"N={N} D={D} K={K}: {us:9.1f} us  {2 * N * K * D / us / 1e6:6.2f} TFLOP/s  "
              f"{N * D * 4 / us / 1e3:7.1f} GB/s  flagged={neg}", flush=True)


if __name__ == "__main__":
    main()
