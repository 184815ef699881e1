"""Time KMEANS_UPDATE (CUDA events, warm, 10 launches per shape; inputs > L2):
    python tools/time_kmupdate.py   -> per shape: us, GB/s of (x + keys)"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_micro_leebsro14_b200 import npp  # noqa: E402
from synth import gen  # noqa: E402

SHAPES = [(1 << 22, 64, 32), (1 << 22, 32, 64), (1 << 22, 16, 128), (1 << 22, 8, 256)]


def main():
    dev = torch.device("cuda:0")
    for N, D, K in SHAPES:
        x, _ = gen.kmeans_inputs(N, D, K, device=dev)
        keys = gen.int_uniform(9, (N,), 0, K - 1, dtype=torch.int32, device=dev)
        p = npp.Plan("KMEANS_UPDATE", (N, D, K), "f32", "AUTO")
        out = p.new_out()
        for _ in range(3):
            p.execute([x, keys], out)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        reps = 10
        e0.record()
        for _ in range(reps):
            p.execute([x, keys], out, pdl=False)
        e1.record()
        torch.cuda.synchronize()
        us = e0.elapsed_time(e1) * 1e3 / reps
        print(f"N={N} D={D} K={K}: {us:9.1f} us  {N * (D + 1) * 4 / us / 1e3:7.1f} GB/s", flush=True)


if __name__ == "__main__":
    main()
