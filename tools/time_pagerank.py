"""Time one PAGERANK step (CUDA events, isolated launches, warm) on the bench graph (4M nodes, ~63M
edges, power-law in-degrees) and a uniform-degree graph; check the first 64K rows against a float64
recompute in torch (measurement tool, not a parity test: tests/test_gpu_nests.py is the parity test).
    python tools/time_pagerank.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_micro_leebsro14_b200 import npp  # noqa: E402
from synth import gen  # noqa: E402


def main():
    dev = torch.device("cuda:0")
    N = 1 << 22
    for name, kw in (("power-law avg 16 cap 1024", dict(avg_deg=16, max_deg=1024)),
                     ("power-law avg 4 cap 64", dict(avg_deg=4, max_deg=64))):
        rowptr, colidx, pr, outdeg = gen.pagerank_inputs(N, seed=7, device=dev, **kw)
        E = colidx.numel()
        p = npp.Plan("PAGERANK", (N, E), "f32", "AUTO")
        out = p.new_out()
        for _ in range(3):
            p.execute([rowptr, colidx, pr, outdeg], out, pdl=False)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        reps = 10
        e0.record()
        for _ in range(reps):
            p.execute([rowptr, colidx, pr, outdeg], out, pdl=False)
        e1.record()
        torch.cuda.synchronize()
        us = e0.elapsed_time(e1) * 1e3 / reps
        n = 1 << 16
        contrib = pr.double() / outdeg.double().clamp(min=1)
        m = int(rowptr[n])
        rows = torch.repeat_interleave(torch.arange(n, device=dev), (rowptr[1:n + 1] - rowptr[:n]))
        ref = torch.zeros(n, dtype=torch.float64, device=dev).index_add_(0, rows, contrib[colidx[:m].long()])
        ref = (1 - 0.85) / N + 0.85 * ref
        err = float(((out[:n].double() - ref).abs() / ref.abs()).max())
        print(f"{name}: E={E}  {us:8.1f} us  {E / us / 1e3:6.1f} G edges/s  max rel err (64K rows) {err:.2e}",
              flush=True)


if __name__ == "__main__":
    main()
