"""Time individual plans back-to-back on rotating input buffers (inputs > L2), CUDA events.

    python tools/time_plans.py [--strategy AUTO] [--iters 40] [--shapes 65536x1024,...] [--patterns ...]

Measurement tool (not the benchmark contract): isolates one kernel family from the bench step.
"""
import argparse
import time
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_micro_leebsro14_b200 import npp  # noqa: E402
from synth import gen  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--strategy", default="AUTO")
    ap.add_argument("--iters", type=int, default=40)
    ap.add_argument("--nbuf", type=int, default=4)
    ap.add_argument("--shapes", default="65536x1024,8192x8192,1024x65536")
    ap.add_argument("--patterns", default="SUM_ROWS,SUM_COLS")
    ap.add_argument("--dtype", default="f32")
    ap.add_argument("--no-pdl", action="store_true", help="NPP_EXEC_NO_PDL launches (isolated kernel timing)")
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    for sh in args.shapes.split(","):
        R, C = (int(v) for v in sh.split("x"))
        bufs = [gen.uniform_f32(50 + i, (R, C), device=dev) if args.dtype == "f32"
                else gen.int_uniform(50 + i, (R, C), -9, 9, device=dev) for i in range(args.nbuf)]
        for pattern in args.patterns.split(","):
            p = npp.Plan(pattern, (R, C), args.dtype, args.strategy)
            out = p.new_out()
            for i in range(3):
                p.execute([bufs[i % args.nbuf]], out, pdl=not args.no_pdl)
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            t0 = time.perf_counter()
            a.record()
            for i in range(args.iters):
                p.execute([bufs[i % args.nbuf]], out, pdl=not args.no_pdl)
            b.record()
            host_us = (time.perf_counter() - t0) * 1e6 / args.iters
            torch.cuda.synchronize()
            us = a.elapsed_time(b) * 1e3 / args.iters
            # the same launches replayed from a CUDA graph (no host work between kernels)
            s = torch.cuda.Stream()
            s.wait_stream(torch.cuda.current_stream())
            g = torch.cuda.CUDAGraph()
            with torch.cuda.stream(s):
                with torch.cuda.graph(g, stream=s):
                    for i in range(args.iters):
                        p.execute([bufs[i % args.nbuf]], out, stream=s, pdl=not args.no_pdl)
            torch.cuda.synchronize()
            g.replay()
            torch.cuda.synchronize()
            a.record()
            g.replay()
            b.record()
            torch.cuda.synchronize()
            gus = a.elapsed_time(b) * 1e3 / args.iters
            nbytes = R * C * bufs[0].element_size()
            m = p.mapping
            print(f"{pattern:9s} [{R},{C}] {args.strategy:7s} eager {us:8.2f} us {nbytes / us / 1e3:8.1f} GB/s "
                  f"(host {host_us:6.1f} us/call) graph {gus:8.2f} us {nbytes / gus / 1e3:8.1f} GB/s "
                  f"staged={m['staged']} grid={m['grid']} k={m['levels'][1]['grid']}", flush=True)
        del bufs


if __name__ == "__main__":
    main()
