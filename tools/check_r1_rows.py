"""RX one-row tiles (SUM_ROWS, row pitch 64-256 KB, a multiple of 32 KB): parity on several shapes and
dtypes, back-to-back and PDL executes, workspace left zero."""
import os
import sys
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import numpy as np
import torch
from paper_conf_micro_leebsro14_b200 import npp
from oracle import sums
from synth import gen
dev = torch.device("cuda:0")
for shape in [(1024, 65536), (1000, 16384), (3, 65536), (4099, 24576), (1, 65536)]:
    for dtype in ("f32", "i32", "i64"):
        C = shape[1] if dtype != "i64" else shape[1] // 2
        sh = (shape[0], C)
        m = gen.uniform_f32(3, sh, device=dev) if dtype == "f32" else (gen.int_uniform(3, sh, -1000, 1000, device=dev) if dtype == "i32" else gen.int64_wide(3, sh, device=dev))
        p = npp.Plan("SUM_ROWS", sh, dtype)
        o1 = p.execute([m], p.new_out()); o2 = p.execute([m], p.new_out(), overlap=True)
        torch.cuda.synchronize()
        want = sums.sum_rows(m.cpu().numpy())
        for o in (o1, o2):
            g = o.cpu().numpy()
            ok = np.allclose(g, want, rtol=1e-5) if dtype == "f32" else np.array_equal(g.astype(np.int64), want.astype(np.int64))
            assert ok, (sh, dtype)
        assert int(p.workspace.count_nonzero()) == 0, (sh, dtype)
        print(sh, dtype, "ok", p.mapping["levels"][0]["chunk"], p.mapping["levels"][1]["chunk"], p.mapping["grid"])
