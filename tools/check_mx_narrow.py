"""MX-narrow strips (SUM_COLS, row pitch >= 64 KB, R <= 1024): parity on ragged shapes, back-to-back and PDL executes, workspace left zero."""
import sys, os
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import numpy as np, torch
from paper_conf_micro_leebsro14_b200 import npp
from oracle import sums
from synth import gen
dev = torch.device("cuda:0")
for shape in [(1024, 65536), (1000, 70000), (777, 16384), (129, 65536), (1, 1 << 20), (1024, 65540)]:
    for dtype in ("f32", "i32", "i64"):
        m = gen.uniform_f32(3, shape, device=dev) if dtype == "f32" else (gen.int_uniform(3, shape, -1000, 1000, device=dev) if dtype == "i32" else gen.int64_wide(3, shape, device=dev))
        p = npp.Plan("SUM_COLS", shape, dtype)
        o1 = p.execute([m], p.new_out()); o2 = p.execute([m], p.new_out(), overlap=True)
        torch.cuda.synchronize()
        want = sums.sum_cols(m.cpu().numpy())
        for o in (o1, o2):
            g = o.cpu().numpy()
            ok = np.allclose(g, want, rtol=1e-5) if dtype == "f32" else np.array_equal(g.astype(np.int64), want.astype(np.int64))
            assert ok, (shape, dtype)
        assert int(p.workspace.count_nonzero()) == 0, (shape, dtype)
        print(shape, dtype, "ok", p.mapping["levels"][0]["chunk"], p.mapping["grid"])
