import sys
sys.path.insert(0, '/root/repo')
import torch
from paper_conf_micro_leebsro14_b200 import npp
from synth import gen
x, y, w = gen.logreg_inputs(1, 1000, 256, device='cuda')
p = npp.Plan("LOGREG_GRAD", (1, 1000, 256), "f32", "AUTO")
try:
    g = p.execute([x, y, w], p.new_out()); torch.cuda.synchronize(); print("ok", g[0, :4])
except Exception as e:
    print("ERR", e)
