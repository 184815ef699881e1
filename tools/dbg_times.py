import os, sys
sys.path.insert(0, '/root/repo')
import torch
from paper_conf_micro_leebsro14_b200 import npp
from synth import gen
dev = torch.device('cuda:0')
for (R, C) in [(65536,1024),(8192,8192),(1024,65536)]:
    bufs = [gen.uniform_f32(50+i, (R, C), device=dev) for i in range(3)]
    for pat in ('SUM_ROWS','SUM_COLS'):
        p = npp.Plan(pat, (R, C), 'f32', 'AUTO'); out = p.new_out()
        print(pat, R, C, flush=True)
        for i in range(4):
            p.execute([bufs[i % 3]], out)
        torch.cuda.synchronize()
