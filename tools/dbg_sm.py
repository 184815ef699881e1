import sys
sys.path.insert(0, '/root/repo')
import torch
from paper_conf_micro_leebsro14_b200 import npp
from synth import gen
dev = torch.device('cuda:0')
R, C = 65536, 1024
bufs = [gen.uniform_f32(50+i, (R, C), device=dev) for i in range(3)]
p = npp.Plan('SUM_ROWS', (R, C), 'f32', 'AUTO'); out = p.new_out()
for i in range(6):
    p.execute([bufs[i % 3]], out)
torch.cuda.synchronize()
