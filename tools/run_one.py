"""Run one plan a few times (for ncu captures): python tools/run_one.py logreg|kmeans|sumrows|sumcols|rowscols [args]"""
import sys
sys.path.insert(0, '/root/repo')
import torch
from paper_conf_micro_leebsro14_b200 import npp
from synth import gen
what = sys.argv[1]
dev = torch.device('cuda:0')
if what == 'logreg':
    B = int(sys.argv[2]) if len(sys.argv) > 2 else 512
    x, y, w = gen.logreg_inputs(B, 4096, 256, device=dev)
    p = npp.Plan('LOGREG_GRAD', (B, 4096, 256), 'f32', 'AUTO'); ins = [x, y, w]
elif what == 'kmeans':
    N = int(sys.argv[2]) if len(sys.argv) > 2 else (1 << 22)
    x, c = gen.kmeans_inputs(N, 64, 32, device=dev)
    p = npp.Plan('KMEANS_ASSIGN', (N, 64, 32), 'f32', 'AUTO'); ins = [x, c]
else:
    R, C = (int(v) for v in sys.argv[2].split('x'))
    m = gen.uniform_f32(1, (R, C), device=dev)
    pat = {'sumrows': 'SUM_ROWS', 'sumcols': 'SUM_COLS', 'rowscols': 'SUM_ROWS_COLS'}[what]
    p = npp.Plan(pat, (R, C), 'f32', 'AUTO'); ins = [m]
out = p.new_out()
for _ in range(4):
    p.execute(ins, out)
torch.cuda.synchronize()
print('done', what)
