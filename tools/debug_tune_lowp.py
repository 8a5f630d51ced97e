"""Debug: tuner on a mixed-dtype medium plan with verbose progress (stderr)."""
import os, sys, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, 'tests'))
import torch
from paper_conf_sc_panzzxwslr0d24_b200 import synth
from test_gpu_lowp import TypedCase, _mixed_dtypes
m = synth.make_model(sys.argv[1] if len(sys.argv) > 1 else 'medium')
bts = [synth.make_batch(m, 7 + i) for i in range(2)]
case = TypedCase(m, bts[0], _mixed_dtypes(m) if len(sys.argv) <= 2 else sys.argv[2], 'int')
plan = case.plan()
hist = [(torch.from_numpy(b.indices).cuda(), torch.from_numpy(b.offsets).cuda(), b.B) for b in bts]
t0 = time.time()
st = plan.tune(hist, case.tables, occupancies=[2, 4], reps=3, verbose=True)
print('tuned', time.time() - t0, st, flush=True)
