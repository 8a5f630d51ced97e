"""Run the tuner once on a small config (debug helper for gpurun)."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sc_panzzxwslr0d24_b200 import synth
from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan

name = sys.argv[1] if len(sys.argv) > 1 else 'fig3'
ks = [int(x) for x in sys.argv[2].split(',')] if len(sys.argv) > 2 else [2, 4, 8]
m = synth.make_model(name)
dev = torch.device('cuda', 0)
phys = [synth.make_table(t, r, d, 'float', device=dev) for t, (r, d) in enumerate(m.tables)]
tables = [phys[f.table] for f in m.features]
bts = [synth.make_batch(m, 7 + i) for i in range(2)]
hist = [(torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev), b.B) for b in bts]
plan = Plan.from_model(m)
out = plan.forward(hist[0][0], hist[0][1], hist[0][2], tables)
torch.cuda.synchronize()
print('forward ok', flush=True)
t = time.time()
st = plan.tune(hist, tables, occupancies=ks, reps=3, verbose=True)
print('tune', st, time.time() - t)
print(plan.export())
