"""Small forwards for compute-sanitizer (memcheck / racecheck / synccheck / initcheck)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_sc_panzzxwslr0d24_b200 import synth  # noqa: E402
from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan, catalog  # noqa: E402

dev = torch.device('cuda', 0)
feats = []
dims = [4, 8, 12, 16, 32, 64, 128, 3]
for i, d in enumerate(dims):
    kind = 'onehot' if i % 3 == 0 else 'uniform'
    feats.append(synth.Feature(rows=500 + i, dim=d, pool=i % 2, kind=kind, coverage=0.7, lo=0, hi=40,
                               lmax=1 if kind == 'onehot' else 40, table=i))
m = synth.custom_model('san', feats, 96)
b = synth.make_batch(m, 3)
phys = [synth.make_table(t, r, d, 'int', device=dev) for t, (r, d) in enumerate(m.tables)]
tables = [phys[f.table] for f in m.features]
bi, bo = torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev)
cat = catalog()
fams = sys.argv[1:] or ['group', 'flat', 'block']
for fam in fams:
    ids = [e['id'] for e in cat if e['family'] == fam]
    plan = Plan.from_model(m)
    plan.occupancy = 8 if fam != 'block' else 4
    n = 0
    for sid in ids[::3]:
        for part in (0, 1):
            for f in range(m.F):
                try:
                    plan.set_schedule(f, sid, part, 16 if part == 0 else 128)
                except Exception:
                    pass
            plan.forward(bi, bo, b.B, tables)
            n += 1
    torch.cuda.synchronize()
    print(fam, 'forwards', n)
