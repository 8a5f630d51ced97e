"""Run every BULK entry at every occupancy on a small long-bag model (debug)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_sc_panzzxwslr0d24_b200 import synth
from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan, catalog
import oracle
dev = torch.device('cuda', 0)
feats = [synth.Feature(rows=20000, dim=d, pool=i % 2, kind='lognormal', mu=60, sigma=0.9, coverage=0.9, lmax=400, table=i)
         for i, d in enumerate([128, 64, 32, 128, 96])]
m = synth.custom_model('bulkdbg', feats, 512)
b = synth.make_batch(m, 3)
tabs = [synth.make_table(f.table, f.rows, f.dim, 'int', device=dev) for f in m.features]
bi, bo = torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev)
ref = oracle.embedding_bag([t.cpu().numpy() for t in tabs], m.dims, [f.pool for f in m.features], b.indices, b.offsets, b.B)
for e in [e for e in catalog() if e['family'] == 'bulk']:
    for k in range(1, 9):
        plan = Plan.from_model(m)
        for f in range(m.F):
            plan.set_schedule(f, e['id'], 0, 64)
        plan.occupancy = k
        t = time.time()
        out = plan.forward(bi, bo, b.B, tabs)
        torch.cuda.synchronize()
        ok = np.array_equal(out.cpu().numpy(), ref.astype(np.float32))
        print(e['id'], 'U', e['U'], 'k', k, 'ok' if ok else 'MISMATCH', '%.1f ms' % ((time.time() - t) * 1e3), flush=True)
