import sys, numpy as np, torch
import os; sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_panzzxwslr0d24_b200 import synth
from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan, l2_flush
dev = torch.device('cuda', 0)
phys = [torch.empty((10_000_000, 128), device=dev) for _ in range(16)]
flush = torch.empty(64 << 20, device=dev)
for lmax in (1000, 300, 150):
    feats = [synth.Feature(rows=10_000_000, dim=128, pool=0, kind='lognormal', mu=100, sigma=0.9, lmax=lmax, table=f % 16) for f in range(100)]
    m = synth.custom_model(f'tail{lmax}', feats, 8192)
    b = synth.make_batch(m, 7)
    bi, bo = torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev)
    out = torch.empty((8192, m.d_tot), device=dev)
    plan = Plan.from_model(m)
    for f in range(m.F): plan.set_schedule(f, 16, 0, 40)
    plan.occupancy = 4
    ts = []
    for r in range(8):
        l2_flush(flush)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); plan.forward(bi, bo, 8192, [phys[f.table] for f in m.features], out=out); e1.record(); torch.cuda.synchronize()
        if r >= 2: ts.append(e0.elapsed_time(e1))
    ms = float(np.median(ts)); print(f'lmax {lmax}: nnz {b.nnz/1e6:.1f} M, {ms:.3f} ms, {b.nnz/ms/1e6:.2f} G rows/s, max L {int(b.lengths().max())}', flush=True)
