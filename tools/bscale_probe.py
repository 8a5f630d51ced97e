import sys, numpy as np, torch
sys.path.insert(0, '/root/repo')
from paper_conf_sc_panzzxwslr0d24_b200 import synth
from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan, l2_flush
dev = torch.device('cuda', 0)
m = synth.make_model('heavy')
phys = [torch.empty((r, d), device=dev) for r, d in m.tables]
tables = [phys[f.table] for f in m.features]
flush = torch.empty(64 << 20, device=dev)
for B in (8192, 16384, 24576):
    b = synth.make_batch(m, 7, B=B)
    alg = synth.algorithmic_bytes(m, b)['total']
    bi, bo = torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev)
    out = torch.empty((B, m.d_tot), device=dev)
    plan = Plan.from_model(m, max_batch=B)
    for sid in (16,):
        for k in (4,):
            for f in range(m.F):
                plan.set_schedule(f, sid, 0, 40)
            plan.occupancy = k
            ts = []
            for r in range(6):
                l2_flush(flush)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(); plan.forward(bi, bo, B, tables, out=out); e1.record(); torch.cuda.synchronize()
                if r: ts.append(e0.elapsed_time(e1))
            ms = float(np.median(ts))
            print(f'B={B} sched {sid} k{k}: {ms:.3f} ms {alg/ms/1e6:.0f} GB/s', flush=True)
    del bi, bo, out, plan
