"""Heavy-config structure experiments: which part of the workload structure
costs bandwidth (bag-length variance, bag transitions, feature count)?

    python tools/heavy_variants.py
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def run(model, label, ids=(15, 16), ks=(4, 6), reps=5):
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan, l2_flush
    dev = torch.device('cuda', 0)
    phys = [synth.make_table(t, r, d, 'float', device=dev) for t, (r, d) in enumerate(model.tables)]
    tables = [phys[f.table] for f in model.features]
    b = synth.make_batch(model, 7)
    alg = synth.algorithmic_bytes(model, b)['total']
    bi, bo = torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev)
    out = torch.empty((model.batch, model.d_tot), device=dev)
    flush = torch.empty(64 << 20, device=dev)
    plan = Plan.from_model(model)
    for sid in ids:
        for f in range(model.F):
            plan.set_schedule(f, sid, 0, 40)
        for k in ks:
            plan.occupancy = k
            ts = []
            for r in range(reps + 1):
                l2_flush(flush)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                plan.forward(bi, bo, model.batch, tables, out=out)
                e1.record()
                torch.cuda.synchronize()
                if r:
                    ts.append(e0.elapsed_time(e1))
            ms = float(np.median(ts))
            print(f'{label:40s} sched {sid} k{k}: {ms:7.3f} ms  {alg / ms / 1e6:6.0f} GB/s', flush=True)
    del phys, tables
    torch.cuda.empty_cache()


def base_heavy():
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    return synth.make_model('heavy')


def main():
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    if len(sys.argv) > 2 and sys.argv[1] == 'heavy':  # one short run of heavy on one schedule (for ncu)
        run(base_heavy(), 'heavy', ids=(int(sys.argv[2]),), ks=(int(sys.argv[3]) if len(sys.argv) > 3 else 4,), reps=1)
        return
    if len(sys.argv) > 1 and sys.argv[1] == 'fixedL100':  # one short run (for ncu)
        feats = [synth.Feature(rows=10_000_000, dim=128, pool=0, kind='fixed', mu=100, lmax=100, table=f % 16)
                 for f in range(100)]
        run(synth.custom_model('fixedL100', feats, 8192), 'fixed L=100, 100 fields', ids=(15,), ks=(4,), reps=1)
        return
    base = synth.make_model('heavy')
    run(base, 'heavy (lognormal L, 100 fields)')
    feats = [synth.Feature(rows=10_000_000, dim=128, pool=0, kind='fixed', mu=100, lmax=100, table=f % 16)
             for f in range(100)]
    run(synth.custom_model('fixedL100', feats, 8192), 'fixed L=100, 100 fields')
    feats = [synth.Feature(rows=10_000_000, dim=128, pool=0, kind='fixed', mu=1000, lmax=1000, table=f % 16)
             for f in range(10)]
    run(synth.custom_model('fixedL1000', feats, 8192), 'fixed L=1000, 10 fields')
    feats = [synth.Feature(rows=10_000_000, dim=128, pool=0, kind='lognormal', mu=100, sigma=0.9, lmax=1000,
                           table=0)]
    run(synth.custom_model('onefield', feats, 819200), 'lognormal, 1 field x 819200 samples')
    # table footprint (TLB reach / DRAM page spread): heavy's lengths, 1 and 4 physical tables
    for nt in (1, 4):
        feats = [synth.Feature(rows=10_000_000, dim=128, pool=0, kind='lognormal', mu=100, sigma=0.9, lmax=1000,
                               table=f % nt) for f in range(100)]
        run(synth.custom_model(f'heavy_t{nt}', feats, 8192), f'heavy lengths, {nt} physical table(s)')


if __name__ == '__main__':
    main()
