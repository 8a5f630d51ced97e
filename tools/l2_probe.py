"""L2 eviction-priority probe (reading C36): time a config's tuned plan in its
plan-specialised kernel under several per-feature L2 policies (CUDA events,
L2 flushed, median over rotating batches).

    python tools/l2_probe.py sharded1000 [--variants none,heuristic,first_only,last_only]
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument('config')
    ap.add_argument('--variants', default='none,heuristic,first_only,last_only')
    ap.add_argument('--l2-mb', type=float, default=126.0)
    ap.add_argument('--reps', type=int, default=30)
    a = ap.parse_args()
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan, l2_flush
    dev = torch.device('cuda', 0)
    m = synth.make_model(a.config)
    phys = [synth.make_table(t, r, d, 'float', device=dev, seed=m.seed) for t, (r, d) in enumerate(m.tables)]
    tables = [phys[f.table] for f in m.features]
    bts = [synth.make_batch(m, 7 + i) for i in range(3)]
    dev_b = [(torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev)) for b in bts]
    out = torch.empty((m.batch, m.d_tot), device=dev)
    flush = torch.empty(64 << 20, device=dev)
    plan = Plan.from_model(m)
    path = os.path.join(ROOT, 'configs', 'tuned', f'{a.config}_w1_r0.json')
    if os.path.exists(path):
        plan.import_(json.load(open(path)))
    heur = plan.l2_policy_heuristic(int(a.l2_mb * 2 ** 20))
    pols = {'none': None, 'heuristic': heur,
            'first_only': [1 if p == 1 else 0 for p in heur],
            'last_only': [2 if p == 2 else 0 for p in heur],
            'all_first': [1] * m.F, 'all_last': [2] * m.F}
    # rows of tables up to X MB with >= 1 lookup per row per batch also allocate in L1 (policy 3)
    for mb in (1, 4, 16):
        pol = list(heur)
        for f, feat in enumerate(m.features):
            tb = feat.rows * feat.dim * 4
            if tb <= mb * 2 ** 20 and m.batch * feat.mean_len() * feat.coverage >= feat.rows:
                pol[f] = 3
        pols[f'l1_{mb}mb'] = pol
    print(json.dumps(dict(config=a.config, heuristic_counts={k: heur.count(i) for i, k in
                                                             enumerate(Plan.L2_POLICIES)})), flush=True)
    for name in a.variants.split(','):
        plan.l2_policy = pols[name]
        info = plan.compile()
        ts = []
        for r in range(a.reps + 2):
            l2_flush(flush)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            plan.forward(*dev_b[r % 3], m.batch, tables, out=out)
            e1.record()
            torch.cuda.synchronize()
            if r >= 2:
                ts.append(e0.elapsed_time(e1))
        print(json.dumps(dict(config=a.config, l2=name, k=plan.occupancy, ms=round(float(np.median(ts)), 4),
                              min_ms=round(float(np.min(ts)), 4), regs=info['registers'],
                              variants=info['variants'])), flush=True)


if __name__ == '__main__':
    main()
