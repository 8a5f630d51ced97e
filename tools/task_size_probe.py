"""Task-size probe: do smaller tasks for fields whose rows recur within a batch raise
L2 reuse?  With feature-major task order the features in flight at any moment are
~(#CTAs / tasks per feature); their distinct-row working sets compete for L2.
Shorter tasks for the recurring (small-table) fields put fewer of them in flight.

    python tools/task_size_probe.py sharded1000 [--factors 1,2,4,8] [--which reuse|all]
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
    ap.add_argument('--factors', default='1,2,4,8')
    ap.add_argument('--which', default='reuse')
    ap.add_argument('--reps', type=int, default=20)
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
    state = json.load(open(os.path.join(ROOT, 'configs', 'tuned', f'{a.config}_w1_r0.json')))
    reuse = [m.batch * f.mean_len() * f.coverage / f.rows for f in m.features]
    for which in a.which.split(','):
        for fac in [int(x) for x in a.factors.split(',')]:
            plan = Plan.from_model(m)
            plan.import_(state)
            n = 0
            for f in range(m.F):
                if which == 'reuse' and reuse[f] < 1.0:
                    continue
                s = plan.get_schedule(f)
                pb = max(1, s['per_block'] // fac) if s['part'] == 0 else max(64, s['per_block'] // fac)
                if pb != s['per_block']:
                    plan.set_schedule(f, s['sched_id'], s['part'], pb)
                    n += 1
            plan.task_order = plan.task_order_heuristic('lpt')
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
            print(json.dumps(dict(config=a.config, which=which, factor=fac, changed=n,
                                  ms=round(float(np.median(ts)), 4), min_ms=round(float(np.min(ts)), 4),
                                  variants=info['variants'])), flush=True)
            plan.close()


if __name__ == '__main__':
    main()
