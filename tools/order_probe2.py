"""More task orders for the shipped plan (columns follow the order, L2 policy as shipped):
LPT (shipped), table bytes ascending / descending, reuse (lookups per row) descending,
and LPT within table-size classes.

    python tools/order_probe2.py sharded1000
"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    config = sys.argv[1]
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan, l2_flush
    dev = torch.device('cuda', 0)
    m = synth.make_model(config)
    phys = [synth.make_table(t, r, d, 'float', device=dev, seed=m.seed) for t, (r, d) in enumerate(m.tables)]
    tables = [phys[f.table] for f in m.features]
    bts = [synth.make_batch(m, 7 + i) for i in range(3)]
    dev_b = [(torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev)) for b in bts]
    out = torch.empty((m.batch, m.d_tot), device=dev)
    flush = torch.empty(64 << 20, device=dev)
    plan = Plan.from_model(m)
    plan.import_(json.load(open(os.path.join(ROOT, 'configs', 'tuned', f'{config}_w1_r0.json'))))
    plan.set_column_order(True)
    plan.compile()
    tb = np.array([f.rows * f.dim * 4 for f in m.features], float)
    reuse = np.array([m.batch * f.mean_len() * f.coverage / f.rows for f in m.features])
    lpt = plan.task_order_heuristic('lpt')
    rank_lpt = np.argsort(lpt)  # position of each feature in LPT
    cls = np.digitize(tb, [8e6, 32e6, 128e6])
    orders = {
        'lpt': lpt,
        'table_asc': list(np.argsort(tb, kind='stable')),
        'table_desc': list(np.argsort(-tb, kind='stable')),
        'reuse_desc': list(np.argsort(-reuse, kind='stable')),
        'class_asc_lpt': list(np.lexsort((rank_lpt, cls))),
        'class_desc_lpt': list(np.lexsort((rank_lpt, -cls))),
    }
    rng = np.random.default_rng(11)
    for i in range(int(os.environ.get('ORDER_PROBE_RANDOM', '0'))):
        orders[f'random{i}'] = list(rng.permutation(m.F))
        # LPT with random swaps of neighbours (a local perturbation)
        o = list(lpt)
        for _ in range(m.F // 4):
            a_ = int(rng.integers(0, m.F - 1))
            o[a_], o[a_ + 1] = o[a_ + 1], o[a_]
        orders[f'lpt_jitter{i}'] = o
    for name, order in orders.items():
        plan.task_order = [int(x) for x in order]
        ts = []
        for r in range(22):
            l2_flush(flush)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            plan.forward(*dev_b[r % 3], m.batch, tables, out=out)
            e1.record()
            torch.cuda.synchronize()
            if r >= 2:
                ts.append(e0.elapsed_time(e1))
        print(json.dumps(dict(config=config, order=name, ms=round(float(np.median(ts)), 4))), flush=True)


if __name__ == '__main__':
    main()
