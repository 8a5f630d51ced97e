"""Task-order probe: does running the longest tasks first shorten the fused kernel?

The fused kernel's persistent CTAs claim tasks from one counter in task-map order,
i.e. in feature order (block_start is an exclusive scan over the features).  A
feature whose tasks are long but which sits late in that order starts its tasks
when the GPU is already draining, and the kernel ends with a tail of few busy
CTAs.  This probe re-orders the features of a config (the output columns move
with them; the work is identical) and times the same per-feature schedules in
each order: model order, decreasing estimated task cost (LPT), increasing.

    python tools/order_probe.py industrial [configs/tuned/industrial_w1_r0.json]
"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def permute_batch(b, order, synth):
    B = b.B
    lens = b.lengths()[order]
    offs = np.zeros(len(order) * B + 1, np.int64)
    np.cumsum(lens.reshape(-1), out=offs[1:])
    parts = [b.indices[b.offsets[f * B]:b.offsets[(f + 1) * B]] for f in order]
    idx = np.concatenate(parts) if parts else np.zeros(0, np.int32)
    return synth.Batch(indices=idx.astype(np.int32), offsets=offs.astype(np.int32), B=B, F=len(order))


def task_cost(feat, sched, cat, B):
    """Estimated bytes one task of this feature moves (hotness stats only)."""
    sid, part, pb = sched[:3]
    rowb = 4 * feat.dim
    L = feat.mean_len() * feat.coverage
    if part == 0:
        return pb * max(L, 1e-3) * rowb
    return pb * rowb


def main():
    config = sys.argv[1]
    path = sys.argv[2] if len(sys.argv) > 2 else os.path.join(ROOT, 'configs/tuned', f'{config}_w1_r0.json')
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan, l2_flush, catalog
    dev = torch.device('cuda', 0)
    m = synth.make_model(config)
    state = json.load(open(path)) if path != 'default' else None
    cat = catalog()
    phys = [synth.make_table(t, r, d, 'float', device=dev, seed=m.seed) for t, (r, d) in enumerate(m.tables)]
    bts = [synth.make_batch(m, 7 + i) for i in range(3)]
    if state is None:
        p0 = Plan.from_model(m)
        state = p0.export()
        p0.close()
    scheds = state['schedules']
    cost = np.array([task_cost(f, scheds[i], cat, m.batch) for i, f in enumerate(m.features)])
    orders = {
        'model': list(range(m.F)),
        'lpt': list(np.argsort(-cost, kind='stable')),
        'spt': list(np.argsort(cost, kind='stable')),
    }
    # (layout, task order) grid: the model's features permuted (KJT layout and
    # output columns move) and/or the plan's task order (recflex_set_task_order)
    lpt = orders['lpt']
    inv = list(np.argsort(lpt))
    runs = {
        'model': (orders['model'], None),
        'layout_lpt+order_lpt': (lpt, None),
        'layout_model+order_lpt': (orders['model'], lpt),
        'layout_lpt+order_model': (lpt, inv),
        'spt': (orders['spt'], None),
        'layout_model+order_spt': (orders['model'], orders['spt']),
        'layout_model+order_lpt+cols': (orders['model'], lpt),
        'layout_model+order_spt+cols': (orders['model'], orders['spt']),
    }
    only = os.environ.get('ORDER_PROBE_ONLY')  # e.g. under ncu: one run, few launches
    if only:
        runs = {k: v for k, v in runs.items() if k in only.split(',')}
    nrep = int(os.environ.get('ORDER_PROBE_REPS', '40'))
    flush = torch.empty(64 << 20, device=dev)
    for name, (order, task_order) in runs.items():
        mm = synth.custom_model(m.name, [m.features[i] for i in order], m.batch)
        tables = [phys[f.table] for f in mm.features]
        st = dict(state)
        st['schedules'] = [scheds[i] for i in order]
        plan = Plan.from_model(mm)
        plan.import_(st)
        info = plan.compile()
        if name.endswith('+cols'):
            plan.set_column_order(True)   # outputs concatenated in task order
        if task_order is not None:
            plan.task_order = [int(x) for x in task_order]
        dev_b = []
        for b in bts:
            pb = permute_batch(b, order, synth)
            dev_b.append((torch.from_numpy(pb.indices).to(dev), torch.from_numpy(pb.offsets).to(dev)))
        out = torch.empty((m.batch, m.d_tot), device=dev)
        ts = []
        for r in range(nrep):
            l2_flush(flush)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            plan.forward(*dev_b[r % 3], m.batch, tables, out=out)
            e1.record()
            torch.cuda.synchronize()
            if r >= min(4, nrep - 1):
                ts.append(e0.elapsed_time(e1))
        print(json.dumps(dict(config=config, order=name, k=plan.occupancy, ms=round(float(np.median(ts)), 4),
                              min_ms=round(float(np.min(ts)), 4), regs=info['registers'],
                              variants=info['variants'])), flush=True)
        plan.close()


if __name__ == '__main__':
    main()
