"""Small-batch makespan experiment (medium config): the tuned plan vs the same
plan with the multi-hot fields on BLOCK schedules (a CTA splits one bag across
8 warps, so a long bag no longer serialises on one lane group)."""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan, catalog, l2_flush
    cfg = sys.argv[1] if len(sys.argv) > 1 else 'medium'
    dev = torch.device('cuda', 0)
    m = synth.make_model(cfg)
    b = synth.make_batch(m, 7)
    phys = [synth.make_table(t, r, d, 'float', device=dev) for t, (r, d) in enumerate(m.tables)]
    tables = [phys[f.table] for f in m.features]
    bi, bo = torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev)
    out = torch.empty((m.batch, m.d_tot), device=dev)
    flush = torch.empty(64 << 20, device=dev)
    plan = Plan.from_model(m)
    path = os.path.join(ROOT, 'configs', 'tuned', f'{cfg}_w1_r0.json')
    if os.path.exists(path):
        plan.import_(json.load(open(path)))
    cat = catalog()

    def t():
        ts = []
        for r in range(12):
            l2_flush(flush)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            plan.forward(bi, bo, m.batch, tables, out=out)
            e1.record()
            torch.cuda.synchronize()
            if r >= 2:
                ts.append(e0.elapsed_time(e1))
        return float(np.median(ts))

    base = [plan.get_schedule(f) for f in range(m.F)]
    print('tuned', plan.occupancy, round(t() * 1e3, 1), 'us', flush=True)
    lens = b.lengths()
    multi = [f for f in range(m.F) if lens[f].max() > 1]
    for k in (plan.occupancy, 2, 4, 8):
        for U in (2, 4):
            for pb in (1, 2, 4):
                plan.occupancy = k
                for f in multi:
                    d = m.dims[f]
                    ids = [e['id'] for e in cat if e['family'] == 'block' and e['dtype'] == 'f32' and e['VEC'] == 4
                           and e['G'] == min(32, d // 4) and e['U'] == U]
                    if ids:
                        plan.set_schedule(f, ids[0], 0, pb)
                print(f'block for {len(multi)} multi-hot fields, k{k} U{U} samples/task {pb}: {t() * 1e3:.1f} us',
                      flush=True)
                for f, s in enumerate(base):
                    plan.set_schedule(f, s['sched_id'], s['part'], s['per_block'])


if __name__ == '__main__':
    main()
