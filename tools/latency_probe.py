"""Small-batch latency probe (medium / fig3): keep the one-hot features on the
tuned plan, put every multi-hot feature on one schedule shape (family, V, U, per
block) with the lane-group size matched to its dim, compile the plan-specialised
kernel and time map + fused (CUDA events, L2 flushed).  Development tool.

    python tools/latency_probe.py medium --ks 4,6,8
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
    ap.add_argument('--ks', default='4,6,8')
    ap.add_argument('--reps', type=int, default=20)
    ap.add_argument('--families', default='group,warp,flat')
    ap.add_argument('--vs', default='4,8')
    ap.add_argument('--us', default='2,4')
    ap.add_argument('--spbs', default='8,16,32,64')
    ap.add_argument('--no-tuned', action='store_true')
    ap.add_argument('--no-jit', action='store_true', help='time the catalog kernel instead')
    ap.add_argument('--onehot', action='store_true',
                    help='sweep the ONE-HOT features instead (multi-hot features keep the plan\'s schedules)')
    ap.add_argument('--base', default='tuned', choices=['tuned', 'default'])
    a = ap.parse_args()
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan, catalog, l2_flush
    dev = torch.device('cuda', 0)
    m = synth.make_model(a.config)
    phys = [synth.make_table(t, r, d, 'float', device=dev, seed=m.seed) for t, (r, d) in enumerate(m.tables)]
    tables = [phys[f.table] for f in m.features]
    bts = [synth.make_batch(m, 7 + i) for i in range(2)]
    dev_b = [(torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev)) for b in bts]
    plan = Plan.from_model(m)
    tuned = os.path.join(ROOT, 'configs', 'tuned', f'{a.config}_w1_r0.json')
    if a.base == 'tuned':
        plan.import_(json.load(open(tuned)))
    base = [plan.get_schedule(f) for f in range(m.F)]
    cat = catalog()
    out = torch.empty((m.batch, m.d_tot), device=dev)
    flush = torch.empty(64 << 20, device=dev)
    plan.set_profiling(True)

    def timeit():
        plan.kernel_times(reset=True)
        ts = []
        for r in range(a.reps + 2):
            l2_flush(flush)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            plan.forward(*dev_b[r % 2], m.batch, tables, out=out)
            e1.record()
            torch.cuda.synchronize()
            if r >= 2:
                ts.append(e0.elapsed_time(e1))
        kt = plan.kernel_times(reset=True)
        n = max(1, kt['forwards'])
        return float(np.median(ts)), kt['map_ms'] / n, kt['fused_ms'] / n

    def find(fam, G, V, U):
        for e in cat:
            if (e['family'], e['G'], e['VEC'], e['C'], e['U'], e['dtype']) == (fam, G, V, 1, U, 'f32'):
                return e['id']
        return None

    multi = [f for f, ft in enumerate(m.features) if (ft.max_len() > 1.5) != a.onehot]
    shapes = [] if a.no_tuned else [('tuned', None, None, None, None)]
    for fam in a.families.split(','):
        for V in [int(x) for x in a.vs.split(',')]:
            for U in [int(x) for x in a.us.split(',')]:
                for spb in [int(x) for x in a.spbs.split(',')]:
                    shapes.append((fam, V, U, spb, None))
    for k in [int(x) for x in a.ks.split(',')]:
        plan.occupancy = k
        for fam, V, U, spb, _ in shapes:
            ok = True
            for f in range(m.F):
                s = base[f]
                plan.set_schedule(f, s['sched_id'], s['part'], s['per_block'])
            if fam != 'tuned':
                for f in multi:
                    d = m.features[f].dim
                    G = max(1, min(32, d // V))
                    sid = find(fam, G, V, U)
                    if sid is None:
                        ok = False
                        break
                    per = spb * (8 if fam == 'flat' else 1)
                    try:
                        plan.set_schedule(f, sid, 0, per)
                    except Exception:
                        ok = False
                        break
            if not ok:
                continue
            if a.no_jit:
                plan.set_jit(False)
            else:
                plan.compile()
            ms, mp, fu = timeit()
            print(json.dumps(dict(config=a.config, k=k, family=fam, V=V, U=U, samples_per_task=spb,
                                  step_ms=round(ms, 4), map_ms=round(mp, 4), fused_ms=round(fu, 4))), flush=True)


if __name__ == '__main__':
    main()
