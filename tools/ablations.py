"""The paper's ablations re-run on B200 with this framework.

  mapping : Fig. 13 / P:328-340 -- runtime thread mapping vs static mapping
            from historical average / maximum block counts, on historical-size
            batches and on a long-tail request 5x larger (2,560 samples).
  swap    : Fig. 12 / P:326 -- in a tuned plan, replace one feature's schedule by
            every other candidate and time the fused kernel; the tuned choice
            should be optimal or near-optimal.

    python tools/ablations.py mapping|swap [--config industrial] [--out gpurun_out/ablations_<x>.md]
"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def timer(plan, batch_dev, B, tables, out, flush, reps=7):
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200.plan import l2_flush
    ts = []
    for r in range(reps + 1):
        l2_flush(flush)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        plan.forward(batch_dev[0], batch_dev[1], B, tables, out=out[:B])
        e1.record()
        torch.cuda.synchronize()
        if r:
            ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))


def setup(config, Bmax):
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    dev = torch.device('cuda', 0)
    m = synth.make_model(config)
    phys = [synth.make_table(t, r, d, 'float', device=dev) for t, (r, d) in enumerate(m.tables)]
    tables = [phys[f.table] for f in m.features]
    out = torch.empty((Bmax, m.d_tot), device=dev)
    flush = torch.empty(64 << 20, device=dev)
    return m, tables, out, flush


def dev_batch(b):
    import torch
    return torch.from_numpy(b.indices).cuda(), torch.from_numpy(b.offsets).cuda()


def ablation_mapping(config, lines):
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan
    import oracle  # noqa: F401  (task map formula is the plan's; we read it back from the library)
    hist_B, tail_B = 512, 2560
    m, tables, out, flush = setup(config, tail_B)
    plan = Plan.from_model(m, max_batch=tail_B)
    runtime = [plan.get_schedule(f) for f in range(m.F)]
    hist = [synth.make_batch(m, 100 + i, B=hist_B) for i in range(4)]
    # tasks each feature needs under the runtime mapping on the historical batches
    # ("we first run the runtime thread mapping kernels to collect the thread block
    # usages")
    per_batch = []
    for hb in hist:
        plan.debug_task_map(dev_batch(hb)[1], hist_B)
        per_batch.append(np.asarray(plan.debug_task_need()))
    per_batch = np.asarray(per_batch)
    static_avg = np.maximum(1, np.rint(per_batch.mean(axis=0))).astype(int)
    static_max = per_batch.max(axis=0).astype(int)
    tests = [('historical-size batch (B=512)', synth.make_batch(m, 7, B=hist_B), hist_B),
             (f'long-tail request (B={tail_B}, P:340)', synth.make_batch(m, 8, B=tail_B), tail_B)]
    lines += [f'## Runtime vs static thread mapping ({config}, Fig. 13 / P:328-340)', '',
              'Static block counts per feature are the runtime mapping\'s counts averaged / maxed over 4 '
              'historical batches of 512 samples; the schedules are identical, only the mapping differs. '
              'Under the static mapping allocated block a performs the needed blocks a, a + n, a + 2n, ... '
              'one after another (P:338, reading C31); every mode runs its plan-specialised kernel.', '',
              '| batch | runtime mapping (ms) | static avg (ms) | static max (ms) | slowdown avg | slowdown max |',
              '|---|---|---|---|---|---|']
    for label, b, B in tests:
        bd = dev_batch(b)
        res = {}
        for mode, counts in (('runtime', None), ('avg', static_avg), ('max', static_max)):
            for f in range(m.F):
                s = runtime[f]
                plan.set_schedule(f, s['sched_id'], s['part'], s['per_block'], 0 if counts is None else int(counts[f]))
            plan.compile()
            res[mode] = timer(plan, bd, B, tables, out, flush)
        lines.append(f"| {label} | {res['runtime']:.3f} | {res['avg']:.3f} | {res['max']:.3f} | "
                     f"{res['avg'] / res['runtime']:.2f}x | {res['max'] / res['runtime']:.2f}x |")
        print(lines[-1], flush=True)
    lines.append('')


def ablation_swap(config, lines, nfeat=3, seed=0):
    import json
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan, catalog
    m, tables, out, flush = setup(config, None or synth.make_model(config).batch)
    plan = Plan.from_model(m)
    tuned = os.path.join(ROOT, 'configs', 'tuned', f'{config}_w1_r0.json')
    src = 'default schedules'
    if os.path.exists(tuned):
        plan.import_(json.load(open(tuned)))
        src = os.path.relpath(tuned, ROOT)
    b = synth.make_batch(m, 7)
    bd = dev_batch(b)
    base = timer(plan, bd, m.batch, tables, out, flush)
    rng = np.random.default_rng(seed)
    multi = [f for f, ft in enumerate(m.features) if ft.kind != 'onehot']
    picks = rng.choice(multi if len(multi) >= nfeat else range(m.F), size=nfeat, replace=False)
    cat = catalog()
    lines += [f'## Schedule swap around the tuned plan ({config}, Fig. 12 / P:326)', '',
              f'Plan: {src}, k={plan.occupancy}; baseline {base:.3f} ms.  For each picked feature, every '
              'single-pass catalog entry is substituted (same partition) and the whole fused kernel timed.', '',
              '| feature (dim, mean L) | tuned schedule | candidates | best (ms) | tuned (ms) | tuned rank | worst (ms) |',
              '|---|---|---|---|---|---|---|']
    for f in picks:
        f = int(f)
        s0 = plan.get_schedule(f)
        times = []
        for e in cat:
            span = e['G'] * e['VEC'] * e['C']
            if m.dims[f] % e['VEC'] or -(-m.dims[f] // span) > 1 or 4 * m.dims[f] < span:
                continue
            try:
                plan.set_schedule(f, e['id'], s0['part'], s0['per_block'] if e['family'] == cat[s0['sched_id']][
                    'family'] else max(1, s0['per_block']))
            except Exception:
                continue
            times.append((timer(plan, bd, m.batch, tables, out, flush, reps=5), e['id']))
        plan.set_schedule(f, s0['sched_id'], s0['part'], s0['per_block'])
        tuned_t = timer(plan, bd, m.batch, tables, out, flush, reps=5)
        times.sort()
        rank = 1 + sum(1 for t, _ in times if t < tuned_t * 0.999)
        e0 = cat[s0['sched_id']]
        lines.append(f"| {f} ({m.dims[f]}, {m.features[f].mean_len():.1f}) | {e0['family']} G{e0['G']} V{e0['VEC']} "
                     f"U{e0['U']} part{s0['part']} | {len(times)} | {times[0][0]:.3f} | {tuned_t:.3f} | {rank} | "
                     f"{times[-1][0]:.3f} |")
        print(lines[-1], flush=True)
    lines.append('')


def ablation_tuning(config, lines, ks=(3, 4, 5, 6)):
    """Fig. 11 / P:324: two-stage interference-simulated tuning vs the
    separate-combine straw man (each candidate timed alone, non-padded)."""
    import time
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan
    m, tables, out, flush = setup(config, synth.make_model(config).batch)
    hist = [synth.make_batch(m, 7 + i) for i in range(2)]
    hist_dev = [(*dev_batch(b), m.batch) for b in hist]
    test = dev_batch(synth.make_batch(m, 50))
    rows = []
    for label, kw in (('default heuristic (untuned)', None),
                      ('separate-combine (straw man 1, P:73)', dict(separate=True, guard=False, refine=False)),
                      ("two-stage co-execution, the paper's Eq. 3 cost", dict(tail=False, guard=False, refine=False)),
                      ('two-stage, tail-aware stage 1 (C33)', dict(tail=True, guard=False, refine=False)),
                      ('two-stage, tail-aware + guard (default)', dict(tail=True, guard=True, refine=False)),
                      ('... + cluster refinement (opt-in, outside O(F*K+K))', dict(tail=True, guard=True,
                                                                                     refine=True))):
        plan = Plan.from_model(m)
        plan.occupancy = 4
        t0 = time.time()
        st = plan.tune(hist_dev, tables, occupancies=list(ks), reps=5, **kw) if kw is not None else {}
        tt = time.time() - t0
        plan.compile()  # every plan timed in its plan-specialised kernel
        ms = timer(plan, test, m.batch, tables, out, flush)
        rows.append((label, ms, tt, st.get('local_launches', 0), st.get('global_launches', 0),
                     st.get('compile_seconds', 0.0), st.get('refine_evals', 0), plan.occupancy))
        print(label, ms, tt, flush=True)
    base = rows[0][1]
    lines += [f'## Tuning strategies ({config}, k in {list(ks)}; Fig. 11 / P:324)', '',
              'Each plan is tuned on 2 historical batches and timed on a held-out batch (median of 7, L2 flushed) in '
              'its plan-specialised kernel.', '',
              '| tuner | k | fused forward (ms) | vs untuned | tuning time (s) | of which NVRTC (s) | local launches | '
              'global launches | refinement forwards |', '|---|---|---|---|---|---|---|---|---|']
    for label, ms, tt, ll, gl, cs, re, k in rows:
        lines.append(f'| {label} | {k} | {ms:.3f} | {base / ms:.2f}x | {tt:.0f} | {cs:.0f} | {ll} | {gl} | {re} |')
    lines.append('')


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument('which', choices=['mapping', 'swap', 'tuning'])
    ap.add_argument('--config', default='industrial')
    ap.add_argument('--out', default='')
    a = ap.parse_args()
    lines = []
    if a.which == 'mapping':
        ablation_mapping(a.config, lines)
    elif a.which == 'tuning':
        ablation_tuning(a.config, lines)
    else:
        ablation_swap(a.config, lines)
    out = a.out or os.path.join(ROOT, 'gpurun_out', f'ablation_{a.which}_{a.config}.md')
    os.makedirs(os.path.dirname(out), exist_ok=True)
    with open(out, 'w') as fh:
        fh.write('\n'.join(lines) + '\n')


if __name__ == '__main__':
    main()
