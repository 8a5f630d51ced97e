"""Measurement-driven refinement of the table-wise partition (open
item "W = 8 per-rank imbalance").  The LPT partition balances the *modelled*
per-rank device time (shard.feature_time); the tuned plans then land at
different occupancies and schedules, so the measured ranks differ (W = 8:
max/mean 1.12).  This closes the loop on measured times, on ONE GPU (each
rank's plan runs the global batch alone, L2 flushed, like tools/rank_sim.py):

  repeat: a = slowest rank, b = fastest rank; try moving one feature of a to b
  (candidates: modelled time, scaled by a's measured/modelled ratio, closest
  to half the gap first).  The moved feature keeps the schedule its tuned plan
  gave it (the plan's per-feature s_k); every other feature and both
  ranks' occupancies stay.  Accept the move if max(t_a', t_b') < t_a;
  stop after --moves accepted moves or when no candidate helps.

Writes DIR/<config>_w<W>_parts.json plus the per-rank plans of every rank it
changed (DIR/<config>_w<W>_r<R>.json); copied into configs/tuned/ they are
what bench.py, rank_sim.py and tune_plan.py load (shard.model_parts).

    python tools/rebalance.py sharded1000 --world 8 [--moves 8] [--out DIR]
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
    ap.add_argument('config', nargs='?', default='sharded1000')
    ap.add_argument('--world', type=int, default=8)
    ap.add_argument('--moves', type=int, default=8)
    ap.add_argument('--tries', type=int, default=6, help='candidates tried per move')
    ap.add_argument('--reps', type=int, default=10)
    ap.add_argument('--out', default=os.path.join(ROOT, 'gpurun_out', 'rebalance'))
    ap.add_argument('--catalog', action='store_true', help='measure the catalog kernel (round 1) instead of the '
                                                           'plan-specialised one')
    a = ap.parse_args()
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import l2_flush
    from paper_conf_sc_panzzxwslr0d24_b200.shard import (ShardedEmbedding, feature_time, model_parts,
                                                          refine_partition, shard_batch)
    os.makedirs(a.out, exist_ok=True)
    dev = torch.device('cuda', 0)
    model = synth.make_model(a.config)
    B, W, F = model.batch, a.world, len(model.features)
    tuned_dir = os.path.join(ROOT, 'configs', 'tuned')
    parts = model_parts(model, W, 'f32', a.config, tuned_dir)
    full = synth.make_batch(model, 7)
    phys = {t: synth.make_table_stored(t, rows, dim, 'f32', 'float', device=dev, seed=model.seed)
            for t, (rows, dim) in enumerate(model.tables)}
    flush = torch.empty(64 << 20, device=dev)

    # per-feature schedule and L2 policy, per-rank occupancy, task-order kind and
    # column layout from the tuned plans (a moved feature keeps its schedule and
    # policy; the receiving rank re-derives its order heuristic)
    sched, l2, occ, kinds, cols = {}, {}, [], [], []
    for r in range(W):
        st = json.load(open(os.path.join(tuned_dir, f'{a.config}_w{W}_r{r}.json')))
        pol = st.get('l2', [0] * len(parts[r]))
        for f, s, q in zip(parts[r], st['schedules'], pol):
            sched[f] = s
            l2[f] = q
        occ.append(st['occupancy'])
        cols.append(st.get('columns'))
        sh = ShardedEmbedding(model, r, W, device=0, parts=parts)
        sh.plan.import_(st)
        kinds.append(next((k for k in sh.plan.ORDER_KINDS if sh.plan.task_order == sh.plan.task_order_heuristic(k)),
                          'feature'))
        del sh
    catalog = st['catalog_size']
    fingerprint = st.get('catalog_fingerprint')

    def state(part, r):
        d = dict(abi=2, catalog_size=catalog, num_features=len(part), occupancy=occ[r],
                 schedules=[sched[f] for f in part], l2=[l2[f] for f in part])
        if fingerprint is not None:
            d['catalog_fingerprint'] = fingerprint
        if cols[r]:
            d['columns'] = cols[r]
        return d

    def rank_plan(parts_, r):
        sh = ShardedEmbedding(model, r, W, device=0, parts=parts_)
        sh.plan.import_(state(parts_[r], r))
        sh.plan.task_order = sh.plan.task_order_heuristic(kinds[r])
        if not a.catalog:
            sh.plan.compile()  # the plan-specialised kernel bench.py runs
        return sh

    def measure(parts_, r, k):
        sh = rank_plan(parts_, r)
        tables = [phys[model.features[f].table] for f in sh.features]
        idx, off = shard_batch(full, sh.features)
        bi, bo = torch.from_numpy(idx).to(dev), torch.from_numpy(off).to(dev)
        out = torch.empty((B, sh.d_local), device=dev)
        ts = []
        for rep in range(a.reps + 2):
            l2_flush(flush)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            sh.plan.forward(bi, bo, B, tables, out=out)
            e1.record()
            torch.cuda.synchronize()
            if rep >= 2:
                ts.append(e0.elapsed_time(e1))
        del sh, bi, bo, out
        return float(np.median(ts))

    est = [feature_time(model.features[f], B) for f in range(F)]
    parts0 = parts
    parts, t, log = refine_partition(parts, lambda p, r: measure(p, r, occ[r]), est, a.moves, a.tries)
    for entry in log:
        print(json.dumps(entry), flush=True)
    changed = {r for r in range(W) if parts[r] != parts0[r]}

    with open(os.path.join(a.out, f'{a.config}_w{W}_parts.json'), 'w') as fh:
        json.dump(dict(config=a.config, world=W, parts=parts, log=log,
                       note='tools/rebalance.py: measured refinement of the LPT partition'), fh)
    for r in range(W):  # every rank's plan follows the (possibly new) partition
        sh = rank_plan(parts, r)
        with open(os.path.join(a.out, f'{a.config}_w{W}_r{r}.json'), 'w') as fh:
            json.dump(sh.plan.export(), fh)
        del sh
    print(json.dumps(dict(done=True, changed=sorted(changed), max=max(t), max_over_mean=max(t) * W / sum(t))), flush=True)


if __name__ == '__main__':
    main()
