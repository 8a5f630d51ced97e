"""Tune a config's plan with the two-stage tuner and export it (tuned
schedules are reused for a long period, re-tuned periodically).

    python tools/tune_plan.py sharded1000 [--world W --rank R] [--ks 2,4,6,8] [--out DIR]

Writes DIR/<config>[_<dtype>]_w<W>_r<R>.json (default DIR = gpurun_out/tuned) plus a
.log with the tuner statistics.  bench.py loads configs/tuned/ automatically.
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument('config')
    ap.add_argument('--world', type=int, default=1)
    ap.add_argument('--rank', type=int, default=-1, help='-1: all ranks sequentially on this GPU')
    ap.add_argument('--ks', default='')
    ap.add_argument('--batches', type=int, default=2)
    ap.add_argument('--reps', type=int, default=5)
    ap.add_argument('--max-candidates', type=int, default=0)
    ap.add_argument('--dtype', default='f32', choices=['f32', 'f16', 'bf16', 'i8', 'fp8'])
    ap.add_argument('--out', default=os.path.join(ROOT, 'gpurun_out', 'tuned'))
    ap.add_argument('--refine', action='store_true', help='also run the (opt-in) cluster refinement')
    ap.add_argument('--no-guard', action='store_true')
    ap.add_argument('--stage2-catalog', action='store_true', help='stage 2 on the catalog kernel (no NVRTC)')
    ap.add_argument('--no-tail', action='store_true', help="stage 1 = the paper's plain block-time sum")
    ap.add_argument('--isolated', action='store_true', help='stage 1: one padded launch per candidate (C34)')
    ap.add_argument('--margin', type=float, default=0.0, help='stage-1 switch margin (reading C38)')
    ap.add_argument('--pad-waves', type=int, default=4, help='stage-1 padding in waves of tasks (P:148)')
    ap.add_argument('--no-post', action='store_true', help='skip the task-size / order / L2 selections')
    ap.add_argument('--balance', action='store_true', help='stage 1: position-balanced candidates (reading C39)')
    ap.add_argument('--from-tuned', action='store_true',
                    help='start from configs/tuned/<name>.json (its schedules, task order and column layout '
                         'are the incoming plan the guard compares against)')
    a = ap.parse_args()
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.shard import ShardedEmbedding, model_parts, shard_batch

    os.makedirs(a.out, exist_ok=True)
    dev = torch.device('cuda', 0)
    model = synth.make_model(a.config)
    parts = model_parts(model, a.world, a.dtype, a.config, os.path.join(ROOT, 'configs', 'tuned'))
    ranks = range(a.world) if a.rank < 0 else [a.rank]
    ks = [int(x) for x in a.ks.split(',')] if a.ks else None
    fulls = [synth.make_batch(model, 7 + i) for i in range(a.batches)]
    for r in ranks:
        sh = ShardedEmbedding(model, r, a.world, device=0, parts=parts, dtype=a.dtype)
        feats = sh.features
        phys = {}
        for f in feats:
            t = model.features[f].table
            if t not in phys:
                rows, dim = model.tables[t]
                phys[t] = synth.make_table_stored(t, rows, dim, a.dtype, 'float', device=dev, seed=model.seed)
        tables = [phys[model.features[f].table] for f in feats]
        name = f'{a.config}_w{a.world}_r{r}' if a.dtype == 'f32' else f'{a.config}_{a.dtype}_w{a.world}_r{r}'
        src = os.path.join(ROOT, 'configs', 'tuned', name + '.json')
        if a.from_tuned and os.path.exists(src):
            with open(src) as fh:
                sh.plan.import_(json.load(fh))
        hist = []
        for full in fulls:
            idx, off = shard_batch(full, feats)
            hist.append((torch.from_numpy(idx).to(dev), torch.from_numpy(off).to(dev), model.batch))
        t0 = time.time()
        st = sh.plan.tune(hist, tables, occupancies=ks, reps=a.reps, max_candidates=a.max_candidates, verbose=True,
                          refine=a.refine, guard=not a.no_guard, stage2_catalog=a.stage2_catalog,
                          tail=not a.no_tail, isolated=a.isolated, switch_margin=a.margin, position_balance=a.balance, pad_waves=a.pad_waves,
                          select_order=not a.no_post, select_l2=not a.no_post, select_task_size=not a.no_post)
        st['wall_s'] = time.time() - t0
        state = sh.plan.export()
        with open(os.path.join(a.out, name + '.json'), 'w') as fh:
            json.dump(state, fh)
        with open(os.path.join(a.out, name + '.log'), 'w') as fh:
            json.dump(st, fh, indent=1)
        print(name, json.dumps(st), flush=True)
        del sh, tables, phys, hist
        torch.cuda.empty_cache()


if __name__ == '__main__':
    main()
