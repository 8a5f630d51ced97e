"""Task-order (reading C35) and L2-policy (C36) selection for the tuned plans bench.py loads: load
configs/tuned/<config>[_<dtype>]_w<W>_r<R>.json, compile, keep the faster kernel
(recflex_select_kernel), then recflex_select_task_order and recflex_select_l2_policy
on a tuning batch (seed 8, as tools/tune_plan.py's second historical batch) and export
the plan, its order and L2 policy included, to DIR (default gpurun_out/tuned).

    python tools/select_order.py sharded1000 [--world W] [--dtype bf16] [--out DIR]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument('config')
    ap.add_argument('--world', type=int, default=1)
    ap.add_argument('--dtype', default='f32', choices=['f32', 'f16', 'bf16', 'i8', 'fp8'])
    ap.add_argument('--reps', type=int, default=9)
    ap.add_argument('--task-size', action='store_true', help='also recflex_select_task_size (C37) first')
    ap.add_argument('--columns', default='plan', choices=['plan', 'feature', 'task-order'],
                    help="output layout to select under: the plan file's, or set it")
    ap.add_argument('--out', default=os.path.join(ROOT, 'gpurun_out', 'tuned'))
    a = ap.parse_args()
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.shard import ShardedEmbedding, model_parts, shard_batch

    os.makedirs(a.out, exist_ok=True)
    dev = torch.device('cuda', 0)
    model = synth.make_model(a.config)
    parts = model_parts(model, a.world, a.dtype, a.config, os.path.join(ROOT, 'configs', 'tuned'))
    full = synth.make_batch(model, 8)
    for r in range(a.world):
        name = f'{a.config}_w{a.world}_r{r}' if a.dtype == 'f32' else f'{a.config}_{a.dtype}_w{a.world}_r{r}'
        path = os.path.join(ROOT, 'configs', 'tuned', name + '.json')
        sh = ShardedEmbedding(model, r, a.world, device=0, parts=parts, dtype=a.dtype)
        feats = sh.features
        phys = {}
        for f in feats:
            t = model.features[f].table
            if t not in phys:
                rows, dim = model.tables[t]
                phys[t] = synth.make_table_stored(t, rows, dim, a.dtype, 'float', device=dev, seed=model.seed)
        tables = [phys[model.features[f].table] for f in feats]
        if os.path.exists(path):
            with open(path) as fh:
                sh.plan.import_(json.load(fh))
        idx, off = shard_batch(full, feats)
        bi, bo = torch.from_numpy(idx).to(dev), torch.from_numpy(off).to(dev)
        if a.columns != 'plan':
            sh.plan.set_column_order(a.columns == 'task-order')
        sh.plan.compile()
        ksel = sh.plan.select_kernel(bi, bo, model.batch, tables, reps=5)
        size = sh.plan.select_task_size(bi, bo, model.batch, tables, reps=a.reps) if a.task_size else None
        res = sh.plan.select_task_order(bi, bo, model.batch, tables, reps=a.reps)
        l2 = sh.plan.select_l2_policy(bi, bo, model.batch, tables, reps=a.reps) if sh.plan.jit_enabled else None
        state = sh.plan.export()
        with open(os.path.join(a.out, name + '.json'), 'w') as fh:
            json.dump(state, fh)
        print(json.dumps(dict(plan=name, kernel=ksel['kernel'], order=res['order'],
                              columns=state.get('columns', 'feature'),
                              task_size=(size['task_size'] if size else None),
                              size_ms=({k: round(v, 4) for k, v in size['ms'].items()} if size else None),
                              l2=(l2['l2'] if l2 else 'n/a (catalog kernel)'),
                              l2_ms=({k: round(v, 4) for k, v in l2['ms'].items()} if l2 else None),
                              ms={k: round(v, 4) for k, v in res['ms'].items()})), flush=True)
        del sh, tables, phys
        torch.cuda.empty_cache()


if __name__ == '__main__':
    main()
