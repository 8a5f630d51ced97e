"""Time two tuned plans of a config in their plan-specialised kernels (map + fused,
CUDA events, L2 flushed, median over rotating batches) and print which is faster.

    python tools/plan_compare.py medium configs/tuned/medium_w1_r0.json gpurun_out/tuned_r02b/medium_w1_r0.json
"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    args = sys.argv[1:]
    catalog = '--catalog' in args      # time the precompiled catalog kernel instead
    args = [x for x in args if x != '--catalog']
    config, paths = args[0], args[1:]
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
    res = []
    for path in paths:
        plan = Plan.from_model(m)
        if path != 'default':
            plan.import_(json.load(open(path)))
        info = plan.compile()
        if catalog:
            plan.set_jit(False)
        ts = []
        for r in range(32):
            l2_flush(flush)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            plan.forward(*dev_b[r % 3], m.batch, tables, out=out)
            e1.record()
            torch.cuda.synchronize()
            if r >= 2:
                ts.append(e0.elapsed_time(e1))
        ms = float(np.median(ts))
        res.append((ms, path))
        print(json.dumps(dict(config=config, plan=path, kernel='catalog' if catalog else 'jit', k=plan.occupancy,
                              ms=round(ms, 4), regs=info['registers'],
                              local_bytes=info['local_bytes'], variants=info['variants'])), flush=True)
    best = min(res)
    print(json.dumps(dict(config=config, best=best[1], ms=round(best[0], 4))), flush=True)


if __name__ == '__main__':
    main()
