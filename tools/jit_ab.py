"""A/B: the precompiled catalog kernel vs the plan-specialised (NVRTC) kernel
on a config's tuned plan, at several occupancies.  Prints fused-kernel device
time (CUDA events, L2 flushed before each forward), effective GB/s, the JIT
kernel's registers / local bytes, and checks both kernels produce identical
bits.  Development tool.

    python tools/jit_ab.py industrial --ks 4,5,6
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
    ap.add_argument('--ks', default='')
    ap.add_argument('--reps', type=int, default=10)
    ap.add_argument('--dtype', default='f32')
    ap.add_argument('--plan', default='auto')
    a = ap.parse_args()
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan, l2_flush
    dev = torch.device('cuda', 0)
    m = synth.make_model(a.config)
    phys = [synth.make_table_stored(t, r, d, a.dtype, 'float', device=dev, seed=m.seed)
            for t, (r, d) in enumerate(m.tables)]
    tables = [phys[f.table] for f in m.features]
    bts = [synth.make_batch(m, 7 + i) for i in range(2)]
    alg = np.mean([synth.algorithmic_bytes(m, b, a.dtype)['total'] for b in bts])
    dev_b = [(torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev)) for b in bts]
    plan = Plan.from_model(m, dtype=a.dtype)
    path = a.plan
    if path == 'auto':
        suffix = '' if a.dtype == 'f32' else f'_{a.dtype}'
        path = os.path.join(ROOT, 'configs', 'tuned', f'{a.config}{suffix}_w1_r0.json')
    if path != 'none' and os.path.exists(path):
        plan.import_(json.load(open(path)))
    k0 = plan.occupancy
    ks = [int(x) for x in a.ks.split(',')] if a.ks else [k0]
    out = torch.empty((m.batch, m.d_tot), device=dev)
    ref = torch.empty_like(out)
    flush = torch.empty(64 << 20, device=dev)

    def timeit():
        ts = []
        for r in range(a.reps + 2):
            bi, bo = dev_b[r % 2]
            l2_flush(flush)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            plan.forward(bi, bo, m.batch, tables, out=out)
            e1.record()
            torch.cuda.synchronize()
            if r >= 2:
                ts.append(e0.elapsed_time(e1))
        return float(np.median(ts))

    print(f'# {a.config} {a.dtype}: {alg / 1e9:.3f} GB algorithmic per batch; plan {os.path.relpath(path, ROOT)} '
          f'(tuned k={k0})', flush=True)
    info = plan.compile(ks)
    for k in ks:
        plan.occupancy = k
        plan.set_jit(False)
        tg = timeit()
        plan.forward(*dev_b[0], m.batch, tables, out=ref)
        plan.set_jit(True)
        tj = timeit()
        plan.forward(*dev_b[0], m.batch, tables, out=out)
        torch.cuda.synchronize()
        same = torch.equal(out, ref)
        ji = plan.jit_info(k)
        print(json.dumps(dict(config=a.config, k=k, generic_ms=round(tg, 4), jit_ms=round(tj, 4),
                              generic_gbs=round(alg / tg / 1e6), jit_gbs=round(alg / tj / 1e6),
                              speedup=round(tg / tj, 3), bitwise_equal=bool(same), jit=ji)), flush=True)
        assert same, 'JIT and catalog kernels differ'


if __name__ == '__main__':
    main()
