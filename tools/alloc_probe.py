"""Does the table allocation layout matter for heavy's gather rate?  16 separate
5 GB allocations (as bench.py) vs 16 views of one 82 GB allocation (values
uninitialised: timing only).  Development probe for DESIGN.md §6."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_panzzxwslr0d24_b200 import synth  # noqa: E402
from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan, l2_flush  # noqa: E402


def timeit(plan, m, tables, b, reps=6):
    dev = torch.device('cuda', 0)
    bi, bo = torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev)
    out = torch.empty((m.batch, m.d_tot), device=dev)
    flush = torch.empty(64 << 20, device=dev)
    ts = []
    for r in range(reps + 1):
        l2_flush(flush)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        plan.forward(bi, bo, m.batch, tables, out=out)
        e1.record()
        torch.cuda.synchronize()
        if r:
            ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))


def main():
    m = synth.make_model('heavy')
    b = synth.make_batch(m, 7)
    alg = synth.algorithmic_bytes(m, b)['total']
    plan = Plan.from_model(m)
    for f in range(m.F):
        plan.set_schedule(f, int(sys.argv[1]) if len(sys.argv) > 1 else 15, 0, 40)
    plan.occupancy = 4
    dev = torch.device('cuda', 0)
    rows, dim = m.tables[0]
    sep = [torch.empty((r, d), device=dev) for r, d in m.tables]
    t = timeit(plan, m, [sep[f.table] for f in m.features], b)
    print(f'16 separate allocations : {t:.3f} ms {alg / t / 1e6:.0f} GB/s', flush=True)
    del sep
    torch.cuda.empty_cache()
    big = torch.empty((len(m.tables) * rows, dim), device=dev)
    views = [big[i * rows:(i + 1) * rows] for i in range(len(m.tables))]
    t = timeit(plan, m, [views[f.table] for f in m.features], b)
    print(f'one allocation, 16 views: {t:.3f} ms {alg / t / 1e6:.0f} GB/s', flush=True)
    one = [views[0] for _ in m.features]
    t = timeit(plan, m, one, b)
    print(f'all features on table 0 : {t:.3f} ms {alg / t / 1e6:.0f} GB/s', flush=True)


if __name__ == '__main__':
    main()
