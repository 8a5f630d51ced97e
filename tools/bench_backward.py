"""Backward (training, NEXT #4) timing: recflex_backward on a BASELINE config.

    python tools/bench_backward.py sharded1000 [--steps 10] [--warmup 3]

One step = map kernel + fused scatter kernel over one batch (dense gradients
into fp32 targets; targets of features that share a physical table alias it,
as a shared table's gradient does).  Device-timed with CUDA events on the
launch stream; inputs (> L2) rotate over 2 batches.  Algorithmic bytes per
step: upstream gradient 4*B*D_tot + lookup IDs 4*nnz + every looked-up target
row read and written once 8*d per lookup (a row hit by several lookups is
counted each time, as the reductions are issued).  Prints one JSON line.
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
    ap.add_argument('--steps', type=int, default=10)
    ap.add_argument('--warmup', type=int, default=3)
    ap.add_argument('--occupancy', type=int, default=0)
    a = ap.parse_args()
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan

    dev = torch.device('cuda', 0)
    m = synth.make_model(a.config)
    B = m.batch
    plan = Plan.from_model(m)
    if a.occupancy:
        plan.occupancy = a.occupancy
    phys = [torch.zeros((r, d), device=dev) for r, d in m.tables]
    targets = [phys[f.table] for f in m.features]
    bts = [synth.make_batch(m, 7 + i) for i in range(2)]
    dev_b = [(torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev)) for b in bts]
    g = torch.empty((B, m.d_tot), device=dev).uniform_(-1, 1)
    dims = np.asarray(m.dims, np.int64)
    alg = []
    for b in bts:
        o = b.offsets.astype(np.int64)
        nnz_f = o[np.arange(1, m.F + 1) * B] - o[np.arange(0, m.F) * B]
        alg.append(4 * B * int(dims.sum()) + 4 * int(nnz_f.sum()) + 8 * int((dims * nnz_f).sum()))
    alg = float(np.mean(alg))
    for i in range(a.warmup):
        bi, bo = dev_b[i % 2]
        plan.backward(bi, bo, B, g, targets, scale=-1e-3)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for i in range(a.steps):
        bi, bo = dev_b[i % 2]
        plan.backward(bi, bo, B, g, targets, scale=-1e-3)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / a.steps
    peak = None
    try:
        with open(os.path.join(ROOT, 'MEASURED_PEAKS.json')) as fh:
            peak = float(json.load(fh)['hbm_gbs'])
    except Exception:
        pass
    gbs = alg / (ms / 1e3) / 1e9
    print(json.dumps({'what': 'recflex_backward (dense gradients, fused scatter)', 'config': a.config, 'B': B,
                      'occupancy': plan.occupancy, 'ms_per_step': ms, 'samples_per_s': B / (ms / 1e3),
                      'algorithmic_gb': alg / 1e9, 'effective_gbs': gbs,
                      'frac_of_hbm_peak': (gbs / peak) if peak else None}), flush=True)


if __name__ == '__main__':
    main()
