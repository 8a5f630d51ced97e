"""Where does sharded1000's time go?  Times the fused forward of feature
subsets (one-hot / multi-hot, by dim) each with a default plan over the
global batch, and reports lookups/s against the ~40 G random accesses/s
ceiling (tools/gather_probe.cu)."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan, l2_flush
    from paper_conf_sc_panzzxwslr0d24_b200.shard import shard_batch
    dev = torch.device('cuda', 0)
    m = synth.make_model('sharded1000')
    b = synth.make_batch(m, 7)
    B = m.batch
    lens = b.lengths()
    phys = {}
    flush = torch.empty(64 << 20, device=dev)
    onehot = [f for f in range(m.F) if lens[f].max() <= 1]
    multi = [f for f in range(m.F) if lens[f].max() > 1]
    subsets = [('one-hot', onehot), ('multi-hot', multi)]
    for d in sorted(set(m.dims)):
        subsets.append((f'multi-hot d={d}', [f for f in multi if m.dims[f] == d]))
        subsets.append((f'one-hot d={d}', [f for f in onehot if m.dims[f] == d]))
    for name, feats in subsets:
        if not feats:
            continue
        for f in feats:
            t = m.features[f].table
            if t not in phys:
                rows, dim = m.tables[t]
                phys[t] = synth.make_table(t, rows, dim, 'float', device=dev, seed=m.seed)
        specs = [dict(rows=m.features[f].rows, dim=m.features[f].dim, pool=m.features[f].pool,
                      mean_len=m.features[f].mean_len(), max_len=m.features[f].max_len(),
                      coverage=m.features[f].coverage) for f in feats]
        plan = Plan(specs, B)
        plan.occupancy = 4
        idx, off = shard_batch(b, feats)
        bi, bo = torch.from_numpy(idx).to(dev), torch.from_numpy(off).to(dev)
        tables = [phys[m.features[f].table] for f in feats]
        out = torch.empty((B, sum(m.dims[f] for f in feats)), device=dev)
        ts = []
        for r in range(8):
            l2_flush(flush)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            plan.forward(bi, bo, B, tables, out=out)
            e1.record()
            torch.cuda.synchronize()
            if r >= 2:
                ts.append(e0.elapsed_time(e1))
        ms = float(np.median(ts))
        nnz = idx.size
        rowbytes = sum(4 * m.dims[f] * (int(off[(k + 1) * B]) - int(off[k * B])) for k, f in enumerate(feats))
        outb = 4 * B * sum(m.dims[f] for f in feats)
        print(f'{name:18s} F={len(feats):4d} {ms:7.3f} ms  lookups {nnz / 1e6:7.2f} M = {nnz / ms / 1e6:5.1f} G/s  '
              f'bags {len(feats) * B / ms / 1e6:6.1f} G/s  rows {rowbytes / 1e9:6.2f} GB out {outb / 1e9:5.2f} GB  '
              f'GB/s {(rowbytes + outb + 4 * nnz) / ms / 1e6:6.0f}', flush=True)
        del plan, bi, bo, out
        torch.cuda.empty_cache()


if __name__ == '__main__':
    main()
