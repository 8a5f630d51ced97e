"""Per-dimension-class timing of a config: run the fused forward on the
sub-model made of the features with one embedding dim, default (or tuned)
schedules, and compare with the random-gather ceiling measured by
tools/gather_probe.cu.

    python tools/dimclass.py sharded1000 [--k 4]
"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

# rows/s measured by tools/gather_probe.cu on B200 (40 GB table, uniform rows)
PROBE_ROWS_PER_S = {16: 40e9, 32: 40.3e9, 64: 37.5e9, 128: 36.5e9, 256: 26.8e9, 512: 13.9e9}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument('config')
    ap.add_argument('--k', type=int, default=4)
    ap.add_argument('--reps', type=int, default=5)
    a = ap.parse_args()
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan, l2_flush
    from paper_conf_sc_panzzxwslr0d24_b200.shard import shard_batch
    dev = torch.device('cuda', 0)
    m = synth.make_model(a.config)
    full = synth.make_batch(m, 7)
    flush = torch.empty(64 << 20, device=dev)
    for d in sorted(set(m.dims)):
        feats = [f for f in range(m.F) if m.dims[f] == d]
        sub = synth.custom_model(f'{a.config}_d{d}', [m.features[f] for f in feats], m.batch)
        # keep the original table ids' contents: tables are generated per original table id
        phys = {}
        for f in feats:
            t = m.features[f].table
            if t not in phys:
                rows, dim = m.tables[t]
                phys[t] = synth.make_table(t, rows, dim, 'float', device=dev, seed=m.seed)
        tables = [phys[m.features[f].table] for f in feats]
        idx, off = shard_batch(full, feats)
        bi, bo = torch.from_numpy(idx).to(dev), torch.from_numpy(off).to(dev)
        plan = Plan.from_model(sub)
        plan.occupancy = a.k
        out = torch.empty((m.batch, sub.d_tot), device=dev)
        ts = []
        for r in range(a.reps + 1):
            l2_flush(flush)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            plan.forward(bi, bo, m.batch, tables, out=out)
            e1.record()
            torch.cuda.synchronize()
            if r:
                ts.append(e0.elapsed_time(e1))
        ms = float(np.median(ts))
        nnz = int(off[-1])
        alg = 4 * nnz + 4 * d * nnz + 4 * m.batch * sub.d_tot
        tb = sum(t.numel() * 4 for t in phys.values())
        floor_ms = nnz / PROBE_ROWS_PER_S[4 * d] * 1e3 + 4 * m.batch * sub.d_tot / 6.5e12 * 1e3
        print(f'dim {d:4d}: {len(feats):4d} fields, {nnz / 1e6:7.2f}M lookups, tables {tb / 1e9:6.2f} GB | '
              f'{ms:7.3f} ms  {alg / ms / 1e6:7.0f} GB/s  {nnz / ms / 1e6:6.1f} G rows/s | '
              f'gather floor {floor_ms:6.3f} ms ({floor_ms / ms:.2f})', flush=True)
        del phys, tables, plan, out
        torch.cuda.empty_cache()


if __name__ == '__main__':
    main()
