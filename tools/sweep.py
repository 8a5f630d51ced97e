"""Uniform-schedule sweep: every feature of a config on the same catalog entry,
for each occupancy k -> fused-kernel time and effective GB/s.  A development
tool for understanding the catalog on B200 (not the tuner).

    python tools/sweep.py heavy --ks 4,6,8 [--ids 15,16,17] [--part 0] [--spb-scale 1]
"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument('config')
    ap.add_argument('--ks', default='4,6,8')
    ap.add_argument('--ids', default='')
    ap.add_argument('--parts', default='0')
    ap.add_argument('--per-block', default='', help='override per_block values (comma list)')
    ap.add_argument('--reps', type=int, default=6)
    ap.add_argument('--dtype', default='f32', choices=['f32', 'f16', 'bf16', 'i8', 'fp8'])
    a = ap.parse_args()
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan, catalog, l2_flush
    dev = torch.device('cuda', 0)
    m = synth.make_model(a.config)
    phys = [synth.make_table_stored(t, r, d, a.dtype, 'float', device=dev) for t, (r, d) in enumerate(m.tables)]
    tables = [phys[f.table] for f in m.features]
    bts = [synth.make_batch(m, 7 + i) for i in range(2)]
    alg = np.mean([synth.algorithmic_bytes(m, b, a.dtype)['total'] for b in bts])
    dev_b = [(torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev)) for b in bts]
    plan = Plan.from_model(m, dtype=a.dtype)
    out = torch.empty((m.batch, m.d_tot), device=dev)
    flush = torch.empty(64 << 20, device=dev)
    cat = catalog()
    ids = [int(x) for x in a.ids.split(',')] if a.ids else [e['id'] for e in cat if e['dtype'] == a.dtype]
    dims = sorted(set(m.dims))
    default = [plan.get_schedule(f) for f in range(m.F)]
    print(f'# {a.config}: {alg / 1e9:.2f} GB algorithmic per batch')
    for sid in ids:
        e = cat[sid]
        for part in [int(p) for p in a.parts.split(',')]:
            pbs = [int(x) for x in a.per_block.split(',')] if a.per_block else [None]
            for pb in pbs:
                ok = True
                for f in range(m.F):
                    d = default[f]
                    per = pb if pb is not None else (d['per_block'] if part == 0 else 4096)
                    if part == 0 and pb is None:
                        # keep ~ the default lookups per task for this group size
                        g_def = cat[d['sched_id']]
                        slots_def = 256 // g_def['G'] if g_def['family'] == 'group' else 1
                        slots = 256 // e['G'] if e['family'] == 'group' else 1
                        per = max(1, d['per_block'] * slots // slots_def) if e['family'] == 'group' else max(
                            1, d['per_block'] // slots_def)
                    try:
                        plan.set_schedule(f, sid, part, per)
                    except Exception:
                        ok = False
                        break
                if not ok:
                    continue
                span = e['G'] * e['VEC'] * e['C']
                if any(-(-d // span) > 1 for d in dims):
                    continue
                res = []
                for k in [int(x) for x in a.ks.split(',')]:
                    plan.occupancy = k
                    ts = []
                    for r in range(a.reps + 1):
                        bi, bo = dev_b[r % 2]
                        l2_flush(flush)
                        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                        e0.record()
                        plan.forward(bi, bo, m.batch, tables, out=out)
                        e1.record()
                        torch.cuda.synchronize()
                        if r:
                            ts.append(e0.elapsed_time(e1))
                    ms = float(np.median(ts))
                    res.append(f'k{k}: {ms:7.3f} ms {alg / ms / 1e6:6.0f} GB/s')
                print(f"{sid:3d} {e['family']:5s} G{e['G']:<2d} V{e['VEC']} C{e['C']} U{e['U']} part{part} "
                      f"pb={pb} | " + ' | '.join(res), flush=True)
    for f in range(m.F):
        plan.set_schedule(f, default[f]['sched_id'], default[f]['part'], default[f]['per_block'])


if __name__ == '__main__':
    main()
