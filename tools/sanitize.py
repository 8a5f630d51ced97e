"""Small forwards for compute-sanitizer (memcheck / racecheck / synccheck / initcheck).

(compute-sanitizer is closed on the round-2 GPU pool; the families still run as plain
forwards, and the GPU tests compare the same paths with the oracle.)"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_sc_panzzxwslr0d24_b200 import synth  # noqa: E402
from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan, catalog  # noqa: E402

dev = torch.device('cuda', 0)
feats = []
dims = [4, 8, 12, 16, 32, 64, 128, 3]
for i, d in enumerate(dims):
    kind = 'onehot' if i % 3 == 0 else 'uniform'
    feats.append(synth.Feature(rows=500 + i, dim=d, pool=i % 2, kind=kind, coverage=0.7, lo=0, hi=40,
                               lmax=1 if kind == 'onehot' else 40, table=i))
m = synth.custom_model('san', feats, 96)
b = synth.make_batch(m, 3)
phys = [synth.make_table(t, r, d, 'int', device=dev) for t, (r, d) in enumerate(m.tables)]
tables = [phys[f.table] for f in m.features]
bi, bo = torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev)
cat = catalog()
fams = sys.argv[1:] or ['group', 'flat', 'block', 'warp', 'jit', 'static', 'order', 'exchange', 'bwd', 'kjt', 'host']
for fam in fams:
    if fam in ('jit', 'static'):
        # plan-specialised kernels: every family in one compiled kernel, runtime or static mapping
        plan = Plan.from_model(m)
        by_fam = {}
        for e in cat:
            if e['dtype'] == 'f32':
                by_fam.setdefault(e['family'], []).append(e['id'])
        n = 0
        for rnd in range(3):
            for f in range(m.F):
                fam_f = ('group', 'warp', 'flat', 'block')[(f + rnd) % 4]
                for sid in by_fam[fam_f][rnd::3]:
                    try:
                        plan.set_schedule(f, sid, f % 2, 16 if f % 2 == 0 else 128, 3 if fam == 'static' else 0)
                        break
                    except Exception:
                        pass
            plan.compile()
            plan.forward(bi, bo, b.B, tables)
            n += 1
        torch.cuda.synchronize()
        print(fam, 'forwards', n)
        continue
    if fam == 'order':
        # task order (C35) with task-order columns, every L2 policy (C36), halved task sizes
        # (C37) and lookup-partitioned features (the one-wave fill kernel), in both kernels
        import numpy as np
        plan = Plan.from_model(m)
        for f in range(m.F):
            s = plan.get_schedule(f)
            plan.set_schedule(f, s['sched_id'], f % 2, 8 if f % 2 == 0 else 24)
        rng = np.random.default_rng(1)
        n = 0
        for rnd, cols in enumerate((False, True)):
            try:
                plan.set_column_order(cols)
            except Exception:
                pass
            for jit in (False, True):
                plan.task_order = rng.permutation(m.F).tolist()
                plan.l2_policy = [(f + rnd) % 4 for f in range(m.F)]
                if jit:
                    plan.compile()
                plan.set_jit(jit)
                plan.forward(bi, bo, b.B, tables)
                n += 1
        torch.cuda.synchronize()
        print('order forwards', n)
        continue
    if fam == 'exchange':
        # recflex_forward_exchange with one rank (its own buffers and flags): kernel epilogue
        # flag publication + the wait kernel, several steps
        from paper_conf_sc_panzzxwslr0d24_b200.plan import DeviceBuffer
        plan = Plan.from_model(m)
        bufs = [DeviceBuffer(b.B, m.d_tot) for _ in range(2)]
        flags = DeviceBuffer(1, 1)
        flags.tensor.zero_()
        for i in range(4):
            plan.forward_exchange(bi, bo, b.B, tables, 1, 0, b.B, m.d_tot, 0, [bufs[0].ptr.value],
                                  [bufs[1].ptr.value], [flags.ptr.value], flags.ptr.value)
        torch.cuda.synchronize()
        print('exchange ok')
        continue
    if fam == 'bwd':
        plan = Plan.from_model(m)
        grad = torch.randn((b.B, m.d_tot), device=dev)
        tg = [torch.zeros((f.rows, f.dim), device=dev) for f in m.features]
        plan.backward(bi, bo, b.B, grad, tg)
        torch.cuda.synchronize()
        print('bwd ok')
        continue
    if fam == 'kjt':
        from paper_conf_sc_panzzxwslr0d24_b200.plan import KJTDist
        W, Bl = 3, 32
        owner = [f % W for f in range(m.F)]
        locs = [synth.make_batch(m, 50 + j, B=Bl) for j in range(W)]
        kds = [KJTDist(owner, W, j, Bl) for j in range(W)]
        sends = []
        for j, lb in enumerate(locs):
            i_d, o_d = torch.from_numpy(lb.indices).to(dev), torch.from_numpy(lb.offsets).to(dev)
            sl = torch.empty(m.F * Bl, dtype=torch.int32, device=dev)
            si = torch.empty(max(1, lb.indices.size), dtype=torch.int32, device=dev)
            dc = torch.empty(W, dtype=torch.int32, device=dev)
            kds[j].pack(i_d, o_d, sl, si, dc)
            sends.append((sl, si, dc.cpu().tolist(), kds[j].send_length_counts))
        for r in range(W):
            rl = torch.cat([sl[sum(lc[:r]):sum(lc[:r]) + lc[r]] for sl, _, _, lc in sends])
            ri = torch.cat([si[sum(dc[:r]):sum(dc[:r]) + dc[r]] for _, si, dc, _ in sends])
            io = torch.empty(max(1, ri.numel()), dtype=torch.int32, device=dev)
            oo = torch.empty(kds[r].num_owned * W * Bl + 1, dtype=torch.int32, device=dev)
            kds[r].unpack(rl, ri, io, oo)
        torch.cuda.synchronize()
        print('kjt ok')
        continue
    if fam == 'lowp':
        lfeats = [synth.Feature(rows=300 + i, dim=d, pool=i % 2, kind='uniform', coverage=1.0, lo=0, hi=30, lmax=30,
                                table=i) for i, d in enumerate([8, 16, 32, 64, 128, 24])]
        lm = synth.custom_model('san_lowp', lfeats, 64)
        lb = synth.make_batch(lm, 3)
        li, lo = torch.from_numpy(lb.indices).to(dev), torch.from_numpy(lb.offsets).to(dev)
        n = 0
        for dt in ('f16', 'bf16', 'i8', 'fp8'):
            tabs = [synth.make_table_stored(f.table, f.rows, f.dim, dt, 'int', device=dev) for f in lm.features]
            specs = [dict(rows=f.rows, dim=f.dim, pool=f.pool, mean_len=15, max_len=30, coverage=1.0, dtype=dt)
                     for f in lm.features]
            plan = Plan(specs, lb.B)
            for e in [e for e in cat if e['dtype'] == dt][::2]:
                for f in range(lm.F):
                    try:
                        plan.set_schedule(f, e['id'], 0, 8)
                    except Exception:
                        pass
                plan.forward(li, lo, lb.B, tabs)
                n += 1
        torch.cuda.synchronize()
        print('lowp forwards', n)
        continue
    if fam == 'host':
        plan = Plan.from_model(m)
        hb = [(torch.from_numpy(b.indices).pin_memory(), torch.from_numpy(b.offsets).pin_memory(), b.B)] * 3
        outs = [torch.empty((b.B, m.d_tot)).pin_memory() for _ in range(3)]
        plan.forward_host_batches(hb, tables, outs)
        print('host ok')
        continue
    ids = [e['id'] for e in cat if e['family'] == fam]
    plan = Plan.from_model(m)
    plan.occupancy = 8 if fam != 'block' else 4
    n = 0
    for sid in ids[::3]:
        for part in (0, 1):
            for f in range(m.F):
                try:
                    plan.set_schedule(f, sid, part, 16 if part == 0 else 128)
                except Exception:
                    pass
            plan.forward(bi, bo, b.B, tables)
            n += 1
    torch.cuda.synchronize()
    print(fam, 'forwards', n)
