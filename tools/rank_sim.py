"""Per-rank device time of the table-wise sharded forward, measured on ONE GPU
(only one B200 is available to this run): for W = 2, 4, 8 every rank's plan
(its LPT feature subset, tuned plan from configs/tuned/ if present) runs the
global batch alone on cuda:0 and is timed with CUDA events (L2 flushed).
The max over ranks is the compute part of the §8e scaling roofline; the
pooled-output all-to-all is reported from its byte count at the measured
NVLink peer bandwidth (770 GB/s per direction, B200_PROFILING.md), since it
cannot be measured with one GPU.

    python tools/rank_sim.py sharded1000 [--worlds 2,4,8]
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

NVLINK_GBS = 770.0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument('config', nargs='?', default='sharded1000')
    ap.add_argument('--worlds', default='1,2,4,8')
    ap.add_argument('--reps', type=int, default=10)
    ap.add_argument('--no-jit', action='store_true')
    ap.add_argument('--tuned-dir', default=os.path.join(ROOT, 'configs', 'tuned'),
                    help='where the per-rank plans <config>_w<W>_r<R>.json are read from')
    a = ap.parse_args()
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import l2_flush
    from paper_conf_sc_panzzxwslr0d24_b200.shard import ShardedEmbedding, model_parts, shard_batch
    dev = torch.device('cuda', 0)
    model = synth.make_model(a.config)
    B = model.batch
    full = synth.make_batch(model, 7)
    phys = {}
    for t, (rows, dim) in enumerate(model.tables):
        phys[t] = synth.make_table_stored(t, rows, dim, 'f32', 'float', device=dev, seed=model.seed)
    flush = torch.empty(64 << 20, device=dev)
    for W in [int(x) for x in a.worlds.split(',')]:
        parts = model_parts(model, W, 'f32', a.config, a.tuned_dir)
        per_rank = []
        for r in range(W):
            sh = ShardedEmbedding(model, r, W, device=0, parts=parts)
            path = os.path.join(a.tuned_dir, f'{a.config}_w{W}_r{r}.json')
            tuned = os.path.exists(path)
            if tuned:
                sh.plan.import_(json.load(open(path)))
            tables = [phys[model.features[f].table] for f in sh.features]
            idx, off = shard_batch(full, sh.features)
            bi, bo = torch.from_numpy(idx).to(dev), torch.from_numpy(off).to(dev)
            if not a.no_jit:  # the kernel bench.py runs: plan-specialised or catalog, whichever is faster
                sh.plan.compile()
                sh.plan.select_kernel(bi, bo, B, tables, reps=5)
            out = torch.empty((B, sh.d_local), device=dev)
            ts = []
            for rep in range(a.reps + 2):
                l2_flush(flush)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                sh.plan.forward(bi, bo, B, tables, out=out)
                e1.record()
                torch.cuda.synchronize()
                if rep >= 2:
                    ts.append(e0.elapsed_time(e1))
            per_rank.append(dict(rank=r, features=len(sh.features), d_local=sh.d_local, ms=float(np.median(ts)),
                                 tuned=tuned, occupancy=sh.plan.occupancy,
                                 kernel='jit' if (not a.no_jit and sh.plan.jit_enabled) else 'catalog'))
            del sh, bi, bo, out
            torch.cuda.empty_cache()
        comp = max(p['ms'] for p in per_rank)
        dims = [p['d_local'] for p in per_rank]
        # per rank: send (W-1)/W of its [B][D_r] block, receive (W-1)/W*B/W... (max over ranks of max(send, recv))
        a2a = 0.0
        for r in range(W):
            send = 4.0 * B * dims[r] * (W - 1) / W
            recv = 4.0 * (B / W) * (sum(dims) - dims[r])
            a2a = max(a2a, max(send, recv))
        a2a_ms = a2a / (NVLINK_GBS * 1e9) * 1e3 if W > 1 else 0.0
        res = dict(config=a.config, world=W, compute_ms_max=comp, compute_ms_min=min(p['ms'] for p in per_rank),
                   a2a_bytes_max=a2a, a2a_ms_at_770=a2a_ms, serial_ms=comp + a2a_ms, overlapped_ms=max(comp, a2a_ms),
                   samples_per_s_serial=B / ((comp + a2a_ms) / 1e3),
                   samples_per_s_overlapped=B / (max(comp, a2a_ms) / 1e3), ranks=per_rank)
        print(json.dumps(res), flush=True)


if __name__ == '__main__':
    main()
