#!/usr/bin/env python
"""bench.py -- RecFlex hot path on B200: fused heterogeneous-schedule
embedding-bag forward (map + fused kernels), table-wise sharded with a pooled-
output NCCL all-to-all at N > 1.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config sharded1000]
    torchrun --nproc-per-node N bench.py --gpus N ...       (N > 1)
    python bench.py --impl reference ...                      (CPU oracle arm)

One step = one pass of the whole hot path over one synthetic batch already
resident in HBM: device-side workload map -> fused kernel (-> alltoallv ->
relayout at N > 1).  Batches rotate over --batches distinct seeded batches
whose index arrays alone exceed L2 (sharded1000: 0.55 GB per batch, tables
28.5 GB), so no L2 flush is needed between steps (configs whose working set
fits in L2 are flushed between steps by a kernel outside the timed events).
Rank 0 prints ONE JSON line.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import tempfile
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

FALLBACK_HBM_GBS = 6650.0   # B200_PROFILING.md fallback, used only if MEASURED_PEAKS.json is absent
L2_BYTES = 126 * 2 ** 20


def _baseline_metric():
    try:
        with open(os.path.join(ROOT, 'BASELINE.json')) as fh:
            return json.load(fh)['metric']
    except Exception:
        return 'pooled samples/s and effective HBM GB/s (% of 8 TB/s) at 1/2/4/8 B200'


def _peaks():
    p = os.path.join(ROOT, 'MEASURED_PEAKS.json')
    if os.path.exists(p):
        with open(p) as fh:
            d = json.load(fh)
        return float(d['hbm_gbs']), 'measured (MEASURED_PEAKS.json hbm_gbs, copy read+write)'
    return FALLBACK_HBM_GBS, 'fallback (B200_PROFILING.md)'


# ------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks/throttle sampling DURING the timed region."""
    Q = ('index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,'
         'clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,'
         'clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap')

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.proc = None
        self.path = None

    def start(self):
        try:
            fd, self.path = tempfile.mkstemp(suffix='.csv')
            os.close(fd)
            self.proc = subprocess.Popen(['nvidia-smi', f'--id={self.gpu}', f'--query-gpu={self.Q}',
                                          '--format=csv,noheader,nounits', '-lms', '100'],
                                         stdout=open(self.path, 'w'), stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return None
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        rows = []
        for line in open(self.path):
            parts = [x.strip() for x in line.split(',')]
            if len(parts) < 9:
                continue
            try:
                rows.append(dict(sm=float(parts[1]), smmax=float(parts[2]), reasons=parts[5:9]))
            except ValueError:
                continue
        os.unlink(self.path)
        if not rows:
            return None
        names = ['hw_slowdown', 'hw_thermal_slowdown', 'sw_thermal_slowdown', 'sw_power_cap']
        seen = set()
        for r in rows:
            for n, v in zip(names, r['reasons']):
                if v.lower().startswith('active'):
                    seen.add(n)
        return {'sm_mhz': float(np.median([r['sm'] for r in rows])), 'sm_max_mhz': rows[0]['smmax'],
                'reasons': sorted(seen), 'samples': len(rows)}


def _cpu_model():
    try:
        with open('/proc/cpuinfo') as fh:
            for line in fh:
                if line.startswith('model name'):
                    return line.split(':', 1)[1].strip()
    except Exception:
        pass
    import platform
    return platform.processor() or 'unknown'


def l2_policy_summary(plan):
    """How many features' row loads carry each L2 eviction priority (reading C36)."""
    pol = plan.l2_policy
    return {name: pol.count(i) for i, name in enumerate(plan.L2_POLICIES) if pol.count(i)}


def task_order_name(plan):
    """Which order the plan's tasks are claimed in (reading C35): a heuristic's name or 'custom'."""
    order = plan.task_order
    for kind in plan.ORDER_KINDS:
        if order == plan.task_order_heuristic(kind):
            return kind
    return 'custom'


def _workload_config(args, model, world):
    """The `config` dict both arms print (identical keys and values for the same run):
    the workload only -- implementation details go to `impl_config`."""
    return {'workload': args.config, 'global_batch': model.batch, 'fields': model.F, 'table_dtype': args.dtype,
            'parallelism': f'tablewise{world}',
            'l2': f'inputs > L2 ({args.batches} rotating batches, each larger than L2) or flushed between steps'}


# ------------------------------------------------------------------------- CPU oracle arm
def oracle_sample_rate(model, batch, n_samples: int, seed: int = 0, nthreads: int = 0, min_seconds: float = 0.0,
                       max_reps: int = 1000, dtype: str = 'f32'):
    """Time the oracle (as it stands) on a bounded sample of the workload.

    Input preparation (regenerating the referenced table rows from the seeded
    generator) is outside the timed region; the timed region is the oracle's
    embedding-bag over the sampled bags of every feature, repeated until
    `min_seconds` of CPU work (at least once).  Returns (samples, seconds, bytes)
    summed over the repetitions."""
    import oracle
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    rng = np.random.default_rng(seed)
    samples = np.sort(rng.choice(batch.B, size=min(n_samples, batch.B), replace=False))
    F, B = batch.F, batch.B
    offs = batch.offsets.astype(np.int64)
    tables, sub_idx, sub_off = [], [], [0]
    for f in range(F):
        bags = [batch.indices[offs[f * B + s]:offs[f * B + s + 1]] for s in samples]
        ids = np.concatenate(bags) if bags else np.zeros(0, np.int32)
        uniq, inv = np.unique(ids, return_inverse=True)
        if uniq.size == 0:
            uniq = np.zeros(1, np.int64)
        feat = model.features[f]
        tables.append(synth.table_rows_stored(feat.table, uniq, feat.dim, dtype, 'float', seed=model.seed))
        pos = 0
        for bag in bags:
            sub_idx.append(inv[pos:pos + bag.size].astype(np.int32))
            pos += bag.size
            sub_off.append(sub_off[-1] + bag.size)
    idx = np.concatenate(sub_idx) if sub_idx else np.zeros(0, np.int32)
    off = np.asarray(sub_off, np.int32)
    S = len(samples)
    # algorithmic bytes of the sample (C26)
    nnz_f = np.asarray([off[(f + 1) * S] - off[f * S] for f in range(F)], np.int64)
    dims = np.asarray(model.dims, np.int64)
    rowb = np.asarray([synth.row_bytes(d, dtype) for d in model.dims], np.int64)
    alg = 4 * int(nnz_f.sum()) + int((rowb * nnz_f).sum()) + 4 * S * int(dims.sum())
    pools = [f.pool for f in model.features]
    reps, dt = 0, 0.0
    while reps == 0 or (dt < min_seconds and reps < max_reps):
        t0 = time.perf_counter()
        oracle.embedding_bag(tables, model.dims, pools, idx, off, S, nthreads=nthreads, dtypes=[dtype] * F)
        dt += time.perf_counter() - t0
        reps += 1
    return S * reps, dt, alg * reps


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle timed on the host cores (rank 0 only)."""
    if rank != 0:
        return 0
    import oracle
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    model = synth.make_model(args.config)
    batch = synth.make_batch(model, 7)
    cores = len(os.sched_getaffinity(0))
    n = args.ref_samples
    for _ in range(args.warmup):
        oracle_sample_rate(model, batch, max(8, n // 8), seed=99, nthreads=cores)
    tot_s, tot_t, tot_b = 0, 0.0, 0
    for i in range(args.steps):
        S, dt, alg = oracle_sample_rate(model, batch, n, seed=i, nthreads=cores)
        tot_s += S
        tot_t += dt
        tot_b += alg
    value = tot_s / tot_t
    line = {
        'impl': 'reference', 'metric': _baseline_metric(), 'value': value, 'unit': 'samples/s',
        'n_gpus': world, 'steps': args.steps, 'warmup': args.warmup, 'ms_per_step': 1e3 * tot_t / args.steps,
        'higher_is_better': True, 'scaling': 'strong', 'vs_baseline': None,
        'dtype': 'f64', 'data': 'synthetic',
        'config': _workload_config(args, model, world),
        'effective_gbs': tot_b / tot_t / 1e9,
        'cpu_baseline': {'value': value, 'unit': 'samples/s', 'cores': cores, 'kind': 'oracle',
                         'cpu_model': _cpu_model(),
                         'sample': f'{args.steps} steps x {n} random samples (all {model.F} fields) of batch seed 7'},
        'e2e': {'value': value, 'unit': 'samples/s', 'h2d_bytes_per_step': 0, 'd2h_bytes_per_step': 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------------- GPU arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument('--gpus', type=int, default=1)
    ap.add_argument('--steps', type=int, default=20)
    ap.add_argument('--warmup', type=int, default=5)
    ap.add_argument('--impl', default='ours', choices=['ours', 'reference'])
    ap.add_argument('--config', default='sharded1000')
    ap.add_argument('--mode', default='float', choices=['float', 'int'])
    ap.add_argument('--dtype', default='f32', choices=['f32', 'f16', 'bf16', 'i8', 'fp8'],
                    help='table row storage (SURVEY NEXT #3); accumulation and output stay fp32')
    ap.add_argument('--batches', type=int, default=3)
    ap.add_argument('--plan', default='auto', help="tuned plan JSON, 'auto' (configs/tuned/) or 'none'")
    ap.add_argument('--tune', action='store_true', help='run the two-stage tuner before timing')
    ap.add_argument('--occupancy', type=int, default=0)
    ap.add_argument('--no-e2e', action='store_true')
    ap.add_argument('--no-cpu-baseline', action='store_true')
    ap.add_argument('--ref-samples', type=int, default=1024, help='reference arm: samples per step')
    ap.add_argument('--cpu-samples', type=int, default=1024, help='cpu_baseline: samples in the bounded sample')
    ap.add_argument('--cpu-seconds', type=float, default=10.0, help='cpu_baseline: minimum timed CPU seconds')
    ap.add_argument('--profile-only', action='store_true', help='short run for ncu (no e2e / cpu / clocks)')
    ap.add_argument('--exchange', default='nccl', choices=['nccl', 'fused'],
                    help='N>1: NCCL alltoallv + relayout kernel, or peer stores fused into the kernel epilogue')
    ap.add_argument('--no-heavy', action='store_true',
                    help='N=1: skip timing the heavy (north-star >= 70 %% HBM) workload in the same run')
    ap.add_argument('--no-jit', action='store_true',
                    help='time the precompiled catalog kernel instead of the plan-specialised (NVRTC) one')
    ap.add_argument('--no-graph', action='store_true',
                    help='N=1: launch each step eagerly instead of replaying its captured CUDA graph')
    ap.add_argument('--input-dist', action='store_true',
                    help='start each step from data-parallel local batches (B/W samples, all features) and run '
                         'the KJT input distribution (pack -> alltoallv -> unpack) inside the timed step')
    args = ap.parse_args()

    world = int(os.environ.get('WORLD_SIZE', '1'))
    rank = int(os.environ.get('RANK', '0'))
    local_rank = int(os.environ.get('LOCAL_RANK', '0'))
    # test plumbing only: run the N > 1 path with several ranks on ONE GPU (gloo,
    # exchange staged through host memory) -- RECFLEX_DIST_BACKEND=gloo RECFLEX_BENCH_DEVICE=0
    backend = os.environ.get('RECFLEX_DIST_BACKEND', 'nccl')
    if os.environ.get('RECFLEX_BENCH_DEVICE') is not None:
        local_rank = int(os.environ['RECFLEX_BENCH_DEVICE'])

    if args.impl == 'reference':
        return run_reference(args, rank, world)

    import torch
    import torch.distributed as dist
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import shard_concat
    from paper_conf_sc_panzzxwslr0d24_b200.shard import (KJTInputDist, ShardedEmbedding, exchange, model_parts,
                                                          sample_slice, shard_batch)

    torch.cuda.set_device(local_rank)
    dev = torch.device('cuda', local_rank)
    if world > 1:
        if backend == 'nccl':
            dist.init_process_group('nccl', device_id=dev)
        else:
            dist.init_process_group(backend)

    model = synth.make_model(args.config)
    B = model.batch
    parts = model_parts(model, world, args.dtype, args.config, os.path.join(ROOT, 'configs', 'tuned'))
    if world > 1 and args.exchange == 'fused':
        from paper_conf_sc_panzzxwslr0d24_b200.shard import FusedShardedEmbedding
        sh = FusedShardedEmbedding(model, rank, world, device=local_rank, parts=parts, dtype=args.dtype)
    else:
        sh = ShardedEmbedding(model, rank, world, device=local_rank, parts=parts, dtype=args.dtype)
    plan = sh.plan
    feats = sh.features

    # tables of my features (physical tables generated once, aliased per feature)
    phys = {}
    for f in feats:
        t = model.features[f].table
        if t not in phys:
            rows, dim = model.tables[t]
            phys[t] = synth.make_table_stored(t, rows, dim, args.dtype, args.mode, device=dev, seed=model.seed)
    tables = [phys[model.features[f].table] for f in feats]

    # batches: the global batch for my features, resident in HBM
    batches, host_batches, alg_bytes, local_batches = [], [], [], []
    dims_local = np.asarray([model.dims[f] for f in feats], np.int64)
    rowb_local = np.asarray([synth.row_bytes(model.dims[f], args.dtype) for f in feats], np.int64)
    for i in range(args.batches):
        full = synth.make_batch(model, 7 + i)
        idx, off = shard_batch(full, feats)
        host_batches.append((idx, off))
        batches.append((torch.from_numpy(idx).to(dev), torch.from_numpy(off).to(dev)))
        if args.input_dist:
            li, lo = sample_slice(full, rank, world)
            local_batches.append((torch.from_numpy(li).to(dev), torch.from_numpy(lo).to(dev)))
        o = off.astype(np.int64)
        nnz_f = o[np.arange(1, len(feats) + 1) * B] - o[np.arange(0, len(feats)) * B]
        # C26: IDs + gathered rows (stored bytes) + pooled fp32 output
        alg_bytes.append(4 * int(nnz_f.sum()) + int((rowb_local * nnz_f).sum()) + 4 * B * int(dims_local.sum()))
    alg_local = float(np.mean(alg_bytes))
    ws = alg_local + sum(t.numel() * t.element_size() for t in tables)
    flush_between = (alg_local < 4 * L2_BYTES)

    # tuned plan (stage-1/2 result exported by tools/tune_plan.py) or live tuning
    plan_src = 'default (untuned heuristic)'
    if args.tune:
        hist = [(bi, bo, B) for (bi, bo) in batches[:2]]
        st = plan.tune(hist, tables, verbose=(rank == 0))
        plan_src = f"tuned live ({st['tune_seconds']:.0f}s, k={st['best_occupancy']})"
    elif args.plan != 'none':
        path = args.plan
        if path == 'auto':
            path = os.path.join(ROOT, 'configs', 'tuned', f'{args.config}_w{world}_r{rank}.json')
        if args.dtype != 'f32' and args.plan == 'auto':
            path = os.path.join(ROOT, 'configs', 'tuned', f'{args.config}_{args.dtype}_w{world}_r{rank}.json')
        if os.path.exists(path):
            try:
                with open(path) as fh:
                    plan.import_(json.load(fh))
                plan_src = os.path.relpath(path, ROOT)
            except Exception as ex:  # stale plan (e.g. a different partition): keep the heuristic defaults
                plan_src = f'default (untuned heuristic; {os.path.relpath(path, ROOT)} rejected: {ex})'
    if args.occupancy:
        plan.occupancy = args.occupancy
    # the paper's fusion compiler: the plan's schedules inlined into one kernel (NVRTC)
    jit = None
    ksel = None
    if not args.no_jit:
        jit = plan.compile()
        # stage 2 over the plan's two kernels (plan-specialised vs catalog) on the first batch
        # small (latency-bound) steps are noisy at 5 repetitions: time them longer
        ksel = plan.select_kernel(batches[0][0], batches[0][1], B, tables, reps=5 if alg_local > 1e9 else 31)
        if not plan.jit_enabled:
            jit = dict(jit, active=0)

    out_local = torch.empty((B, sh.d_local), dtype=torch.float32, device=dev)
    out_x = torch.empty((B // world, sh.d_tot), dtype=torch.float32, device=dev) if world > 1 else None
    flush_buf = torch.empty(2 * L2_BYTES // 4, dtype=torch.float32, device=dev) if flush_between else None
    stream = torch.cuda.current_stream()

    ind = KJTInputDist(parts, model.F, rank, world, B // world, device=local_rank) if args.input_dist else None

    def step(i):
        if ind is not None:
            bi, bo = ind.forward(*local_batches[i % len(local_batches)])
        else:
            bi, bo = batches[i % len(batches)]
        return sh.forward(bi, bo, B, tables, out_local=out_local, out=out_x)

    def barrier():
        if world > 1:
            dist.barrier()

    from paper_conf_sc_panzzxwslr0d24_b200.plan import l2_flush

    for i in range(args.warmup):
        step(i)
    torch.cuda.synchronize()

    # N = 1: each rotating batch's forward (map + fused kernel, PDL-chained) captured
    # once as a CUDA graph and replayed per step -- no host launch work in the loop
    graphs = None
    eager_step = step
    if world == 1 and ind is None and not args.no_graph and not args.profile_only:
        try:
            graphs = []
            cap = torch.cuda.Stream()
            cap.wait_stream(torch.cuda.current_stream())
            for j in range(len(batches)):
                g = torch.cuda.CUDAGraph()
                with torch.cuda.graph(g, stream=cap):
                    step(j)
                graphs.append(g)
            torch.cuda.current_stream().wait_stream(cap)
            torch.cuda.synchronize()

            def step(i):  # noqa: F811
                graphs[i % len(graphs)].replay()
            for i in range(args.warmup):
                step(i)
            torch.cuda.synchronize()
        except Exception as ex:  # capture unsupported here: stay eager
            print(f'[bench] CUDA graph capture failed ({ex}); timing eager launches', file=sys.stderr)
            graphs = None
            step = eager_step

    clocks = ClockSampler(local_rank) if not args.profile_only else None
    if clocks:
        clocks.start()
        time.sleep(0.3)
    barrier()
    torch.cuda.synchronize()
    # every step bracketed by events on the launching stream: the headline is the
    # first-to-last span (or, with L2 flushes between steps, the sum of the steps)
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    for i in range(args.steps):
        if flush_between:
            l2_flush(flush_buf)
        evs[i][0].record(stream)
        step(i)
        evs[i][1].record(stream)
    torch.cuda.synchronize()
    per_step = [a_.elapsed_time(b_) for a_, b_ in evs]
    elapsed_ms = sum(per_step) if flush_between else evs[0][0].elapsed_time(evs[-1][1])
    barrier()
    clk = clocks.stop() if clocks else None

    def max_over_ranks(x):
        if world == 1:
            return float(x)
        t = torch.tensor([float(x)], dtype=torch.float64, device=dev if backend == 'nccl' else 'cpu')
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def sum_over_ranks(x):
        if world == 1:
            return float(x)
        t = torch.tensor([float(x)], dtype=torch.float64, device=dev if backend == 'nccl' else 'cpu')
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        return float(t.item())

    elapsed_ms = max_over_ranks(elapsed_ms)
    median_ms = max_over_ranks(float(np.median(per_step)))
    ms_per_step = elapsed_ms / args.steps
    value = B * args.steps / (elapsed_ms / 1e3)
    alg_all = sum_over_ranks(alg_local)  # every rank's algorithmic bytes of one step

    # per-kernel device time (events on the launch stream; PDL off in this pass)
    plan.set_profiling(True)
    plan.kernel_times(reset=True)
    for i in range(args.steps):
        if flush_between:
            l2_flush(flush_buf)
        bi, bo = batches[i % len(batches)]
        plan.forward(bi, bo, B, tables, out=out_local)
    kt = plan.kernel_times(reset=True)
    plan.set_profiling(False)
    fused_ms = kt['fused_ms'] / max(1, kt['forwards'])
    map_ms = kt['map_ms'] / max(1, kt['forwards'])
    peak, peak_src = _peaks()
    achieved = alg_local / (fused_ms / 1e3) / 1e9
    eff_gbs_step = alg_all / (ms_per_step / 1e3) / 1e9

    # N > 1: the step split into this rank's compute (map + fused) and the exchange,
    # per-rank medians, max over ranks; bounds from the NVLink all-to-all
    multi = None
    if world > 1 and ind is None:
        comp, tot = [], []
        for i in range(max(3, min(args.steps, 10))):
            bi, bo = batches[i % len(batches)]
            barrier()
            e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
            e[0].record(stream)
            plan.forward(bi, bo, B, tables, out=out_local)
            e[1].record(stream)
            if args.exchange == 'nccl':
                # the exchange alone: alltoallv of this rank's pooled rows + relayout kernel
                recv = exchange(out_local, sh.dims_per_rank, B)
                shard_concat(recv, sh.dims_per_rank, B // world, out_x)
            else:
                step(i)  # fused: compute + peer stores + completion wait, as timed
            e[2].record(stream)
            torch.cuda.synchronize()
            comp.append(e[0].elapsed_time(e[1]))
            tot.append(e[1].elapsed_time(e[2]))
        comp_ms = float(np.median(comp))
        # nccl: step = compute + exchange; fused: the fused step itself
        step_ms = comp_ms + float(np.median(tot)) if args.exchange == 'nccl' else float(np.median(tot))
        rows = B // world
        send = rows * sh.d_local * 4 * (world - 1)
        recv = rows * (sh.d_tot - sh.d_local) * 4
        a2a_bytes = max(send, recv)
        nvlink = 770e9  # measured peer copy per direction (B200_PROFILING.md; nominal 900 GB/s)
        a2a_ms = a2a_bytes / nvlink * 1e3
        relayout_ms = (2.0 * rows * sh.d_tot * 4) / (peak * 1e9) * 1e3 if args.exchange == 'nccl' else 0.0
        comp_max = max_over_ranks(comp_ms)
        a2a_max = max_over_ranks(a2a_ms)
        multi = {
            'compute_ms_max_rank': comp_max,
            'compute_ms_this_rank': comp_ms,
            'step_ms_max_rank': max_over_ranks(step_ms),
            'exchange_ms_max_rank': max_over_ranks(step_ms - comp_ms),
            'exchange': ('NCCL alltoallv + relayout kernel' if args.exchange == 'nccl' else
                         'peer stores in the fused kernel epilogue + device-side flags (recflex_forward_exchange)'),
            'nvlink': {'a2a_bytes_max_rank': max_over_ranks(a2a_bytes), 'gbs_per_direction': nvlink / 1e9,
                       'gbs_source': 'measured B200 peer copy, B200_PROFILING.md (nominal 900)',
                       'a2a_ms_at_peak': a2a_max, 'relayout_ms_at_hbm_peak': max_over_ranks(relayout_ms),
                       'serial_bound_ms': comp_max + a2a_max + max_over_ranks(relayout_ms),
                       'overlapped_bound_ms': max(comp_max, a2a_max),
                       'samples_per_s_serial_bound': B / ((comp_max + a2a_max + max_over_ranks(relayout_ms)) / 1e3),
                       'samples_per_s_overlapped_bound': B / (max(comp_max, a2a_max) / 1e3)},
            'note': 'compute = this plan\'s map + fused kernels alone; step = the timed step (compute + exchange)',
        }

    # DRAM traffic of the fused kernel from a committed ncu capture of THIS workload and rank plan
    traffic = None
    tname = f'ncu_traffic_{args.config}' + ('' if args.dtype == 'f32' else f'_{args.dtype}') + \
        ('' if world == 1 else f'_w{world}_r{rank}') + '.json'
    tp = os.path.join(ROOT, 'profiles', tname)
    if os.path.exists(tp):
        try:
            with open(tp) as fh:
                traffic = json.load(fh).get('dram_bytes_per_launch')
        except Exception:
            traffic = None

    # end-to-end through the public API from pinned host buffers
    e2e = None
    if not args.no_e2e and not args.profile_only:
        hb = [(torch.from_numpy(i).pin_memory(), torch.from_numpy(o).pin_memory()) for i, o in host_batches]
        if world == 1:
            # the public serving entry point over host batches: H2D of step i+1 and
            # D2H of step i-1 overlap the forward of step i (recflex_forward_host_batches)
            houts = [torch.empty((B, sh.d_local), dtype=torch.float32).pin_memory() for _ in range(2)]
            hout = houts[0]
            plan.forward_host_batches([(hb[0][0], hb[0][1], B)], tables, [houts[0]])
            torch.cuda.synchronize()
            ke = max(3, min(args.steps, 10))
            seq = [(hb[i % len(hb)][0], hb[i % len(hb)][1], B) for i in range(ke)]
            t0 = time.perf_counter()
            plan.forward_host_batches(seq, tables, [houts[i % 2] for i in range(ke)])
            dt = time.perf_counter() - t0
            h2d = float(np.mean([hi.numel() * 4 + ho.numel() * 4 for hi, ho in hb]))
            d2h = hout.numel() * 4
        else:
            hout = torch.empty((B // world, sh.d_tot), dtype=torch.float32).pin_memory()
            di = [torch.empty_like(b[0], device=dev) for b in hb]
            do = [torch.empty_like(b[1], device=dev) for b in hb]
            ke = max(3, min(args.steps, 10))
            barrier()
            t0 = time.perf_counter()
            for i in range(ke):
                j = i % len(hb)
                di[j].copy_(hb[j][0], non_blocking=True)
                do[j].copy_(hb[j][1], non_blocking=True)
                o = sh.forward(di[j], do[j], B, tables, out_local=out_local, out=out_x)
                hout.copy_(o, non_blocking=True)
                torch.cuda.current_stream().synchronize()
            dt = time.perf_counter() - t0
            dt = max_over_ranks(dt)
            h2d = float(np.mean([hi.numel() * 4 + ho.numel() * 4 for hi, ho in hb]))
            d2h = hout.numel() * 4
        e2e = {'value': B * ke / dt, 'unit': 'samples/s', 'h2d_bytes_per_step': int(h2d),
               'd2h_bytes_per_step': int(d2h), 'steps': ke, 'timing': 'wall clock per rank, max over ranks',
               'api': ('recflex_forward_host_batches (pinned host KJT in, pinned host output back; copies '
                       'overlapped with the forwards of neighbouring steps)' if world == 1 else
                       'torch H2D copies + ShardedEmbedding.forward + D2H, serial per step')}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline and not args.profile_only:
        try:
            from paper_conf_sc_panzzxwslr0d24_b200 import synth as _s
            full = _s.make_batch(model, 7)
            cores = len(os.sched_getaffinity(0))
            S, dt, alg = oracle_sample_rate(model, full, args.cpu_samples, seed=0, nthreads=cores,
                                            min_seconds=args.cpu_seconds, dtype=args.dtype)
            cpu = {'value': S / dt, 'unit': 'samples/s', 'cores': cores, 'kind': 'oracle', 'cpu_model': _cpu_model(),
                   'sample': f'{args.cpu_samples} random samples x all {model.F} fields of batch seed 7, '
                             f'oracle repeated to {dt:.1f} s ({S} samples total; fp64 C oracle, OpenMP)',
                   'effective_gbs': alg / dt / 1e9, 'seconds': dt}
        except Exception as ex:  # never fail the bench line on the baseline leg
            cpu = {'value': None, 'unit': 'samples/s', 'cores': None, 'kind': 'oracle', 'sample': f'failed: {ex}'}

    launches_per_step = 2 + (1 if plan.export() and any(s[1] == 1 for s in plan.export()['schedules']) else 0)
    launches_per_step += 1 if (world > 1 and args.exchange == 'nccl') else 0   # relayout kernel
    launches_per_step += 1 if (world > 1 and args.exchange == 'fused') else 0  # exchange wait kernel
    launches_per_step += 5 if args.input_dist else 0  # pack scan + copy, unpack reduce + scan + main

    # the north-star target configuration (>= 70 % of HBM on the large multi-hot
    # model), timed in the same run at N = 1 (the headline stays the config above)
    launch_desc = 'CUDA graph replay per step' if graphs else 'eager'
    heavy = None
    if world == 1 and args.config != 'heavy' and not args.no_heavy and not args.profile_only:
        del tables, phys, batches, graphs
        torch.cuda.empty_cache()
        try:
            heavy = time_config('heavy', args, dev, peak)
        except Exception as ex:  # never fail the bench line on the extra leg
            heavy = {'failed': str(ex)[:300]}

    if rank == 0:
        line = {
            'metric': _baseline_metric(),
            'value': value,
            'unit': 'samples/s',
            'n_gpus': world,
            'steps': args.steps,
            'warmup': args.warmup,
            'ms_per_step': ms_per_step,
            'ms_per_step_median': median_ms,
            'higher_is_better': True,
            'scaling': 'strong',
            'vs_baseline': None,
            'dtype': 'f32' if args.dtype == 'f32' else f'{args.dtype} rows, f32 accumulate/output',
            'data': 'synthetic (seeded generator, SURVEY §8d recipe; tables: counter-based hash U[-1,1))',
            'config': _workload_config(args, model, world),
            'impl_config': {'plan': plan_src, 'occupancy': plan.occupancy,
                            **({'dist_backend': backend} if world > 1 else {}),
                            'exchange': (args.exchange if world > 1 else 'none'),
                            'launch': launch_desc,
                            'kernel': (f"plan-specialised (NVRTC, {jit['variants']} variants, {jit['registers']} "
                                       f"regs, {jit['local_bytes']} B local)" if jit and jit['active'] else 'catalog'),
                            'kernel_selection': ksel,
                            'task_order': task_order_name(plan),
                            'l2_policy': l2_policy_summary(plan),
                            'output_columns': ('task order (features concatenated in the order their tasks '
                                               'run; recflex_get_columns)' if plan.export().get('columns')
                                               else 'feature order'),
                            'input': ('data-parallel local batches + KJT input dist in the timed step'
                                      if args.input_dist else 'table-wise KJT resident per rank'),
                            'l2': 'flushed between steps' if flush_between else
                                  f'inputs > L2 ({alg_local / 1e9:.2f} GB algorithmic per step per rank, '
                                  f'{args.batches} rotating batches)'},
            'effective_hbm_gbs': eff_gbs_step,
            'pct_of_8tbs': 100.0 * eff_gbs_step / (8000.0 * world),
            'roofline': {'bound': 'hbm', 'achieved': achieved, 'peak': peak, 'unit': 'GB/s',
                         'frac': achieved / peak, 'traffic': traffic,
                         'kernel': (f'recflex_fused_jit_k{plan.occupancy}' if jit and jit['active']
                                    else 'recflex_fused_kernel'),
                         'peak_source': peak_src, 'fused_ms': fused_ms, 'map_ms': map_ms,
                         'algorithmic_bytes_per_launch': alg_local,
                         'traffic_source': (os.path.relpath(tp, ROOT) if traffic is not None else
                                            'no ncu capture of this workload / rank plan committed')},
            'multi_gpu': multi,
            'heavy': heavy,
            'e2e': e2e,
            'gpu_launches': launches_per_step * args.steps,
            'clocks': clk,
            'cpu_baseline': cpu,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def time_config(config, args, dev, peak, steps=20, warmup=5, nbatches=3):
    """One extra workload at N = 1 in the same run: tuned plan, plan-specialised
    kernel, CUDA-graph replay per rotating batch, event-timed K steps (inputs >
    L2), clocks sampled during the timed region, fused-kernel roofline."""
    import torch
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan
    m = synth.make_model(config)
    phys = {}
    for f in m.features:
        if f.table not in phys:
            rows, dim = m.tables[f.table]
            phys[f.table] = synth.make_table_stored(f.table, rows, dim, 'f32', 'float', device=dev, seed=m.seed)
    tables = [phys[f.table] for f in m.features]
    plan = Plan.from_model(m)
    path = os.path.join(ROOT, 'configs', 'tuned', f'{config}_w1_r0.json')
    if os.path.exists(path):
        with open(path) as fh:
            plan.import_(json.load(fh))
    plan.compile()
    bts, alg = [], []
    for i in range(nbatches):
        b = synth.make_batch(m, 7 + i)
        bts.append((torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev)))
        alg.append(synth.algorithmic_bytes(m, b, 'f32')['total'])
    ksel = plan.select_kernel(bts[0][0], bts[0][1], m.batch, tables, reps=5)
    alg_b = float(np.mean(alg))
    out = torch.empty((m.batch, m.d_tot), dtype=torch.float32, device=dev)
    for i in range(warmup):
        plan.forward(*bts[i % nbatches], m.batch, tables, out=out)
    cap = torch.cuda.Stream()
    cap.wait_stream(torch.cuda.current_stream())
    graphs = []
    for j in range(nbatches):
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=cap):
            plan.forward(*bts[j], m.batch, tables, out=out, stream=cap)
        graphs.append(g)
    torch.cuda.current_stream().wait_stream(cap)
    for i in range(warmup):
        graphs[i % nbatches].replay()
    torch.cuda.synchronize()
    clocks = ClockSampler(dev.index)
    clocks.start()
    time.sleep(0.3)
    stream = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for i in range(steps):
        graphs[i % nbatches].replay()
    e1.record(stream)
    torch.cuda.synchronize()
    clk = clocks.stop()
    ms = e0.elapsed_time(e1) / steps
    plan.set_profiling(True)
    plan.kernel_times(reset=True)
    for i in range(steps):
        plan.forward(*bts[i % nbatches], m.batch, tables, out=out)
    kt = plan.kernel_times(reset=True)
    plan.set_profiling(False)
    fused_ms = kt['fused_ms'] / max(1, kt['forwards'])
    res = {'workload': config, 'global_batch': m.batch, 'fields': m.F, 'steps': steps, 'warmup': warmup,
           'ms_per_step': ms, 'samples_per_s': m.batch / (ms / 1e3),
           'effective_hbm_gbs': alg_b / (ms / 1e3) / 1e9, 'pct_of_8tbs': 100.0 * alg_b / (ms / 1e3) / 8e12,
           'roofline': {'bound': 'hbm', 'achieved': alg_b / (fused_ms / 1e3) / 1e9, 'peak': peak, 'unit': 'GB/s',
                        'frac': alg_b / (fused_ms / 1e3) / 1e9 / peak, 'fused_ms': fused_ms,
                        'kernel': f'recflex_fused_jit_k{plan.occupancy}' if plan.jit_enabled else 'recflex_fused_kernel',
                        'algorithmic_bytes_per_launch': alg_b},
           'plan': os.path.relpath(path, ROOT), 'occupancy': plan.occupancy, 'kernel_selection': ksel,
           'task_order': task_order_name(plan),
           'output_columns': 'task order' if plan.export().get('columns') else 'feature order',
           'l2': f'inputs > L2 ({alg_b / 1e9:.1f} GB algorithmic per step, {nbatches} rotating batches)',
           'launch': 'CUDA graph replay per step', 'clocks': clk}
    del graphs, tables, phys, bts
    torch.cuda.empty_cache()
    return res


if __name__ == '__main__':
    sys.exit(main())
