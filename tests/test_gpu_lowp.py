"""GPU parity for reduced-precision table rows: float16,
bfloat16, rowwise int8 and FP8 E4M3 storage, fp32 accumulation, fp32 output.

The oracle decodes every stored element in fp64 (oracle_decode: IEEE binary16
from its fields, bfloat16 as the upper half of a binary32, int8 as scale*q+bias)
and pools in fp64; the CUDA path widens in registers and pools in fp32.  Bars,
as for fp32 rows:
  * 'int' tables (every stored value an exact small integer, i8 with scale 1
    and an integer bias): BIT-EXACT;
  * 'float' tables: |gpu - oracle| <= 1e-5 * (1 + |oracle|) * sqrt(L).
"""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_sc_panzzxwslr0d24_b200 import synth

from test_gpu_parity import bitexact, check_tol

pytestmark = pytest.mark.gpu

LOWP = ('f16', 'bf16', 'i8', 'fp8')


def _P():
    from paper_conf_sc_panzzxwslr0d24_b200 import plan
    return plan


class TypedCase:
    """Model + batch + stored tables on cuda:0; dtypes per feature."""

    def __init__(self, model, batch, dtypes, mode='float'):
        self.model, self.batch, self.mode = model, batch, mode
        self.dtypes = [dtypes] * model.F if isinstance(dtypes, str) else list(dtypes)
        dev = torch.device('cuda', 0)
        cache = {}
        self.tables = []
        for f, feat in enumerate(model.features):
            key = (feat.table, self.dtypes[f])
            if key not in cache:
                rows, dim = model.tables[feat.table]
                cache[key] = synth.make_table_stored(feat.table, rows, dim, self.dtypes[f], mode, device=dev,
                                                     seed=model.seed)
            self.tables.append(cache[key])
        self.idx = torch.from_numpy(batch.indices).to(dev)
        self.off = torch.from_numpy(batch.offsets).to(dev)
        self.B = batch.B

    def plan(self, max_batch=None):
        P = _P()
        specs = [dict(rows=f.rows, dim=f.dim, pool=f.pool, mean_len=f.mean_len(), max_len=f.max_len(),
                      coverage=f.coverage, dtype=self.dtypes[i]) for i, f in enumerate(self.model.features)]
        return P.Plan(specs, max_batch or self.B)

    def run(self, plan):
        out = plan.forward(self.idx, self.off, self.B, self.tables)
        torch.cuda.synchronize()
        return out.cpu().numpy()

    def oracle(self, samples=None):
        """fp64 oracle on the sampled bags; rows regenerated on the host in storage format."""
        if samples is None:
            samples = np.arange(self.B)
        m, b = self.model, self.batch
        F, B = b.F, b.B
        samples = np.asarray(samples, np.int64)
        offs = b.offsets.astype(np.int64)
        tabs, sub_idx, sub_off = [], [], [0]
        lens = np.zeros((samples.size, F), np.int64)
        for f, feat in enumerate(m.features):
            bags = [b.indices[offs[f * B + s]:offs[f * B + s + 1]] for s in samples]
            for k, bag in enumerate(bags):
                lens[k, f] = bag.size
            ids = np.concatenate(bags) if bags else np.zeros(0, np.int32)
            uniq, inv = np.unique(ids, return_inverse=True)
            if uniq.size == 0:
                uniq = np.zeros(1, np.int64)
            tabs.append(synth.table_rows_stored(feat.table, uniq, feat.dim, self.dtypes[f], self.mode,
                                                seed=m.seed))
            pos = 0
            for bag in bags:
                sub_idx.append(inv[pos:pos + bag.size].astype(np.int32))
                pos += bag.size
                sub_off.append(sub_off[-1] + bag.size)
        idx = np.concatenate(sub_idx) if sub_idx else np.zeros(0, np.int32)
        ref = oracle.embedding_bag(tabs, m.dims, [f.pool for f in m.features], idx, np.asarray(sub_off, np.int32),
                                   samples.size, dtypes=self.dtypes)
        return ref, lens


def _check(case, out, samples=None):
    ref, lens = case.oracle(samples)
    got = out if samples is None else out[samples]
    if case.mode == 'int':
        assert bitexact(got, ref)
    else:
        check_tol(got, ref, lens, case.model.dims)


# ---------------------------------------------------------------------------- configs

@pytest.mark.parametrize('dtype', LOWP)
@pytest.mark.parametrize('name', ['tiny', 'medium', 'fig3'])
def test_configs_full(name, dtype):
    m = synth.make_model(name)
    b = synth.make_batch(m, 7)
    for mode in ('int', 'float'):
        case = TypedCase(m, b, dtype, mode)
        _check(case, case.run(case.plan()))


@pytest.mark.parametrize('dtype', LOWP)
def test_industrial_sampled(dtype):
    m = synth.make_model('industrial')
    b = synth.make_batch(m, 7)
    case = TypedCase(m, b, dtype, 'float')
    out = case.run(case.plan())
    rng = np.random.default_rng(0)
    _check(case, out, np.unique(np.concatenate([[0, b.B - 1], rng.integers(0, b.B, 150)])))


@pytest.mark.parametrize('name,dtype', [('heavy', 'bf16'), ('heavy', 'i8'), ('heavy', 'fp8'), ('sharded1000', 'f16')])
def test_full_size_sampled(name, dtype):
    """BASELINE.json full sizes in bench.py's launch configuration (tuned plan if present); sampled rows,
    int bit-exact."""
    import json
    import os
    m = synth.make_model(name)
    b = synth.make_batch(m, 7)
    case = TypedCase(m, b, dtype, 'int')
    plan = case.plan()
    # the tuned plan bench.py --dtype loads, when there is one (its launch configuration)
    path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), 'configs', 'tuned',
                        f'{name}_{dtype}_w1_r0.json')
    if os.path.exists(path):
        plan.import_(json.load(open(path)))
    out = case.run(plan)
    rng = np.random.default_rng(2)
    _check(case, out, np.unique(np.concatenate([[0, b.B - 1], rng.integers(0, b.B, 40)])))
    del case
    torch.cuda.empty_cache()


# ---------------------------------------------------------------------------- every entry

def _lowp_model(dtype):
    dims = ([8, 16, 24, 32, 48, 64, 96, 128, 256, 8, 16, 40] if dtype in ('i8', 'fp8')
            else [4, 8, 12, 16, 24, 32, 64, 96, 128, 256, 40, 20])
    feats = []
    for i, d in enumerate(dims):
        kind = 'onehot' if i % 3 == 0 else 'uniform'
        feats.append(synth.Feature(rows=991 + 17 * i, dim=d, pool=i % 2, kind=kind,
                                   coverage=0.7 if kind == 'onehot' else 1.0, lo=0, hi=33 + 6 * i,
                                   lmax=1 if kind == 'onehot' else 33 + 6 * i, table=i))
    return synth.custom_model(f'lowp_{dtype}', feats, 257)


@pytest.mark.parametrize('dtype', LOWP)
@pytest.mark.parametrize('part', [0, 1])
def test_every_lowp_catalog_entry_int_bitexact(dtype, part):
    P = _P()
    m = _lowp_model(dtype)
    b = synth.make_batch(m, 3)
    case = TypedCase(m, b, dtype, 'int')
    ref, _ = case.oracle()
    col = np.cumsum([0] + m.dims)
    entries = [e for e in P.catalog() if e['dtype'] == dtype]
    assert len(entries) >= 20
    tested = 0
    for e in entries:
        for per_block in {0: (7, 64), 1: (5, 300)}[part]:
            plan = case.plan()
            used = []
            for f in range(m.F):
                try:
                    plan.set_schedule(f, e['id'], part, per_block)
                    used.append(f)
                except Exception:
                    pass  # entry not valid for this dim
            if not used:
                continue
            out = case.run(plan)
            for f in used:
                a, z = col[f], col[f + 1]
                assert bitexact(out[:, a:z], ref[:, a:z]), (e, f, per_block)
            tested += 1
    assert tested >= len(entries)


def test_fp32_entries_rejected_for_lowp_features_and_vice_versa():
    P = _P()
    m = _lowp_model('bf16')
    case = TypedCase(m, synth.make_batch(m, 3), 'bf16', 'int')
    plan = case.plan()
    for e in P.catalog():
        if e['dtype'] == 'f32':
            with pytest.raises(Exception):
                plan.set_schedule(1, e['id'], 0, 64)   # dim 8 bf16 feature
            break
    with pytest.raises(Exception):
        P.Plan([dict(rows=10, dim=6, dtype='f16')], 8)   # 16-bit rows need dim % 4 == 0
    with pytest.raises(Exception):
        P.Plan([dict(rows=10, dim=12, dtype='i8')], 8)   # int8 rows need dim % 8 == 0
    with pytest.raises(Exception):
        P.Plan([dict(rows=10, dim=12, dtype='fp8')], 8)  # fp8 rows need dim % 8 == 0
    with pytest.raises(ValueError):
        plan.forward(case.idx, case.off, case.B, [t.float() if t.dtype == torch.bfloat16 else t
                                                   for t in case.tables])


# ---------------------------------------------------------------------------- mixed storage in one kernel

def _mixed_dtypes(m):
    cyc = ['f32', 'f16', 'bf16', 'i8', 'fp8']
    return [cyc[i % 5] if (cyc[i % 5] not in ('i8', 'fp8') or f.dim % 8 == 0) else 'bf16'
            for i, f in enumerate(m.features)]


@pytest.mark.parametrize('mode', ['int', 'float'])
def test_mixed_dtypes_one_fused_kernel(mode):
    """Features with different storage types in ONE fused kernel (per-feature
    schedule switch, Fig. 8): industrial model, dtype cycling per feature."""
    m = synth.make_model('industrial')
    b = synth.make_batch(m, 9)
    case = TypedCase(m, b, _mixed_dtypes(m), mode)
    out = case.run(case.plan())
    rng = np.random.default_rng(4)
    _check(case, out, np.unique(np.concatenate([[0, b.B - 1], rng.integers(0, b.B, 100)])))


@pytest.mark.parametrize('k', [1, 3, 8])
def test_mixed_dtypes_occupancy_variants(k):
    m = _lowp_model('i8')
    case = TypedCase(m, synth.make_batch(m, 5), _mixed_dtypes(m), 'int')
    plan = case.plan()
    plan.occupancy = k
    _check(case, case.run(plan))


def test_tuner_on_lowp_plan_keeps_parity():
    m = synth.make_model('medium')
    bts = [synth.make_batch(m, 7 + i) for i in range(2)]
    case = TypedCase(m, bts[0], _mixed_dtypes(m), 'int')
    plan = case.plan()
    hist = [(torch.from_numpy(b.indices).cuda(), torch.from_numpy(b.offsets).cuda(), b.B) for b in bts]
    st = plan.tune(hist, case.tables, occupancies=[2, 4], reps=3)
    assert st['local_evals'] == m.F * 2
    for f in range(m.F):
        e = _P().catalog()[plan.get_schedule(f)['sched_id']]
        assert e['dtype'] == case.dtypes[f]
    _check(case, case.run(plan))
