"""GPU parity of every tuned plan bench.py can load (configs/tuned/<config>[_<dtype>]_w1_r0.json)
at the BASELINE.json full size, in BOTH kernels that can run it: the precompiled catalog kernel
and the plan-specialised kernel (recflex_plan_compile, the configuration bench.py times).

Bars: integer-valued tables bit-exact against the oracle; U[-1,1) tables within
|gpu - oracle| <= 1e-5 (1 + |oracle|) sqrt(L); the two kernels bitwise identical to each other
(same schedule templates, same accumulation order).  Batches of B <= 4096 (fig3, medium,
industrial) are checked on EVERY sample; heavy (8192) and sharded1000 (16384) on 1024 random
samples plus the first and last.
"""
import glob
import json
import os

import numpy as np
import pytest
import torch

from fullsize import sampled_oracle
from paper_conf_sc_panzzxwslr0d24_b200 import synth
from test_gpu_parity import bitexact, check_tol, feature_columns

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
TUNED = os.path.join(ROOT, 'configs', 'tuned')
DTYPES = ('f16', 'bf16', 'i8', 'fp8')


def _plans():
    out = []
    for p in sorted(glob.glob(os.path.join(TUNED, '*_w1_r0.json'))):
        name = os.path.basename(p)[:-len('_w1_r0.json')]
        cfg, _, dt = name.rpartition('_')
        out.append((cfg, dt) if dt in DTYPES else (name, 'f32'))
    return out


def _samples(B, n=1024, seed=5):
    if B <= 4096:
        return np.arange(B)
    rng = np.random.default_rng(seed)
    return np.unique(np.concatenate([[0, B - 1], rng.choice(B, n, replace=False)]))


def test_every_bench_plan_is_listed():
    """bench.py --config X --dtype D loads configs/tuned/X[_D]_w1_r0.json: all of them are here."""
    assert {'medium', 'industrial', 'heavy', 'sharded1000', 'fig3'} <= {c for c, _ in _plans()}
    assert len(_plans()) == len(glob.glob(os.path.join(TUNED, '*_w1_r0.json')))


@pytest.mark.parametrize('mode', ['int', 'float'])
@pytest.mark.parametrize('config,dtype', _plans())
def test_tuned_plan_both_kernels_vs_oracle(config, dtype, mode):
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan
    dev = torch.device('cuda', 0)
    m = synth.make_model(config)
    b = synth.make_batch(m, 7)
    phys = {}
    for feat in m.features:
        if feat.table not in phys:
            rows, dim = m.tables[feat.table]
            phys[feat.table] = synth.make_table_stored(feat.table, rows, dim, dtype, mode, device=dev, seed=m.seed)
    tables = [phys[f.table] for f in m.features]
    plan = Plan.from_model(m, dtype=dtype)
    path = os.path.join(TUNED, f'{config}_w1_r0.json' if dtype == 'f32' else f'{config}_{dtype}_w1_r0.json')
    plan.import_(json.load(open(path)))
    idx = torch.from_numpy(b.indices).to(dev)
    off = torch.from_numpy(b.offsets).to(dev)
    plan.set_jit(False)
    out_cat = plan.forward(idx, off, b.B, tables)
    plan.compile()
    plan.set_jit(True)
    info = plan.jit_info()
    assert info['active'] == 1 and info['blocks_per_sm'] == plan.occupancy, info
    out_jit = plan.forward(idx, off, b.B, tables)
    torch.cuda.synchronize()
    assert torch.equal(out_cat, out_jit), 'plan-specialised kernel differs from the catalog kernel'
    samples = _samples(b.B)
    ref, lens = sampled_oracle(m, b, samples, tables, dtype)
    got = feature_columns(out_jit[torch.as_tensor(samples, device=dev)].cpu().numpy(), plan, m.dims)
    if mode == 'int':
        assert bitexact(got, ref)
    else:
        check_tol(got, ref, lens, m.dims)
    del phys, tables, out_cat, out_jit
    torch.cuda.empty_cache()
