"""GPU parity for the backward (training) path, SURVEY §8f NEXT #4:
recflex_backward against the fp64 oracle adjoint (oracle.embedding_bag_backward).

Bars:
  * integer data (gradients, initial targets and scale are small integers; MEAN
    features get gradients that are integer multiples of the bag length so
    G / L is an integer): every partial sum is exact in fp32, so the result is
    BIT-EXACT whatever order the L2 reductions happen in;
  * float data: per element |gpu - oracle| <= 2^-22 * n * (|T0| + A) + 1e-30,
    n = terms added to the row, A = sum of their magnitudes (the recursive
    summation bound n*u*sum|x_i| with u = 2^-24, 4x slack) -- the order of the
    reductions is not fixed.
"""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_sc_panzzxwslr0d24_b200 import synth

pytestmark = pytest.mark.gpu


def _P():
    from paper_conf_sc_panzzxwslr0d24_b200 import plan
    return plan


def _grad(model, batch, mode, seed):
    rng = np.random.default_rng(seed)
    B = batch.B
    if mode == 'float':
        return rng.uniform(-1, 1, (B, model.d_tot)).astype(np.float32)
    G = rng.integers(-8, 8, (B, model.d_tot)).astype(np.float64)
    lens = batch.lengths()  # [F][B]
    col = 0
    for f, feat in enumerate(model.features):
        if feat.pool == 1:
            G[:, col:col + feat.dim] *= np.maximum(lens[f], 1)[:, None]
        col += feat.dim
    return G.astype(np.float32)


def _run(model, batch, mode, scale=1.0, init=None, plan=None, seed=0, features=None):
    """Backward on the GPU over the whole batch; oracle per checked feature (the
    adjoint of one feature only reads that feature's bags).  Checked features:
    all of them for small models, else a seeded sample of 12 (incl. first/last)."""
    P = _P()
    dev = torch.device('cuda', 0)
    plan = plan or P.Plan.from_model(model, max_batch=batch.B)
    G = _grad(model, batch, mode, seed)
    gen = torch.Generator(device=dev)
    gen.manual_seed(seed + 1)
    targets = []
    for f in model.features:
        if init == 'int':
            targets.append(torch.randint(-8, 8, (f.rows, f.dim), generator=gen, device=dev).float())
        elif init == 'float':
            targets.append(torch.rand((f.rows, f.dim), generator=gen, device=dev) * 2 - 1)
        else:
            targets.append(torch.zeros((f.rows, f.dim), device=dev))
    if features is None:
        if sum(f.rows * f.dim for f in model.features) < 5e7:
            features = list(range(model.F))
        else:
            rng = np.random.default_rng(seed)
            features = sorted(set([0, model.F - 1] + rng.integers(0, model.F, 10).tolist()))
    T0 = {f: targets[f].cpu().numpy() for f in features}
    plan.backward(torch.from_numpy(batch.indices).to(dev), torch.from_numpy(batch.offsets).to(dev), batch.B,
                  torch.from_numpy(G).to(dev), targets, scale=scale)
    torch.cuda.synchronize()
    B = batch.B
    col = np.cumsum([0] + model.dims)
    res = []
    for f in features:
        feat = model.features[f]
        lo, hi = batch.offsets[f * B], batch.offsets[(f + 1) * B]
        off_f = (batch.offsets[f * B:(f + 1) * B + 1] - lo).astype(np.int32)
        ref, cnt, ab = oracle.embedding_bag_backward([feat.rows], [feat.dim], [feat.pool], batch.indices[lo:hi],
                                                     off_f, B, G[:, col[f]:col[f + 1]].astype(np.float64),
                                                     scale=scale, targets=[T0[f]])
        res.append((f, targets[f].cpu().numpy(), ref[0], cnt[0], ab[0], T0[f]))
    del targets
    return res


def _check(res, mode):
    for f, got, ref, cnt, ab, T0 in res:
        if mode == 'int':
            assert np.array_equal(got, ref.astype(np.float32)), f
        else:
            n = cnt[:, None].astype(np.float64)
            tol = 2.0 ** -22 * n * (np.abs(T0) + ab) + 1e-30
            err = np.abs(got.astype(np.float64) - ref)
            assert np.all(err <= tol), (f, float(np.max(err - tol)))
            untouched = cnt == 0
            assert np.array_equal(got[untouched], T0[untouched])


@pytest.mark.parametrize('name', ['tiny', 'medium', 'fig3'])
@pytest.mark.parametrize('mode', ['int', 'float'])
def test_backward_configs(name, mode):
    m = synth.make_model(name)
    b = synth.make_batch(m, 7)
    _check(_run(m, b, mode), mode)


def test_backward_industrial_sum_and_mean_float():
    m = synth.make_model('industrial')   # even features SUM, odd MEAN
    b = synth.make_batch(m, 7)
    _check(_run(m, b, 'float', init='float', scale=-0.03), 'float')


@pytest.mark.parametrize('scale,init', [(1.0, 'int'), (-1.0, 'int'), (-2.0, None)])
def test_backward_scale_and_initial_targets_int(scale, init):
    m = synth.make_model('medium')
    b = synth.make_batch(m, 8)
    _check(_run(m, b, 'int', scale=scale, init=init), 'int')


def _odd_model():
    dims = [1, 3, 4, 6, 8, 12, 16, 20, 32, 64, 128, 256]   # scalar and vector paths, several passes
    feats = []
    for i, d in enumerate(dims):
        kind = 'onehot' if i % 3 == 0 else 'uniform'
        feats.append(synth.Feature(rows=97 + 13 * i, dim=d, pool=i % 2, kind=kind,
                                   coverage=0.6 if kind == 'onehot' else 1.0, lo=0, hi=40 + 3 * i,
                                   lmax=1 if kind == 'onehot' else 40 + 3 * i, table=i))
    return synth.custom_model('bwd_odd', feats, 203)


@pytest.mark.parametrize('part', [0, 1])
def test_backward_odd_dims_all_partitions(part):
    """Unaligned dims (scalar atomics, and a plan whose D_tot % 4 != 0 forces the
    scalar path everywhere), heavy row collisions (~100 rows per table), every
    task-partition mode of the shared task map."""
    P = _P()
    m = _odd_model()
    b = synth.make_batch(m, 4)
    plan = P.Plan.from_model(m, max_batch=b.B)
    for f in range(m.F):
        s = plan.get_schedule(f)
        plan.set_schedule(f, s['sched_id'], part, {0: 5, 1: 200}[part])
    for mode in ('int', 'float'):
        _check(_run(m, b, mode, plan=plan, init=mode), mode)


def test_backward_empty_and_long_bags():
    m = _odd_model()
    lens = np.zeros((m.F, 40), np.int64)
    lens[2, 3] = 900       # one long bag (many reductions to a ~130-row table)
    lens[8, 39] = 1
    b = synth.batch_from_lengths(lens, [f.rows for f in m.features], seed=5)
    _check(_run(m, b, 'int', init='int'), 'int')


def test_backward_batch_zero_and_bad_args():
    P = _P()
    m = synth.make_model('tiny')
    b = synth.make_batch(m, 7)
    plan = P.Plan.from_model(m, max_batch=b.B)
    dev = torch.device('cuda', 0)
    targets = [torch.zeros((f.rows, f.dim), device=dev) for f in m.features]
    off0 = torch.zeros(1, dtype=torch.int32, device=dev)
    plan.backward(torch.zeros(1, dtype=torch.int32, device=dev), off0, 0,
                  torch.zeros((0, m.d_tot), device=dev), targets)
    assert all(float(t.abs().sum()) == 0 for t in targets)
    idx = torch.from_numpy(b.indices).to(dev)
    off = torch.from_numpy(b.offsets).to(dev)
    with pytest.raises(ValueError):
        plan.backward(idx, off, b.B, torch.zeros((b.B, m.d_tot + 1), device=dev), targets)
    with pytest.raises(ValueError):
        plan.backward(idx, off, b.B, torch.zeros((b.B, m.d_tot), device=dev),
                      [t.half() for t in targets])


def test_sgd_step_then_forward_matches_oracle():
    """One fused SGD step on fp32 tables, then the fused forward on the updated
    tables: both against the oracle (integer data, bit-exact)."""
    P = _P()
    m = synth.make_model('fig3')
    b = synth.make_batch(m, 7)
    dev = torch.device('cuda', 0)
    plan = P.Plan.from_model(m, max_batch=b.B)
    phys = [synth.make_table(t, r, d, 'int', device=dev, seed=m.seed) for t, (r, d) in enumerate(m.tables)]
    tables = [phys[f.table].clone() for f in m.features]
    T0 = [t.cpu().numpy() for t in tables]
    G = _grad(m, b, 'int', 3)
    idx = torch.from_numpy(b.indices).to(dev)
    off = torch.from_numpy(b.offsets).to(dev)
    plan.sgd_step(idx, off, b.B, torch.from_numpy(G).to(dev), tables, lr=2.0)
    out = plan.forward(idx, off, b.B, tables)
    torch.cuda.synchronize()
    newT, _, _ = oracle.embedding_bag_backward([f.rows for f in m.features], m.dims, [f.pool for f in m.features],
                                               b.indices, b.offsets, b.B, G.astype(np.float64), scale=-2.0,
                                               targets=T0)
    for f in range(m.F):
        assert np.array_equal(tables[f].cpu().numpy(), newT[f].astype(np.float32))
    ref = oracle.embedding_bag([t.astype(np.float32) for t in newT], m.dims, [f.pool for f in m.features],
                               b.indices, b.offsets, b.B)
    assert np.array_equal(out.cpu().numpy(), ref.astype(np.float32))


def test_backward_full_size_sharded1000_sampled_features():
    """BASELINE full size (sharded1000: 1000 features, B = 16384, 131 M lookups),
    dense gradients into 28.5 GB of fp32 targets, in the bench's default
    (untuned) launch configuration; integer data; a sample of features checked
    whole against the oracle."""
    m = synth.make_model('sharded1000')
    b = synth.make_batch(m, 7)
    _check(_run(m, b, 'int', seed=11), 'int')
    torch.cuda.empty_cache()
