"""Task order (reading C35, a B200 addition): the order in which the features'
tasks are laid out in the task map -- and claimed by the persistent CTAs --
must not change any output bit, in either kernel, for any mapping; the task map
under an order is the oracle's per-feature task counts scanned in that order;
the order travels with the exported plan; the backward scatters into the right
tables under a permuted order.  (The full-size check of a plan with task-order columns is
the tuned sharded1000 plan in test_gpu_parity / test_gpu_tuned_plans, which bench.py times.)"""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_sc_panzzxwslr0d24_b200 import synth

from test_gpu_parity import Case, _mixed_model, bitexact, feature_columns, run_plan

pytestmark = pytest.mark.gpu


def _P():
    from paper_conf_sc_panzzxwslr0d24_b200 import plan
    return plan


def _orders(plan, F, seed=0):
    rng = np.random.default_rng(seed)
    out = {k: plan.task_order_heuristic(k) for k in plan.ORDER_KINDS}
    out['random'] = rng.permutation(F).tolist()
    out['reversed'] = list(range(F))[::-1]
    return out


def _to_feature_columns(out, plan, dims):
    """Reassemble an output laid out by plan.columns into feature-order concatenation."""
    cols = plan.columns
    return np.concatenate([out[:, c:c + d] for c, d in zip(cols, dims)], axis=1)


def _aligned(plan, order, dims):
    """Would every vector-store schedule keep a 16-byte aligned column with the
    outputs concatenated in this task order?"""
    cat = _P().catalog()
    col, c = {}, 0
    for f in order:
        col[f] = c
        c += dims[f]
    return all(cat[plan.get_schedule(f)['sched_id']]['VEC'] == 1 or col[f] % 4 == 0 for f in range(len(dims)))


@pytest.mark.parametrize('columns', ['feature', 'task-order'])
@pytest.mark.parametrize('kernel', ['catalog', 'plan-specialised'])
@pytest.mark.parametrize('mapping', ['part0', 'part1', 'mixed'])
def test_every_order_bitexact(kernel, mapping, columns):
    P = _P()
    m = _mixed_model()
    b = synth.make_batch(m, 5)
    case = Case(m, b, 'int')
    ref, _ = case.oracle()
    plan = P.Plan.from_model(m, max_batch=b.B)
    rng = np.random.default_rng(1)
    for f in range(m.F):
        s = plan.get_schedule(f)
        part = {'part0': 0, 'part1': 1, 'mixed': int(rng.integers(0, 2))}[mapping]
        plan.set_schedule(f, s['sched_id'], part, int(rng.choice([3, 16, 64])) if part == 0 else 40)
    if kernel == 'plan-specialised':
        assert plan.compile()['active'] == 1
    else:
        plan.set_jit(False)
    if columns == 'task-order':
        plan.set_column_order(True)
    ran = 0
    for name, order in _orders(plan, m.F).items():
        if columns == 'task-order' and not _aligned(plan, order, m.dims):
            with pytest.raises(RuntimeError):
                plan.task_order = order
            continue
        plan.task_order = order
        assert plan.task_order == list(order)
        if columns == 'task-order':
            exp, c = [], 0
            for f in order:
                exp.append(c)
                c += m.dims[f]
            assert plan.columns == [exp[list(order).index(f)] for f in range(m.F)]
        _, out = run_plan(case, plan)
        assert bitexact(_to_feature_columns(out, plan, m.dims), ref), name
        ran += 1
    assert ran >= 2
    plan.task_order = None
    assert plan.task_order == list(range(m.F))
    assert plan.columns == np.cumsum([0] + m.dims)[:-1].tolist()


def test_heuristics_are_permutations_and_sorted():
    P = _P()
    m = synth.make_model('industrial')
    plan = P.Plan.from_model(m)
    st = plan.export()
    est = []
    for f, feat in enumerate(m.features):
        sid, part, pb = st['schedules'][f][:3]
        rb = 4 * feat.dim
        est.append(pb * rb if part == 1 else pb * max(0.05, feat.mean_len() * feat.coverage) * rb)
    est = np.array(est)
    for kind in plan.ORDER_KINDS:
        o = plan.task_order_heuristic(kind)
        assert sorted(o) == list(range(m.F))
        e = est[o]
        if kind == 'lpt':
            assert np.all(np.diff(e) <= 1e-6 * e[:-1])
        elif kind == 'spt':
            assert np.all(np.diff(e) >= -1e-6 * e[1:])
        else:
            assert o == list(range(m.F))


def test_task_map_under_order_vs_oracle():
    P = _P()
    m = _mixed_model()
    b = synth.make_batch(m, 12)
    plan = P.Plan.from_model(m, max_batch=b.B)
    rng = np.random.default_rng(4)
    mode, pb, slots = [], [], []
    for f in range(m.F):
        s = plan.get_schedule(f)
        part = int(rng.integers(0, 2))
        per = int(rng.choice([2, 64, 700])) if part else int(rng.integers(1, 300))
        plan.set_schedule(f, s['sched_id'], part, per)
        mode.append(part)
        pb.append(per)
        slots.append(plan.task_slots(f))
    order = rng.permutation(m.F).tolist()
    plan.task_order = order
    off = torch.from_numpy(b.offsets).cuda()
    bs, ranges = plan.debug_task_map(off, b.B, ranges=True)
    blocks, tf, tr, need, npb = oracle.task_map(b.B, mode, pb, b.offsets, slots=slots, full=True)
    exp = np.concatenate([[0], np.cumsum(np.asarray(blocks)[order])]).tolist()
    assert bs == exp
    assert plan.debug_task_need() == need.tolist()   # reported in feature order
    for e, f in enumerate(order):
        if mode[f] != 1:
            continue
        s0, s1 = oracle.nnz_task_ranges(b.B, int(npb[f]), b.offsets[f * b.B:(f + 1) * b.B + 1], int(blocks[f]))
        got = ranges[bs[e]:bs[e + 1]]
        assert [g[0] for g in got] == s0.tolist()
        assert [g[1] for g in got] == s1.tolist()


def test_order_export_import_and_invalid():
    P = _P()
    m = _mixed_model()
    plan = P.Plan.from_model(m, max_batch=64)
    order = np.random.default_rng(2).permutation(m.F).tolist()
    plan.task_order = order
    st = plan.export()
    assert st['order'] == order
    p2 = P.Plan.from_model(m, max_batch=64)
    p2.import_(st)
    assert p2.task_order == order and p2.export() == st
    del st['order']
    p2.import_(st)                      # a plan without "order" runs in feature order
    assert p2.task_order == list(range(m.F))
    # column layout in task order travels with the plan
    m4 = synth.make_model('medium')     # dims multiples of 4: every order keeps columns aligned
    p3 = P.Plan.from_model(m4)
    o4 = p3.task_order_heuristic('lpt')
    p3.set_column_order(True)
    p3.task_order = o4
    st4 = p3.export()
    assert st4['columns'] == 'task-order' and st4['order'] == o4
    p4 = P.Plan.from_model(m4)
    p4.import_(st4)
    assert p4.columns == p3.columns and p4.export() == st4
    assert p4.columns != np.cumsum([0] + m4.dims)[:-1].tolist()
    for bad in ([0] * m.F, list(range(m.F - 1)) + [m.F], list(range(1, m.F)) + [-1]):
        with pytest.raises(RuntimeError):
            plan.task_order = bad
    assert plan.task_order == order     # unchanged by the rejected calls


def test_select_task_order_keeps_parity():
    P = _P()
    m = synth.make_model('medium')
    b = synth.make_batch(m, 7)
    case = Case(m, b, 'int')
    plan = P.Plan.from_model(m)
    res = plan.select_task_order(case.idx, case.off, b.B, case.tables, reps=3)
    assert res['order'] in plan.ORDER_KINDS
    assert all(v > 0 for v in res['ms'].values())
    assert plan.task_order == plan.task_order_heuristic(res['order'])
    samples = np.arange(0, b.B, 7)
    out = plan.forward(case.idx, case.off, b.B, case.tables).cpu().numpy()[samples]
    ref, _ = case.oracle(samples)
    assert bitexact(out, ref)


@pytest.mark.parametrize('mode', ['int', 'float'])
def test_backward_under_order(mode):
    from test_gpu_backward import _check, _run
    P = _P()
    m = _mixed_model()
    b = synth.make_batch(m, 9)
    plan = P.Plan.from_model(m, max_batch=b.B)
    plan.task_order = np.random.default_rng(3).permutation(m.F).tolist()
    _check(_run(m, b, mode, plan=plan), mode)


@pytest.mark.parametrize('order', ['feature', 'lpt'])
def test_select_task_size_keeps_parity(order):
    """recflex_select_task_size (reading C37): the kept scale is applied to every
    feature's per-task size, a heuristic order is re-derived, outputs stay bit-exact."""
    P = _P()
    m = synth.make_model('fig3')
    b = synth.make_batch(m, 7)
    case = Case(m, b, 'int')
    plan = P.Plan.from_model(m)
    plan.task_order = plan.task_order_heuristic(order)
    before = [plan.get_schedule(f)['per_block'] for f in range(m.F)]
    parts = [plan.get_schedule(f)['part'] for f in range(m.F)]
    res = plan.select_task_size(case.idx, case.off, b.B, case.tables, reps=3)
    assert res['task_size'] in plan.TASK_SIZES and all(v > 0 for v in res['ms'].values())
    num, den = {'x1': (1, 1), 'x1/2': (1, 2), 'x2': (2, 1)}[res['task_size']]
    after = [plan.get_schedule(f)['per_block'] for f in range(m.F)]
    assert after == [max(16 if parts[f] else 1, before[f] * num // den) for f in range(m.F)]
    assert plan.task_order == plan.task_order_heuristic(order)
    _, out = run_plan(case, plan)
    ref, _ = case.oracle()
    assert bitexact(feature_columns(out, plan, m.dims), ref)


def test_order_change_under_captured_graph():
    """A CUDA graph captured before recflex_set_task_order replays consistently after it:
    the device descriptors and the compiled kernel's variant ids change together (the
    descriptors are uploaded by the setter, not deferred to the next eager forward)."""
    P = _P()
    m = _mixed_model()
    b = synth.make_batch(m, 8)
    case = Case(m, b, 'int')
    ref, _ = case.oracle()
    plan = P.Plan.from_model(m, max_batch=b.B)
    plan.compile()
    out = torch.empty((b.B, m.d_tot), device='cuda')
    plan.forward(case.idx, case.off, b.B, case.tables, out=out)   # uploads descriptors before capture
    torch.cuda.synchronize()
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        plan.forward(case.idx, case.off, b.B, case.tables, out=out, stream=s)
    torch.cuda.current_stream().wait_stream(s)
    for order in (np.random.default_rng(5).permutation(m.F).tolist(), list(range(m.F))[::-1], None):
        plan.task_order = order
        out.zero_()
        g.replay()
        torch.cuda.synchronize()
        assert bitexact(out.cpu().numpy(), ref), order
