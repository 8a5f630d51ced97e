"""L2 eviction priorities of row loads (reading C36, a B200 addition): the
cache-policy hints change where rows live in L2, never which rows are summed or
in what order -- outputs stay bit-exact under every policy; the policy is part
of the compiled kernel's signature and of the exported plan."""
import json
import os

import numpy as np
import pytest
import torch

from paper_conf_sc_panzzxwslr0d24_b200 import synth

from test_gpu_parity import Case, _mixed_model, bitexact, feature_columns, run_plan

pytestmark = pytest.mark.gpu


def _P():
    from paper_conf_sc_panzzxwslr0d24_b200 import plan
    return plan


@pytest.mark.parametrize('mapping', ['part0', 'part1'])
def test_every_policy_bitexact(mapping):
    P = _P()
    m = _mixed_model()
    b = synth.make_batch(m, 6)
    case = Case(m, b, 'int')
    ref, _ = case.oracle()
    plan = P.Plan.from_model(m, max_batch=b.B)
    for f in range(m.F):
        s = plan.get_schedule(f)
        plan.set_schedule(f, s['sched_id'], 1 if mapping == 'part1' else 0, 40 if mapping == 'part1' else 16)
    rng = np.random.default_rng(0)
    variants = None
    for pol in ([0] * m.F, [1] * m.F, [2] * m.F, [3] * m.F, rng.integers(0, 4, m.F).tolist()):
        plan.l2_policy = pol
        assert plan.l2_policy == pol
        info = plan.compile()
        assert info['active'] == 1
        if pol == [0] * m.F:
            variants = info['variants']
        _, out = run_plan(case, plan)
        assert bitexact(out, ref), pol
    # a mixed policy splits variants that share (entry, d, pool, pitch)
    assert info['variants'] >= variants


def test_lowp_rows_with_policies_bitexact():
    """Typed row loads (f16 / bf16 / i8 / fp8 words) take the same hints."""
    from test_gpu_lowp import TypedCase, _lowp_model
    for dtype in ('f16', 'bf16', 'i8', 'fp8'):
        m = _lowp_model(dtype)
        b = synth.make_batch(m, 4)
        case = TypedCase(m, b, dtype, 'int')
        plan = case.plan()
        plan.l2_policy = [1 + (f % 3) for f in range(m.F)]
        plan.compile()
        out = case.run(plan)
        ref, _ = case.oracle()
        assert bitexact(out, ref), dtype


def test_policy_export_import_invalid_and_heuristic():
    P = _P()
    m = synth.make_model('sharded1000')
    plan = P.Plan.from_model(m)
    h = plan.l2_policy_heuristic()
    assert set(h) <= {0, 1, 2} and len(h) == m.F
    assert 1 in h and 2 in h            # sharded1000 has both streaming and recurring tables
    plan.l2_policy = h
    st = plan.export()
    assert st['l2'] == h
    p2 = P.Plan.from_model(m)
    p2.import_(st)
    assert p2.l2_policy == h and p2.export() == st
    del st['l2']
    p2.import_(st)
    assert p2.l2_policy == [0] * m.F and 'l2' not in p2.export()
    with pytest.raises(RuntimeError):
        plan.l2_policy = [4] * m.F
    assert plan.l2_policy == h


def test_select_l2_policy_keeps_parity():
    P = _P()
    m = synth.make_model('fig3')
    b = synth.make_batch(m, 7)
    case = Case(m, b, 'int')
    plan = P.Plan.from_model(m)
    plan.compile()
    res = plan.select_l2_policy(case.idx, case.off, b.B, case.tables, reps=3)
    assert res['l2'] in plan.L2_CANDIDATES and all(v > 0 for v in res['ms'].values())
    _, out = run_plan(case, plan)
    ref, _ = case.oracle()
    assert bitexact(feature_columns(out, plan, m.dims), ref)
    plan.set_jit(False)
    with pytest.raises(RuntimeError):
        plan.select_l2_policy(case.idx, case.off, b.B, case.tables, reps=3)
