"""Generator tests (no GPU): determinism, CSR well-formedness, distribution
shape, and the table hash recomputed with Python ints."""
import os
import re

import numpy as np
import pytest
import torch

from paper_conf_sc_panzzxwslr0d24_b200 import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize('name', ['tiny', 'medium', 'fig3'])
def test_batch_deterministic_and_wellformed(name):
    m = synth.make_model(name)
    b1 = synth.make_batch(m, 7)
    b2 = synth.make_batch(m, 7)
    b3 = synth.make_batch(m, 8)
    assert np.array_equal(b1.indices, b2.indices) and np.array_equal(b1.offsets, b2.offsets)
    assert not np.array_equal(b1.offsets, b3.offsets)
    assert b1.offsets.dtype == np.int32 and b1.indices.dtype == np.int32
    assert b1.offsets[0] == 0 and np.all(np.diff(b1.offsets.astype(np.int64)) >= 0)
    assert b1.offsets.shape[0] == m.F * m.batch + 1
    for f, feat in enumerate(m.features):
        a, e = b1.offsets[f * b1.B], b1.offsets[(f + 1) * b1.B]
        ids = b1.indices[a:e]
        assert ids.size == 0 or (ids.min() >= 0 and ids.max() < feat.rows)
        L = b1.lengths()[f]
        assert L.max() <= feat.max_len()


def test_model_shapes_match_survey():
    assert synth.make_model('tiny').F == 4
    med = synth.make_model('medium')
    assert med.F == 50 and med.batch == 1024 and set(med.dims) == {16, 32, 64}
    ind = synth.make_model('industrial')
    assert ind.F == 300 and sum(f.kind == 'onehot' for f in ind.features) == 120
    hv = synth.make_model('heavy')
    assert hv.F == 100 and len(hv.tables) == 16 and hv.d_tot == 12800
    sh = synth.make_model('sharded1000')
    assert sh.F == 1000 and sh.batch == 16384 and sum(f.kind == 'onehot' for f in sh.features) == 500


def test_fig3_coverage_and_fixed_lengths():
    m = synth.make_model('fig3')
    b = synth.make_batch(m, 7, B=20000)
    L = b.lengths()
    cov = np.mean(L[0] > 0)
    assert abs(cov - 0.3) < 0.02
    assert abs(L[0][L[0] > 0].mean() - 50) < 1.0
    assert np.all(L[1] == 50)


def _mix32_py(x):
    M = 0xFFFFFFFF
    x ^= x >> 16
    x = (x * 0x7FEB352D) & M
    x ^= x >> 15
    x = (x * 0x6C8E9CF5) & M
    x ^= x >> 16
    return x


def test_table_hash_matches_python_ints():
    t, seed = 3, synth.MODEL_SEED
    rows = synth.table_rows(t, 100, 104, 6, 'float').numpy()
    irows = synth.table_rows(t, 100, 104, 6, 'int').numpy()
    M = 0xFFFFFFFF
    h0 = _mix32_py(((t * 0x27D4EB2F) + (seed * 0x165667B1)) & M)
    for i, r in enumerate(range(100, 104)):
        h1 = _mix32_py((h0 ^ r) & M)
        for c in range(6):
            h2 = _mix32_py((h1 + ((c * 0x61C88647) & M)) & M)
            assert rows[i, c] == np.float32((h2 >> 8) * 2.0 ** -23 - 1.0)
            assert irows[i, c] == (h2 >> 28) - 8


def test_table_chunking_invariant():
    a = synth.make_table(1, 1000, 16, chunk_rows=1000)
    b = synth.make_table(1, 1000, 16, chunk_rows=77)
    assert torch.equal(a, b)
    assert float(a.min()) >= -1.0 and float(a.max()) < 1.0


def test_algorithmic_bytes_formula():
    m = synth.make_model('tiny')
    b = synth.make_batch(m, 7)
    ab = synth.algorithmic_bytes(m, b)
    assert ab['index'] == 4 * b.nnz
    assert ab['rows'] == 4 * 16 * b.nnz
    assert ab['out'] == 4 * b.B * 64


def test_oracle_and_product_do_not_import_each_other():
    """the oracle shares no code with the CUDA path."""
    pkg = os.path.join(ROOT, 'paper_conf_sc_panzzxwslr0d24_b200')
    for dirpath, _, files in os.walk(pkg):
        for fn in files:
            if fn.endswith(('.py', '.cu', '.cuh', '.cpp', '.h')):
                src = open(os.path.join(dirpath, fn)).read()
                assert not re.search(r'^\s*(import|from)\s+oracle\b', src, re.M), fn
                assert 'liboracle' not in src, fn
    for fn in os.listdir(os.path.join(ROOT, 'oracle')):
        if fn.endswith(('.py', '.c', '.h')):
            src = open(os.path.join(ROOT, 'oracle', fn)).read()
            assert 'csrc' not in src and 'recflex.h' not in src, fn
            assert not re.search(r'paper_conf_sc_panzzxwslr0d24_b200\.(_lib|plan|shard)', src), fn


def test_models_from_recipes_match_golden():
    """configs/models/<name>.json recipes reproduce the models the tuned plans were made for."""
    import dataclasses
    import json
    import os
    g = json.load(open(os.path.join(os.path.dirname(__file__), 'golden', 'models_r02.json')))['models']
    for n in synth.CONFIG_NAMES:
        m = synth.make_model(n)
        assert m.batch == g[n]['batch'], n
        assert [list(t) for t in m.tables] == g[n]['tables'], n
        assert [list(dataclasses.astuple(f)) for f in m.features] == g[n]['features'], n


def test_recipe_variant_changes_model():
    """A recipe is data: changing it changes the model (no hidden hard-coded config)."""
    r = synth.load_recipe('medium')
    r['batch'] = 256
    r['dim'] = {'cycle': [8]}
    m = synth.make_model('medium', recipe=r)
    assert m.batch == 256 and set(m.dims) == {8} and m.F == 50
