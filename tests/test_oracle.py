"""Pins for the CPU oracle (no GPU).  Each test names what fixes the value
independently of the oracle's own code: the paper's definition worked by hand
(tests/golden), a library routine (torch embedding_bag in fp64), brute force
in Python loops, or a closed-form invariant."""
import json
import os

import numpy as np
import pytest
import torch

import oracle
from paper_conf_sc_panzzxwslr0d24_b200 import synth

GOLD = os.path.join(os.path.dirname(__file__), 'golden', 'worked_example.json')


def _gold():
    with open(GOLD) as fh:
        return json.load(fh)


# ---------------------------------------------------------------- worked examples (hand-computed)

@pytest.mark.parametrize('pool', [0, 1])
def test_worked_example_single_feature(pool):
    g = _gold()['single_feature']
    T = np.asarray(g['table'], np.float32)
    out = oracle.embedding_bag([T], [4], [pool], g['indices'], g['offsets'], g['B'])
    if pool == 0:
        exp = np.asarray(g['sum'], np.float64)
    else:
        exp = np.asarray(g['mean_num'], np.float64) / np.asarray(g['mean_den'], np.float64)
        exp[1] = 0.0  # empty bag -> 0 (reading C1)
    assert np.array_equal(out, exp)


def test_worked_example_two_features_concat():
    g = _gold()['two_features']
    tabs = [np.asarray(t, np.float32) for t in g['tables']]
    out = oracle.embedding_bag(tabs, g['dims'], g['pools'], g['indices'], g['offsets'], g['B'])
    exp = np.asarray(g['out_num'], np.float64) / np.asarray(g['out_den'], np.float64)
    assert np.array_equal(out, exp)


def test_worked_task_map_p338():
    g = _gold()['task_map_static_example']
    F = len(g['mode'])
    off = np.zeros(F * g['B'] + 1, np.int32)
    blocks, tf, tr = oracle.task_map(g['B'], g['mode'], g['per_block'], off)
    assert blocks.tolist() == g['blocks_map']
    assert tf.tolist() == g['task_feature']
    assert tr.tolist() == g['task_rel']


# ---------------------------------------------------------------- library routine: torch embedding_bag fp64

def _torch_ref(tables, dims, pools, indices, offsets, B):
    F = len(dims)
    outs = []
    for f in range(F):
        off = torch.as_tensor(offsets[f * B:(f + 1) * B + 1].astype(np.int64))
        base = int(off[0])
        idx = torch.as_tensor(indices[base:int(off[-1])].astype(np.int64))
        W = torch.as_tensor(np.asarray(tables[f], np.float64))
        mode = 'sum' if pools[f] == 0 else 'mean'
        outs.append(torch.nn.functional.embedding_bag(idx, W, off - base, mode=mode,
                                                      include_last_offset=True).numpy())
    return np.concatenate(outs, axis=1)


@pytest.mark.parametrize('name', ['tiny', 'fig3'])
def test_vs_torch_embedding_bag_configs(name):
    m = synth.make_model(name)
    b = synth.make_batch(m, 7, B=min(m.batch, 256))
    tabs_np = []
    for f in m.features:
        tabs_np.append(synth.make_table(f.table, min(f.rows, 5000), f.dim).numpy())
    # keep ids in range of the truncated tables
    idx = b.indices % np.int32(5000)   # keep ids inside the truncated tables
    pools = [f.pool for f in m.features]
    out = oracle.embedding_bag(tabs_np, m.dims, pools, idx, b.offsets, b.B)
    ref = _torch_ref(tabs_np, m.dims, pools, idx, b.offsets, b.B)
    np.testing.assert_allclose(out, ref, rtol=1e-12, atol=1e-12)


def test_vs_torch_embedding_bag_mixed_dims_pools():
    rng = np.random.default_rng(3)
    F, B = 7, 37
    dims = [4, 8, 12, 16, 3, 128, 1]
    pools = [0, 1, 0, 1, 1, 0, 1]
    rows = [11, 50, 7, 300, 5, 64, 9]
    lens = rng.integers(0, 9, size=(F, B))
    lens[2, :5] = 0
    b = synth.batch_from_lengths(lens, rows, seed=5)
    tabs = [rng.standard_normal((rows[f], dims[f])).astype(np.float32) for f in range(F)]
    out = oracle.embedding_bag(tabs, dims, pools, b.indices, b.offsets, B)
    ref = _torch_ref(tabs, dims, pools, b.indices, b.offsets, B)
    np.testing.assert_allclose(out, ref, rtol=1e-12, atol=1e-12)


# ---------------------------------------------------------------- brute force (pure Python loops)

def test_brute_force_tiny():
    rng = np.random.default_rng(11)
    F, B = 3, 5
    dims = [2, 3, 4]
    pools = [1, 0, 1]
    rows = [4, 6, 3]
    tabs = [rng.integers(-5, 6, size=(rows[f], dims[f])).astype(np.float32) for f in range(F)]
    lens = rng.integers(0, 4, size=(F, B))
    b = synth.batch_from_lengths(lens, rows, seed=2)
    out = oracle.embedding_bag(tabs, dims, pools, b.indices, b.offsets, B)
    D = sum(dims)
    exp = [[0.0] * D for _ in range(B)]
    col = 0
    for f in range(F):
        for s in range(B):
            a, e = int(b.offsets[f * B + s]), int(b.offsets[f * B + s + 1])
            for c in range(dims[f]):
                acc = 0.0
                for j in range(a, e):
                    acc += float(tabs[f][int(b.indices[j])][c])
                if pools[f] == 1:
                    acc = acc / (e - a) if e > a else 0.0
                exp[s][col + c] = acc
        col += dims[f]
    assert np.array_equal(out, np.asarray(exp))


# ---------------------------------------------------------------- closed-form invariants

def _rand_case(seed=0, F=4, B=20, maxlen=6, dims=(4, 8, 16, 5), rows=(10, 20, 30, 7)):
    rng = np.random.default_rng(seed)
    lens = rng.integers(0, maxlen + 1, size=(F, B))
    b = synth.batch_from_lengths(lens, list(rows), seed=seed + 1)
    tabs = [rng.uniform(-1, 1, size=(rows[f], dims[f])).astype(np.float32) for f in range(F)]
    return b, tabs, list(dims)


def test_one_hot_is_row_copy():
    b, tabs, dims = _rand_case(maxlen=1)
    lens = b.lengths()
    out = oracle.embedding_bag(tabs, dims, [0] * 4, b.indices, b.offsets, b.B)
    col = np.cumsum([0] + dims)
    for f in range(4):
        for s in range(b.B):
            a = int(b.offsets[f * b.B + s])
            piece = out[s, col[f]:col[f + 1]]
            if lens[f, s] == 1:
                assert np.array_equal(piece, tabs[f][b.indices[a]].astype(np.float64))
            else:
                assert np.all(piece == 0.0)


def test_empty_bags_zero_both_pools():
    F, B = 2, 6
    lens = np.zeros((F, B), np.int64)
    b = synth.batch_from_lengths(lens, [3, 3])
    tabs = [np.ones((3, 4), np.float32)] * 2
    for pool in (0, 1):
        out = oracle.embedding_bag(tabs, [4, 4], [pool, pool], b.indices, b.offsets, B)
        assert np.all(out == 0.0) and not np.any(np.isnan(out))


def test_mean_is_sum_over_len():
    b, tabs, dims = _rand_case(seed=4)
    s = oracle.embedding_bag(tabs, dims, [0] * 4, b.indices, b.offsets, b.B)
    m = oracle.embedding_bag(tabs, dims, [1] * 4, b.indices, b.offsets, b.B)
    lens = b.lengths()
    col = np.cumsum([0] + dims)
    for f in range(4):
        L = lens[f][:, None].astype(np.float64)
        exp = np.where(L > 0, s[:, col[f]:col[f + 1]] / np.maximum(L, 1), 0.0)
        assert np.array_equal(m[:, col[f]:col[f + 1]], exp)


def test_linearity_scaling_by_two_exact():
    b, tabs, dims = _rand_case(seed=5)
    o1 = oracle.embedding_bag(tabs, dims, [0, 1, 0, 1], b.indices, b.offsets, b.B)
    o2 = oracle.embedding_bag([2 * t for t in tabs], dims, [0, 1, 0, 1], b.indices, b.offsets, b.B)
    assert np.array_equal(o2, 2 * o1)


def test_permutation_within_bag_invariant_integer_tables():
    rng = np.random.default_rng(6)
    b, tabs, dims = _rand_case(seed=6, maxlen=9)
    tabs = [np.round(t * 8).astype(np.float32) for t in tabs]   # integer values -> exact fp64 sums
    o1 = oracle.embedding_bag(tabs, dims, [0, 1, 0, 1], b.indices, b.offsets, b.B)
    idx2 = b.indices.copy()
    for k in range(b.F * b.B):
        a, e = int(b.offsets[k]), int(b.offsets[k + 1])
        idx2[a:e] = rng.permutation(idx2[a:e])
    o2 = oracle.embedding_bag(tabs, dims, [0, 1, 0, 1], idx2, b.offsets, b.B)
    assert np.array_equal(o1, o2)


def test_batch_split_invariance():
    b, tabs, dims = _rand_case(seed=7, B=24)
    full = oracle.embedding_bag(tabs, dims, [0, 1, 1, 0], b.indices, b.offsets, b.B)
    # split samples [0,10) and [10,24): rebuild each half's KJT from the full one
    for lo, hi in ((0, 10), (10, 24)):
        Bh = hi - lo
        idx, off = [], [0]
        for f in range(b.F):
            for s in range(lo, hi):
                a, e = int(b.offsets[f * b.B + s]), int(b.offsets[f * b.B + s + 1])
                idx.extend(b.indices[a:e].tolist())
                off.append(off[-1] + e - a)
        part = oracle.embedding_bag(tabs, dims, [0, 1, 1, 0], np.asarray(idx, np.int32),
                                    np.asarray(off, np.int32), Bh)
        assert np.array_equal(part, full[lo:hi])


def test_integer_mode_tables_give_exact_integers():
    m = synth.make_model('tiny')
    b = synth.make_batch(m, 7)
    tabs = [synth.make_table(f.table, f.rows, f.dim, mode='int').numpy() for f in m.features]
    assert all(t.min() >= -8 and t.max() <= 7 for t in tabs)
    out = oracle.embedding_bag(tabs, m.dims, [0] * 4, b.indices, b.offsets, b.B)
    assert np.array_equal(out, np.round(out))


def test_duplicate_ids_counted_with_multiplicity():
    T = np.arange(12, dtype=np.float32).reshape(3, 4)
    out = oracle.embedding_bag([T], [4], [0], [1, 1, 1], [0, 3], 1)
    assert np.array_equal(out[0], 3 * T[1].astype(np.float64))


def test_out_of_range_index_rejected():
    T = np.zeros((3, 4), np.float32)
    with pytest.raises(oracle.OracleError):
        oracle.embedding_bag([T], [4], [0], [3], [0, 1], 1)
    with pytest.raises(oracle.OracleError):
        oracle.embedding_bag([T], [4], [0], [0, 1], [0, 2, 1], 2)


def test_thread_count_does_not_change_result():
    b, tabs, dims = _rand_case(seed=8, B=64)
    o1 = oracle.embedding_bag(tabs, dims, [0, 1, 0, 1], b.indices, b.offsets, b.B, nthreads=1)
    o4 = oracle.embedding_bag(tabs, dims, [0, 1, 0, 1], b.indices, b.offsets, b.B, nthreads=4)
    assert np.array_equal(o1, o4)


# ---------------------------------------------------------------- task map (Fig. 8) pins

def _brute_task_map(B, mode, pb, off, cap, slots, static):
    F = len(mode)
    tasks = []
    blocks = []
    for f in range(F):
        if mode[f] == 0:
            n = -(-B // pb[f])
        else:
            nnz = int(off[(f + 1) * B]) - int(off[f * B])
            npb = pb[f]
            if slots[f] > 0:
                npb = max(npb, -(-nnz // (slots[f] - 2)))
            n = nnz // npb + 1
        if static[f] > 0:  # static mapping: fixed allocated block count
            n = static[f]
        if cap[f] > 0:
            n = min(n, cap[f])
        blocks.append(n)
        tasks += [(f, r) for r in range(n)]
    return blocks, tasks


@pytest.mark.parametrize('seed', range(5))
def test_task_map_vs_brute_force(seed):
    rng = np.random.default_rng(seed)
    F, B = int(rng.integers(1, 9)), int(rng.integers(1, 70))
    lens = rng.integers(0, 30, size=(F, B))
    b = synth.batch_from_lengths(lens, [100] * F, seed=seed)
    mode = rng.integers(0, 2, size=F).tolist()
    pb = [int(rng.integers(1, 40)) for _ in range(F)]
    cap = [int(rng.integers(0, 4)) if rng.random() < 0.3 else 0 for _ in range(F)]
    slots = [int(rng.integers(3, 12)) if rng.random() < 0.5 else 0 for _ in range(F)]
    static = [int(rng.integers(1, 6)) if rng.random() < 0.3 else 0 for _ in range(F)]
    blocks, tf, tr = oracle.task_map(B, mode, pb, b.offsets, cap, slots, static)
    eb, et = _brute_task_map(B, mode, pb, b.offsets, cap, slots, static)
    assert blocks.tolist() == eb
    assert list(zip(tf.tolist(), tr.tolist())) == et
    bs = oracle.block_start_from_task_map(F, tf)
    assert bs[-1] == sum(eb) and np.all(np.diff(bs) == np.asarray(eb))


def test_worked_static_mapping_p338():
    """P:338 golden: 2 allocated blocks, 3 needed -> allocated block 0 performs needed
    blocks 0 and 2 one after another, block 1 performs needed block 1."""
    g = _gold()['task_map_p338_static']
    off = np.zeros(g['B'] + 1, np.int32)
    blocks, tf, tr, need, _ = oracle.task_map(g['B'], [0], [g['per_block']], off, static_blocks=[g['static_blocks']],
                                              full=True)
    assert need.tolist() == [g['need']] and blocks.tolist() == [g['blocks_map']]
    assert tr.tolist() == list(range(g['blocks_map']))
    alloc, seq = oracle.static_assignment(g['need'], g['static_blocks'])
    assert alloc.tolist() == g['alloc_of'] and seq.tolist() == g['seq_of']
    # the sample ranges each allocated block walks, in order
    got = [[] for _ in range(g['blocks_map'])]
    for q in sorted(range(g['need']), key=lambda q: (alloc[q], seq[q])):
        got[alloc[q]].append([q * g['per_block'], min(g['B'], (q + 1) * g['per_block'])])
    assert got == g['samples_of_allocated']


def test_static_assignment_invariants():
    for need in range(0, 20):
        for nalloc in range(1, 8):
            a, q = oracle.static_assignment(need, nalloc)
            pairs = sorted(zip(a.tolist(), q.tolist()))
            assert len(set(pairs)) == need                      # each needed block exactly once
            for blk in range(nalloc):                            # each allocated block: steps 0, 1, 2, ...
                steps = sorted(s for x, s in pairs if x == blk)
                assert steps == list(range(len(steps)))
            if need:
                loads = np.bincount(a, minlength=nalloc)
                assert loads.max() - loads.min() <= 1             # balanced round robin
                assert loads.max() == -(-need // nalloc)


def test_worked_nnz_partitioned_task_map():
    """Hand-worked lookup-partitioned map incl. the npb raise for short task slots (C12)."""
    g = _gold()['task_map_nnz_partitioned']
    off = np.asarray(g['offsets'], np.int32)
    for c in g['cases']:
        blocks, tf, tr, need, npb = oracle.task_map(g['B'], [1], [c['per_block']], off, slots=[c['slots']], full=True)
        assert npb.tolist() == [c['npb_eff']] and need.tolist() == [c['need']] and blocks.tolist() == [c['need']]
        s0, s1 = oracle.nnz_task_ranges(g['B'], c['npb_eff'], off, c['need'])
        assert [[a, b] for a, b in zip(s0.tolist(), s1.tolist())] == c['ranges']


def test_nnz_task_ranges_partition():
    rng = np.random.default_rng(9)
    for trial in range(20):
        B = int(rng.integers(1, 50))
        lens = rng.integers(0, 40, size=B)
        lens[rng.random(B) < 0.2] = 0
        off = np.zeros(B + 1, np.int32)
        off[1:] = np.cumsum(lens) + 5
        off[0] = 5
        npb = int(rng.integers(1, 60))
        nnz = int(off[-1] - off[0])
        blocks = nnz // npb + 1
        s0, s1 = oracle.nnz_task_ranges(B, npb, off, blocks)
        # ranges are ordered, contiguous, cover [0, B) exactly once
        assert s0[0] == 0 and s1[-1] == B
        assert np.all(s1 >= s0)
        assert np.all(s0[1:] == s1[:-1])
        for s in range(B):
            q = (int(off[s]) - int(off[0])) // npb
            assert s0[q] <= s < s1[q]


# ---------------------------------------------------------------- reduced-precision storage (NEXT #3)

LOWP = os.path.join(os.path.dirname(__file__), 'golden', 'lowp_rows.json')


def _lowp():
    with open(LOWP) as fh:
        return json.load(fh)


def _i8_row(codes, scale, bias):
    d = len(codes)
    row = np.zeros(oracle.row_bytes('i8', d), np.uint8)
    row[:d] = np.asarray(codes, np.int8).view(np.uint8)
    row[d:d + 8] = np.asarray([scale, bias], np.float32).view(np.uint8)
    return row


def test_decode_f16_worked_values():
    g = _lowp()['f16']
    v = oracle.decode_rows(np.asarray(g['bits'], np.uint16).reshape(-1, 1), 1, 'f16')
    assert v[:, 0].tolist() == g['values']


def test_decode_bf16_worked_values():
    g = _lowp()['bf16']
    v = oracle.decode_rows(np.asarray(g['bits'], np.uint16).reshape(-1, 1), 1, 'bf16')
    assert v[:, 0].tolist() == g['values']


def test_decode_f16_exhaustive_vs_numpy():
    """All 2^16 binary16 patterns against numpy's float16 -> float64 (library routine)."""
    bits = np.arange(1 << 16, dtype=np.uint32).astype(np.uint16)
    v = oracle.decode_rows(bits.reshape(-1, 4), 4, 'f16').reshape(-1)
    ref = bits.view(np.float16).astype(np.float64)
    assert np.array_equal(np.isnan(v), np.isnan(ref))
    ok = ~np.isnan(ref)
    assert np.array_equal(v[ok], ref[ok])
    assert np.array_equal(np.signbit(v[ok]), np.signbit(ref[ok]))  # -0.0 stays -0.0


def test_decode_bf16_exhaustive_vs_torch():
    """All 2^16 bfloat16 patterns against torch's bfloat16 -> float64 (library routine)."""
    bits = torch.arange(1 << 16, dtype=torch.int32).to(torch.int16)
    v = oracle.decode_rows(bits.numpy().view(np.uint16).reshape(-1, 4), 4, 'bf16').reshape(-1)
    ref = bits.view(torch.bfloat16).double().numpy()
    assert np.array_equal(np.isnan(v), np.isnan(ref))
    ok = ~np.isnan(ref)
    assert np.array_equal(v[ok], ref[ok])


def test_decode_fp8_worked_values():
    g = _lowp()['fp8']
    v = oracle.decode_rows(np.asarray(g['bits'], np.uint8).reshape(-1, 1), 1, 'fp8')[:, 0]
    assert v.tolist() == g['values']
    assert np.signbit(v[-1])  # 0x80 = -0.0
    nan = oracle.decode_rows(np.asarray(g['nan_bits'], np.uint8).reshape(-1, 1), 1, 'fp8')[:, 0]
    assert np.all(np.isnan(nan))


def test_decode_fp8_exhaustive_vs_torch():
    """All 256 FP8 E4M3 codes against torch's float8_e4m3fn -> float64 (library routine)."""
    bits = torch.arange(256, dtype=torch.int32).to(torch.uint8)
    v = oracle.decode_rows(bits.numpy().reshape(-1, 8), 8, 'fp8').reshape(-1)
    ref = bits.view(torch.float8_e4m3fn).double().numpy()
    assert np.array_equal(np.isnan(v), np.isnan(ref))
    ok = ~np.isnan(ref)
    assert np.array_equal(v[ok], ref[ok])
    assert np.array_equal(np.signbit(v[ok]), np.signbit(ref[ok]))


def test_fp8_tables_equal_upcast_f32_tables():
    """An FP8 stored table pools exactly like its library up-cast to float32."""
    m = synth.make_model('tiny')
    b = synth.make_batch(m, 7)
    rng = np.random.default_rng(2)
    codes = [rng.integers(0, 256, (f.rows, f.dim)).astype(np.uint8) for f in m.features]
    codes = [np.where((c & 0x7F) == 0x7F, 0x38, c).astype(np.uint8) for c in codes]   # no NaN codes
    up = [torch.from_numpy(c).view(torch.float8_e4m3fn).float().numpy() for c in codes]
    pools = [0, 1, 0, 1]
    got = oracle.embedding_bag(codes, m.dims, pools, b.indices, b.offsets, b.B, dtypes=['fp8'] * m.F)
    exp = oracle.embedding_bag(up, m.dims, pools, b.indices, b.offsets, b.B)
    assert np.array_equal(got, exp)


def test_decode_i8_worked_row():
    g = _lowp()['i8']
    row = _i8_row(g['codes'], g['scale'], g['bias'])
    v = oracle.decode_rows(row.reshape(1, -1), g['dim'], 'i8')
    assert v[0].tolist() == g['values']


@pytest.mark.parametrize('pool', [0, 1])
def test_i8_bag_worked_example(pool):
    g = _lowp()
    r0 = _i8_row(g['i8']['codes'], g['i8']['scale'], g['i8']['bias'])
    r1 = _i8_row(g['i8_bag']['codes_r1'], g['i8_bag']['scale_r1'], g['i8_bag']['bias_r1'])
    T = np.stack([r0, r1])
    out = oracle.embedding_bag([T], [8], [pool], g['i8_bag']['indices'], g['i8_bag']['offsets'], 2, dtypes=['i8'])
    exp0 = np.asarray(g['i8_bag']['sum_s0'], np.float64)
    if pool == 1:
        exp0 = exp0 / 3.0
    assert np.array_equal(out[0], exp0)
    assert np.array_equal(out[1], np.zeros(8))  # empty bag -> 0 (reading C1)


@pytest.mark.parametrize('dtype', ['f16', 'bf16'])
def test_half_tables_equal_upcast_f32_tables(dtype):
    """A 16-bit stored table pools exactly like its library up-cast to float32
    (every 16-bit value is exactly representable in float32)."""
    m = synth.make_model('tiny')
    b = synth.make_batch(m, 7)
    st = [synth.table_rows_stored(f.table, np.arange(m.tables[f.table][0]), f.dim, dtype, 'float', seed=m.seed)
          for f in m.features]
    up = [t.float().numpy() for t in st]
    pools = [1, 0, 1, 0]
    a = oracle.embedding_bag(st, m.dims, pools, b.indices, b.offsets, b.B, dtypes=[dtype] * m.F)
    r = oracle.embedding_bag(up, m.dims, pools, b.indices, b.offsets, b.B)
    assert np.array_equal(a, r)


def test_i8_tables_vs_torch_weighted_embedding_bag():
    """Rowwise int8 pooling = torch embedding_bag of the codes with per-lookup
    weights scale[id], plus embedding_bag of the bias column (library routine,
    fp64), since sum_j (s_j q_j + b_j) = sum_j s_j q_j + sum_j b_j."""
    m = synth.make_model('tiny')
    b = synth.make_batch(m, 8)
    F, B = m.F, b.B
    st = [synth.table_rows_stored(f.table, np.arange(m.tables[f.table][0]), f.dim, 'i8', 'float', seed=m.seed)
          for f in m.features]
    out = oracle.embedding_bag(st, m.dims, [0] * F, b.indices, b.offsets, B, dtypes=['i8'] * F)
    col = 0
    for f in range(F):
        d = m.dims[f]
        raw = st[f].numpy()
        q = torch.from_numpy(raw[:, :d].view(np.int8).astype(np.float64))
        sb = raw[:, d:d + 8].copy().view(np.float32).astype(np.float64)
        lo, hi = b.offsets[f * B], b.offsets[(f + 1) * B]
        ids = torch.from_numpy(b.indices[lo:hi].astype(np.int64))
        offs = torch.from_numpy((b.offsets[f * B:(f + 1) * B + 1] - lo).astype(np.int64))
        w = torch.from_numpy(sb[:, 0])[ids]
        ref = torch.nn.functional.embedding_bag(ids, q, offs, mode='sum', per_sample_weights=w,
                                                include_last_offset=True)
        ref += torch.nn.functional.embedding_bag(ids, torch.from_numpy(sb[:, 1:2]), offs, mode='sum',
                                                 include_last_offset=True)
        assert np.allclose(out[:, col:col + d], ref.numpy(), rtol=1e-13, atol=1e-12)
        col += d


def test_i8_int_mode_exact_integers():
    m = synth.make_model('tiny')
    b = synth.make_batch(m, 7)
    st = [synth.table_rows_stored(f.table, np.arange(m.tables[f.table][0]), f.dim, 'i8', 'int', seed=m.seed)
          for f in m.features]
    out = oracle.embedding_bag(st, m.dims, [0] * m.F, b.indices, b.offsets, b.B, dtypes=['i8'] * m.F)
    assert np.array_equal(out, np.rint(out))


# ---------------------------------------------------------------- backward / adjoint (NEXT #4)

@pytest.mark.parametrize('pool', [0, 1])
def test_backward_worked_example(pool):
    g = _gold()['backward']
    tg, cn, _ = oracle.embedding_bag_backward([g['rows']], [g['dim']], [pool], g['indices'], g['offsets'], g['B'],
                                              np.asarray(g['grad'], np.float64))
    if pool == 0:
        exp = np.asarray(g['sum'], np.float64)
    else:
        exp = np.asarray(g['mean_num'], np.float64) / g['mean_den']
    assert np.allclose(tg[0], exp, rtol=0, atol=1e-15)
    assert cn[0].tolist() == g['counts']


@pytest.mark.parametrize('name', ['tiny', 'fig3'])
def test_backward_vs_torch_autograd(name):
    """Library routine: torch autograd of embedding_bag (fp64) gives the same table gradients."""
    m = synth.make_model(name)
    b = synth.make_batch(m, 7)
    F, B = m.F, b.B
    pools = [f % 2 for f in range(F)]
    rng = np.random.default_rng(3)
    G = rng.standard_normal((B, m.d_tot))
    tg, _, _ = oracle.embedding_bag_backward([f.rows for f in m.features], m.dims, pools, b.indices, b.offsets, B, G)
    col = 0
    for f in range(F):
        d = m.dims[f]
        W = torch.zeros((m.features[f].rows, d), dtype=torch.float64, requires_grad=True)
        lo, hi = b.offsets[f * B], b.offsets[(f + 1) * B]
        ids = torch.from_numpy(b.indices[lo:hi].astype(np.int64))
        offs = torch.from_numpy((b.offsets[f * B:(f + 1) * B + 1] - lo).astype(np.int64))
        out = torch.nn.functional.embedding_bag(ids, W, offs, mode=('sum', 'mean')[pools[f]],
                                                include_last_offset=True)
        out.backward(torch.from_numpy(G[:, col:col + d]))
        assert np.allclose(tg[f], W.grad.numpy(), rtol=1e-12, atol=1e-12)
        col += d


def test_backward_adjoint_identity():
    """<G, A(T)> == <A^T(G), T> for the linear map A = embedding bag (fixed indices)."""
    m = synth.make_model('tiny')
    b = synth.make_batch(m, 9)
    pools = [0, 1, 1, 0]
    rng = np.random.default_rng(5)
    T = [rng.standard_normal((f.rows, f.dim)).astype(np.float32) for f in m.features]
    G = rng.standard_normal((b.B, m.d_tot))
    fwd = oracle.embedding_bag(T, m.dims, pools, b.indices, b.offsets, b.B)
    tg, _, _ = oracle.embedding_bag_backward([f.rows for f in m.features], m.dims, pools, b.indices, b.offsets, b.B, G)
    lhs = float(np.sum(G * fwd))
    rhs = float(sum(np.sum(tg[f] * T[f].astype(np.float64)) for f in range(m.F)))
    assert abs(lhs - rhs) <= 1e-10 * max(1.0, abs(lhs))


def test_backward_scale_and_initial_targets():
    """SGD form: targets start at T0 and receive scale * gradient (exact for scale = -0.5)."""
    m = synth.make_model('tiny')
    b = synth.make_batch(m, 7)
    rows = [f.rows for f in m.features]
    rng = np.random.default_rng(1)
    G = rng.integers(-8, 8, (b.B, m.d_tot)).astype(np.float64)
    T0 = [rng.integers(-8, 8, (f.rows, f.dim)).astype(np.float64) for f in m.features]
    g1, cn, ab = oracle.embedding_bag_backward(rows, m.dims, [0] * m.F, b.indices, b.offsets, b.B, G)
    g2, _, _ = oracle.embedding_bag_backward(rows, m.dims, [0] * m.F, b.indices, b.offsets, b.B, G, scale=-0.5,
                                             targets=T0)
    for f in range(m.F):
        assert np.array_equal(g2[f], T0[f] - 0.5 * g1[f])
        assert np.all(ab[f] >= np.abs(g1[f]))
        nnz = b.offsets[(f + 1) * b.B] - b.offsets[f * b.B]
        assert cn[f].sum() == nnz


# ---- table-wise input distribution -------------------

KJTD = os.path.join(os.path.dirname(__file__), 'golden', 'kjt_input_dist.json')


def test_kjt_input_dist_golden():
    """Hand-worked 2-rank example (tests/golden/kjt_input_dist.json)."""
    g = json.load(open(KJTD))
    locs = [(np.asarray(k['indices'], np.int32), np.asarray(k['offsets'], np.int32)) for k in g['local_kjts']]
    # the golden local KJTs are the hand-written bags, laid out feature-major
    for j, kjt in enumerate(locs):
        bags = g['local_bags'][f'rank{j}']
        flat = [bag for f in range(3) for bag in bags[f'f{f}']]
        assert kjt[0].tolist() == [i for bag in flat for i in bag]
        assert np.diff(kjt[1]).tolist() == [len(bag) for bag in flat]
    got = oracle.kjt_input_dist(locs, g['parts'], g['local_batch'])
    for r, exp in enumerate(g['expected']):
        assert got[r][0].tolist() == exp['indices']
        assert got[r][1].tolist() == exp['offsets']


def _sample_split(idx, off, F, B, W):
    """Global KJT -> W data-parallel local KJTs (rank j: samples [j*B/W, (j+1)*B/W))."""
    Bl = B // W
    out = []
    for j in range(W):
        lens = np.diff(off.astype(np.int64)).reshape(F, B)[:, j * Bl:(j + 1) * Bl]
        ids = np.concatenate([idx[off[f * B + j * Bl]:off[f * B + (j + 1) * Bl]] for f in range(F)])
        o = np.concatenate([[0], np.cumsum(lens.reshape(-1))]).astype(np.int32)
        out.append((ids.astype(np.int32), o))
    return out


@pytest.mark.parametrize('W', [1, 2, 4])
def test_kjt_input_dist_equals_feature_restriction(W):
    """Splitting a global KJT by samples and redistributing it by features gives
    exactly the global KJT restricted to each rank's features (the operation's
    defining property; both sides written here with plain slicing)."""
    m = synth.make_model('tiny')
    b = synth.make_batch(m, 11)
    F, B = m.F, b.B
    rng = np.random.default_rng(W)
    owner = rng.integers(0, W, F)
    parts = [[f for f in range(F) if owner[f] == r] for r in range(W)]
    got = oracle.kjt_input_dist(_sample_split(b.indices, b.offsets, F, B, W), parts, B // W)
    for r in range(W):
        ids = [b.indices[b.offsets[f * B]:b.offsets[(f + 1) * B]] for f in parts[r]]
        lens = [np.diff(b.offsets[f * B:(f + 1) * B + 1]) for f in parts[r]]
        exp_idx = np.concatenate(ids) if ids else np.zeros(0, np.int32)
        exp_off = np.concatenate([[0], np.cumsum(np.concatenate(lens))]) if lens else np.zeros(1)
        assert np.array_equal(got[r][0], exp_idx)
        assert np.array_equal(got[r][1], exp_off)
    # invariants: every ID arrives exactly once, W = 1 with all features is the identity
    assert sum(g[0].size for g in got) == b.indices.size
    if W == 1:
        assert np.array_equal(got[0][0], b.indices) and np.array_equal(got[0][1], b.offsets)
