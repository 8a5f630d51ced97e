"""CPU oracle for the RecFlex hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product path never imports it and shares no code with it.

The arithmetic lives in ``oracle.c`` (plain C, fp64 accumulation); this file
only builds it with gcc, marshals numpy arrays through ctypes and, for the
full-size sampled checks, extracts the bags to check into a compact sub-batch
(pure input selection -- the pooled values are still computed by the C code).

Functions and the passages they follow (PAPER.md "P:n"):
  embedding_bag  -- P:41, P:51 (§II-A): gather the rows named by each sample's
                    lookup IDs, pool them by elementwise reduction, concatenate
                    per-feature outputs.  Readings C1, C2, C6.
  decode_rows    -- the value of a stored row element per storage type (SURVEY
                    NEXT #3: f16 / bf16 / rowwise int8); embedding_bag takes
                    stored tables and decodes every element with it.
  embedding_bag_backward -- the adjoint (training):
                    dense gradient / SGD update of every table row.
  task_map       -- Fig. 8: d_blocks_map and d_task_map, reading C12
                    (incl. the npb raise for reserved task slots).
  static_assignment -- P:338 static thread mapping: which allocated block runs
                    which needed block, in which order (reading C31).
  nnz_task_ranges-- reading C12 for nnz-partitioned schedules.
  kjt_input_dist -- table-wise input distribution (P:350
                    "place different embedding tables on multiple GPUs"):
                    the data-parallel KJTs of W ranks regrouped so that every
                    rank holds all B samples of the features it owns.  Pure
                    integer data movement, written in numpy (no C needed).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, 'oracle.c')
_LIB = os.path.join(_HERE, 'liboracle.so')
_lock = threading.Lock()
_lib = None

POOL_SUM = 0
POOL_MEAN = 1


def build(force: bool = False) -> str:
    """Compile oracle.c -> liboracle.so (gcc -O2 -fopenmp, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f'.tmp{os.getpid()}'
        subprocess.check_call(['gcc', '-O2', '-fopenmp', '-fPIC', '-shared', '-std=c11', '-Wall',
                               '-o', tmp, _SRC, '-lm'])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_LIB)
            P = ctypes.POINTER
            L.oracle_embedding_bag.restype = ctypes.c_int
            L.oracle_embedding_bag.argtypes = [
                ctypes.c_int, ctypes.c_int, P(ctypes.c_int), P(ctypes.c_int),
                P(ctypes.c_void_p), P(ctypes.c_int64), P(ctypes.c_int32), P(ctypes.c_int32),
                P(ctypes.c_double), ctypes.c_int]
            L.oracle_embedding_bag_typed.restype = ctypes.c_int
            L.oracle_embedding_bag_typed.argtypes = [
                ctypes.c_int, ctypes.c_int, P(ctypes.c_int), P(ctypes.c_int), P(ctypes.c_int),
                P(ctypes.c_void_p), P(ctypes.c_int64), P(ctypes.c_int32), P(ctypes.c_int32),
                P(ctypes.c_double), ctypes.c_int]
            L.oracle_decode_rows.restype = ctypes.c_int
            L.oracle_decode_rows.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int,
                                             P(ctypes.c_double)]
            L.oracle_row_bytes.restype = ctypes.c_int64
            L.oracle_row_bytes.argtypes = [ctypes.c_int, ctypes.c_int]
            L.oracle_embedding_bag_backward.restype = ctypes.c_int
            L.oracle_embedding_bag_backward.argtypes = [
                ctypes.c_int, ctypes.c_int, P(ctypes.c_int), P(ctypes.c_int), P(ctypes.c_int64),
                P(ctypes.c_int32), P(ctypes.c_int32), P(ctypes.c_double), ctypes.c_double,
                P(ctypes.c_void_p), P(ctypes.c_void_p), P(ctypes.c_void_p)]
            L.oracle_task_map.restype = ctypes.c_int
            L.oracle_task_map.argtypes = [
                ctypes.c_int, ctypes.c_int, P(ctypes.c_int), P(ctypes.c_int), P(ctypes.c_int), P(ctypes.c_int),
                P(ctypes.c_int), P(ctypes.c_int32), P(ctypes.c_int), P(ctypes.c_int), P(ctypes.c_int),
                P(ctypes.c_int), P(ctypes.c_int), ctypes.c_int64, P(ctypes.c_int64)]
            L.oracle_static_assignment.restype = ctypes.c_int
            L.oracle_static_assignment.argtypes = [ctypes.c_int, ctypes.c_int, P(ctypes.c_int), P(ctypes.c_int)]
            L.oracle_nnz_task_ranges.restype = ctypes.c_int
            L.oracle_nnz_task_ranges.argtypes = [
                ctypes.c_int, ctypes.c_int, P(ctypes.c_int32), ctypes.c_int, P(ctypes.c_int), P(ctypes.c_int)]
            L.oracle_max_threads.restype = ctypes.c_int
            _lib = L
    return _lib


def _ptr(a, ct):
    return a.ctypes.data_as(ctypes.POINTER(ct))


class OracleError(RuntimeError):
    pass


def max_threads() -> int:
    return int(lib().oracle_max_threads())


DTYPES = {'f32': 0, 'f16': 1, 'bf16': 2, 'i8': 3, 'fp8': 4}


def row_bytes(dtype, dim: int) -> int:
    return int(lib().oracle_row_bytes(DTYPES.get(dtype, dtype), int(dim)))


def _stored(t, dtype, dim):
    """A stored table (numpy array or CPU torch tensor) as contiguous raw bytes [rows][row_bytes]."""
    code = DTYPES.get(dtype, dtype)
    if code == 0:
        a = np.ascontiguousarray(t.numpy() if hasattr(t, 'numpy') else t, dtype=np.float32)
        if a.ndim != 2 or a.shape[1] != dim:
            raise ValueError(f'table shape {a.shape} vs dim {dim}')
        return a
    if hasattr(t, 'view') and hasattr(t, 'dtype') and not isinstance(t, np.ndarray):  # torch (bf16 has no numpy)
        import torch
        t = t.contiguous().view(torch.uint8).numpy()
    a = np.ascontiguousarray(t).view(np.uint8)
    a = a.reshape(a.shape[0], -1)
    if a.shape[1] != row_bytes(code, dim):
        raise ValueError(f'stored row bytes {a.shape[1]} vs {row_bytes(code, dim)} for dim {dim} dtype {dtype}')
    return a


def decode_rows(rows, dim: int, dtype) -> np.ndarray:
    """fp64 values of stored rows (oracle_decode), [n][dim]."""
    a = _stored(rows, dtype, dim)
    out = np.zeros((a.shape[0], dim), np.float64)
    rc = lib().oracle_decode_rows(DTYPES.get(dtype, dtype), a.ctypes.data, a.shape[0], int(dim),
                                  _ptr(out, ctypes.c_double))
    if rc != 0:
        raise OracleError(rc)
    return out


def embedding_bag(tables, dims, pools, indices, offsets, B, nthreads: int = 0, dtypes=None) -> np.ndarray:
    """fp64 pooled output [B][sum(dims)].

    tables: list of F stored tables (one per feature; aliasing allowed):
    float32 arrays [rows_f][d_f] when dtypes is None, else per dtypes[f]
    ('f32', 'f16', 'bf16', 'i8' -- numpy arrays or CPU torch tensors; an i8
    row is d int8 codes, float32 scale, float32 bias, zero padding to 16 bytes).
    """
    F = len(dims)
    dts = [DTYPES.get(d, d) for d in (dtypes if dtypes is not None else [0] * F)]
    tabs = [_stored(t, dts[f], dims[f]) for f, t in enumerate(tables)]
    dims_a = np.asarray(dims, np.intc)
    pools_a = np.asarray(pools, np.intc)
    rows_a = np.asarray([t.shape[0] for t in tabs], np.int64)
    ptrs = (ctypes.c_void_p * F)(*[t.ctypes.data for t in tabs])
    idx = np.ascontiguousarray(indices, np.int32)
    off = np.ascontiguousarray(offsets, np.int32)
    if off.shape[0] != F * B + 1:
        raise ValueError('offsets must have F*B+1 entries')
    out = np.zeros((B, int(dims_a.sum())), np.float64)
    if idx.size == 0:
        idx = np.zeros(1, np.int32)
    dt_a = np.asarray(dts, np.intc)
    rc = lib().oracle_embedding_bag_typed(F, B, _ptr(dims_a, ctypes.c_int), _ptr(pools_a, ctypes.c_int),
                                          _ptr(dt_a, ctypes.c_int), ptrs, _ptr(rows_a, ctypes.c_int64),
                                          _ptr(idx, ctypes.c_int32), _ptr(off, ctypes.c_int32),
                                          _ptr(out, ctypes.c_double), int(nthreads))
    if rc != 0:
        raise OracleError({-1: 'index out of range', -2: 'bad offsets', -3: 'bad argument'}.get(rc, rc))
    return out


def embedding_bag_backward(rows, dims, pools, indices, offsets, B, grad, scale=1.0, targets=None):
    """Adjoint of embedding_bag: fp64 per-feature updates.

    rows: per-feature row counts; grad: [B][sum(dims)] (cast to fp64);
    targets: optional list of F initial arrays [rows_f][d_f] (copied to fp64;
    default zeros).  Returns (targets, counts, abssum): the updated targets,
    the number of terms per row and the per-element sum of |term|.
    """
    F = len(dims)
    dims_a = np.asarray(dims, np.intc)
    pools_a = np.asarray(pools, np.intc)
    rows_a = np.asarray(rows, np.int64)
    g = np.ascontiguousarray(grad, np.float64)
    if g.shape != (B, int(dims_a.sum())):
        raise ValueError(f'grad shape {g.shape}')
    tg = [np.array(targets[f], np.float64, copy=True).reshape(int(rows_a[f]), dims[f]) if targets is not None
          else np.zeros((int(rows_a[f]), dims[f]), np.float64) for f in range(F)]
    cn = [np.zeros(int(rows_a[f]), np.int64) for f in range(F)]
    ab = [np.zeros((int(rows_a[f]), dims[f]), np.float64) for f in range(F)]
    idx = np.ascontiguousarray(indices, np.int32)
    off = np.ascontiguousarray(offsets, np.int32)
    if off.shape[0] != F * B + 1:
        raise ValueError('offsets must have F*B+1 entries')
    if idx.size == 0:
        idx = np.zeros(1, np.int32)
    P = ctypes.c_void_p
    rc = lib().oracle_embedding_bag_backward(
        F, B, _ptr(dims_a, ctypes.c_int), _ptr(pools_a, ctypes.c_int), _ptr(rows_a, ctypes.c_int64),
        _ptr(idx, ctypes.c_int32), _ptr(off, ctypes.c_int32), _ptr(g, ctypes.c_double), float(scale),
        (P * F)(*[t.ctypes.data for t in tg]), (P * F)(*[c.ctypes.data for c in cn]),
        (P * F)(*[a.ctypes.data for a in ab]))
    if rc != 0:
        raise OracleError({-1: 'index out of range', -2: 'bad offsets', -3: 'bad argument'}.get(rc, rc))
    return tg, cn, ab


def task_map(B, mode, per_block, offsets, cap=None, slots=None, static_blocks=None, full=False):
    """Fig. 8 arrays: (blocks_map[F], task_feature[T], task_rel[T]); with full=True also
    need_map[F] (blocks the batch needs) and npb_map[F] (effective lookups per block)."""
    F = len(mode)
    mode_a = np.asarray(mode, np.intc)
    pb = np.asarray(per_block, np.intc)
    z = [0] * F
    cap_a = np.asarray(cap if cap is not None else z, np.intc)
    slots_a = np.asarray(slots if slots is not None else z, np.intc)
    st_a = np.asarray(static_blocks if static_blocks is not None else z, np.intc)
    off = np.ascontiguousarray(offsets, np.int32)
    # upper bound on tasks for the output buffers
    ub = 0
    for f in range(F):
        if st_a[f] > 0:
            ub += int(st_a[f])
        elif mode[f] == 0:
            ub += (B + pb[f] - 1) // pb[f]
        else:
            ub += (int(off[(f + 1) * B]) - int(off[f * B])) // max(1, int(pb[f])) + 1
    ub = max(ub, 1)
    blocks = np.zeros(F, np.intc)
    need = np.zeros(F, np.intc)
    npb = np.zeros(F, np.intc)
    tf = np.zeros(ub, np.intc)
    tr = np.zeros(ub, np.intc)
    n = ctypes.c_int64(0)
    rc = lib().oracle_task_map(F, B, _ptr(mode_a, ctypes.c_int), _ptr(pb, ctypes.c_int),
                               _ptr(slots_a, ctypes.c_int), _ptr(st_a, ctypes.c_int),
                               _ptr(cap_a, ctypes.c_int), _ptr(off, ctypes.c_int32),
                               _ptr(need, ctypes.c_int), _ptr(npb, ctypes.c_int),
                               _ptr(blocks, ctypes.c_int), _ptr(tf, ctypes.c_int), _ptr(tr, ctypes.c_int),
                               ub, ctypes.byref(n))
    if rc != 0:
        raise OracleError(rc)
    if full:
        return blocks, tf[:n.value].copy(), tr[:n.value].copy(), need, npb
    return blocks, tf[:n.value].copy(), tr[:n.value].copy()


def static_assignment(need: int, nalloc: int):
    """P:338 static mapping: (alloc_of[need], seq_of[need]) -- the allocated block that
    performs needed block q, and at which sequential step."""
    a = np.zeros(max(1, need), np.intc)
    q = np.zeros(max(1, need), np.intc)
    rc = lib().oracle_static_assignment(int(need), int(nalloc), _ptr(a, ctypes.c_int), _ptr(q, ctypes.c_int))
    if rc != 0:
        raise OracleError(rc)
    return a[:need].copy(), q[:need].copy()


def block_start_from_task_map(F, task_feature):
    """Exclusive-scan view of d_task_map: first task index of every feature, plus total."""
    counts = np.bincount(np.asarray(task_feature, np.int64), minlength=F)[:F]
    bs = np.zeros(F + 1, np.int64)
    np.cumsum(counts, out=bs[1:])
    return bs


def nnz_task_ranges(B, npb, feature_offsets, blocks):
    off = np.ascontiguousarray(feature_offsets, np.int32)
    s0 = np.zeros(max(blocks, 1), np.intc)
    s1 = np.zeros(max(blocks, 1), np.intc)
    rc = lib().oracle_nnz_task_ranges(int(B), int(npb), _ptr(off, ctypes.c_int32), int(blocks),
                                      _ptr(s0, ctypes.c_int), _ptr(s1, ctypes.c_int))
    if rc != 0:
        raise OracleError(rc)
    return s0[:blocks].copy(), s1[:blocks].copy()


def kjt_input_dist(local_kjts, parts, local_batch):
    """Table-wise input distribution, the plain definition.

    local_kjts[j] = (indices, offsets) of rank j: a feature-major KJT over ALL F
    features and rank j's Bl = local_batch samples (global samples
    j*Bl .. (j+1)*Bl-1), offsets[F*Bl+1].  parts[r] = the features rank r owns.
    Returns, for every rank r, (indices, offsets) of the KJT over r's features
    (in the order given by parts[r]) and all B = W*Bl global samples in global
    order: bag (k, s) of the result = bag (parts[r][k], s mod Bl) of rank
    s // Bl.  Bags keep their IDs in order.
    """
    W, Bl = len(local_kjts), int(local_batch)
    out = []
    for r in range(len(parts)):
        ids, lens = [], []
        for f in parts[r]:
            for j in range(W):                       # global sample order = (source rank, local sample)
                idx_j = np.asarray(local_kjts[j][0])
                off_j = np.asarray(local_kjts[j][1], np.int64)
                for s in range(Bl):
                    a, b = off_j[f * Bl + s], off_j[f * Bl + s + 1]
                    if b < a:
                        raise OracleError('bad offsets')
                    ids.append(idx_j[a:b])
                    lens.append(b - a)
        off = np.zeros(len(lens) + 1, np.int64)
        np.cumsum(np.asarray(lens, np.int64), out=off[1:])
        out.append((np.concatenate(ids).astype(np.int32) if ids else np.zeros(0, np.int32), off.astype(np.int32)))
    return out


# ---------------------------------------------------------------------------
# Full-size sampled checks: compute selected samples one by one.
# ---------------------------------------------------------------------------

def sampled_forward(model, batch, samples, table_getter, dtype='f32'):
    """Oracle output rows for the given sample ids of a (possibly huge) batch.

    table_getter(feature_index, unique_row_ids) -> stored rows [n] of that
    feature's table in `dtype` (from the seeded generator).  Returns fp64
    [len(samples)][D_tot] and the per-(sample, feature) bag lengths [len(samples)][F].
    """
    F, B = batch.F, batch.B
    samples = np.asarray(samples, np.int64)
    S = samples.size
    offs = batch.offsets.astype(np.int64)
    sub_off = [0]
    sub_idx = []
    tables = []
    lens = np.zeros((S, F), np.int64)
    for f in range(F):
        bags = []
        for k, s in enumerate(samples):
            a, b = offs[f * B + s], offs[f * B + s + 1]
            bags.append(batch.indices[a:b])
            lens[k, f] = b - a
        allids = np.concatenate(bags) if bags else np.zeros(0, np.int32)
        uniq, inv = np.unique(allids, return_inverse=True)
        if uniq.size == 0:
            uniq = np.zeros(1, np.int64)
        rows_f = table_getter(f, uniq)
        if DTYPES.get(dtype, dtype) == 0:
            rows_f = np.asarray(rows_f, np.float32).reshape(uniq.size, model.features[f].dim)
        tables.append(rows_f)
        pos = 0
        for bag in bags:
            sub_idx.append(inv[pos:pos + bag.size].astype(np.int32))
            pos += bag.size
            sub_off.append(sub_off[-1] + bag.size)
    idx = np.concatenate(sub_idx) if sub_idx else np.zeros(0, np.int32)
    off = np.asarray(sub_off, np.int32)
    out = embedding_bag(tables, model.dims, [f.pool for f in model.features], idx, off, S,
                        dtypes=[dtype] * F)
    return out, lens
