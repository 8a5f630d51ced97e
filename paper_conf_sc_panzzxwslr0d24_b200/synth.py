"""Seeded synthetic inputs shared by the CUDA path's tests/bench and the oracle.

This module holds NONE of the method's arithmetic (no gather, no pooling, no
thread mapping).  It only draws the inputs the paper says its data-synthesis
script draws: per-feature pooling factors from a stated distribution, lookup
IDs uniform over each table, and table contents (PAPER.md P:260, P:505 --
"indices with specified pooling factor distribution and embedding table
shape"; coverage as in Fig. 3).

Readings:
  C9  coverage c = P(L > 0); L = 0 w.p. 1-c, else a draw from the length model,
      rounded half-to-even (numpy ``rint``) and clipped to [1, Lmax].
  C10 lookup IDs i.i.d. uniform over [0, rows_f) with replacement.
  C11 table contents are a counter-based hash of (table, row, column):
        'float' mode -> U[-1, 1) on a 2^-23 grid (exactly representable in fp32)
        'int'   mode -> integers in [-8, 7] (every fp32 partial sum is exact)
      The hash uses only int64 ops whose products stay < 2^63, so torch on CPU
      and torch on CUDA produce identical bits; any row can be regenerated on
      the host for sampled oracle checks without copying it from the device.
  C25 heavy: 100 fields whose 10M-row index ranges alias 16 physical tables.

Layout produced (KJT feature-major CSR):
  indices int32[nnz], offsets int32[F*B + 1]; bag (f, s) is
  indices[offsets[f*B+s] : offsets[f*B+s+1]].
"""
from __future__ import annotations

import dataclasses
import json
import math
import os
from typing import List, Optional

import numpy as np

POOL_SUM = 0
POOL_MEAN = 1

MODEL_SEED = 1234
M32 = 0xFFFFFFFF


@dataclasses.dataclass
class Feature:
    rows: int                 # index range of the field (== rows of its physical table)
    dim: int
    pool: int                 # POOL_SUM / POOL_MEAN
    kind: str                 # 'onehot' | 'normal' | 'lognormal' | 'uniform' | 'fixed'
    coverage: float = 1.0
    mu: float = 1.0           # mean of the length model (normal / lognormal) or fixed L
    sigma: float = 0.0        # normal: std; lognormal: sigma of log
    lo: int = 0               # uniform model: L ~ U{lo..hi}
    hi: int = 0
    lmax: int = 1
    table: int = 0            # physical table id (aliasing, C25)

    # hotness stats an operator would pass to recflex_plan_create (from history)
    def mean_len(self) -> float:
        if self.kind == 'onehot':
            return 1.0
        if self.kind == 'uniform':
            # E[L | L > 0] for U{lo..hi}
            vals = [v for v in range(self.lo, self.hi + 1) if v > 0]
            return float(sum(vals)) / max(1, len(vals))
        if self.kind == 'fixed':
            return float(self.mu)
        return float(min(self.mu, self.lmax))

    def max_len(self) -> float:
        if self.kind == 'onehot':
            return 1.0
        if self.kind == 'uniform':
            return float(self.hi)
        if self.kind == 'fixed':
            return float(self.mu)
        return float(self.lmax)


@dataclasses.dataclass
class Model:
    name: str
    features: List[Feature]
    tables: List[tuple]       # (rows, dim) per physical table
    batch: int
    seed: int = MODEL_SEED

    @property
    def F(self) -> int:
        return len(self.features)

    @property
    def dims(self) -> List[int]:
        return [f.dim for f in self.features]

    @property
    def d_tot(self) -> int:
        return sum(self.dims)


# ---------------------------------------------------------------------------
# Model definitions (SURVEY §8d generator table; BASELINE.json "configs")
# ---------------------------------------------------------------------------

def _log_uniform(rng, lo, hi, size=None):
    return np.exp(rng.uniform(math.log(lo), math.log(hi), size=size))


MODEL_DIR = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), 'configs', 'models')


def _draw(rng, spec):
    """A scalar from a recipe spec: {"fixed": v} | {"uniform": [a, b]} | {"log_uniform": [a, b]}."""
    if 'fixed' in spec:
        return spec['fixed']
    if 'uniform' in spec:
        return float(rng.uniform(*spec['uniform']))
    if 'log_uniform' in spec:
        return float(_log_uniform(rng, *spec['log_uniform']))
    raise ValueError(f'bad spec {spec}')


def load_recipe(name: str) -> dict:
    path = os.path.join(MODEL_DIR, f'{name}.json')
    if not os.path.exists(path):
        raise ValueError(f'unknown model {name!r} (no {path})')
    with open(path) as fh:
        return json.load(fh)


def make_model(name: str, seed: int = MODEL_SEED, recipe: Optional[dict] = None) -> Model:
    """The synthetic model of a BASELINE config from its recipe configs/models/<name>.json
    (SURVEY §8d).  Draws, per field in order: the dim (if chosen at random), the rows (if
    log-uniform), then the coverage (one-hot) or the mean length and the coverage
    (multi-hot); the one-hot set is a random permutation prefix drawn first when the
    recipe says so.  tests/golden/models_r02.json pins the result."""
    r = recipe if recipe is not None else load_recipe(name)
    rng = np.random.Generator(np.random.PCG64([seed, _name_key(name)]))
    feats: List[Feature] = []
    if 'explicit' in r:
        feats = [Feature(**f) for f in r['explicit']]
        B = int(r['batch'])
    else:
        F = int(r['fields'])
        oh = r['onehot']
        if oh['rule'] == 'random':
            onehot = set(rng.permutation(F)[:oh['count']].tolist())
        elif oh['rule'] == 'even':
            onehot = set(range(0, F, 2))
        elif oh['rule'] == 'first':
            onehot = set(range(oh['count']))
        else:
            onehot = set()
        mh = r.get('multihot', {})
        for f in range(F):
            ds = r['dim']
            if 'choice' in ds:
                dim = int(rng.choice(ds['choice'], p=ds['p']))
            elif 'cycle' in ds:
                dim = int(ds['cycle'][f % len(ds['cycle'])])
            else:
                dim = int(ds['fixed'])
            rows = int(_draw(rng, r['rows']))
            pool = {'sum': POOL_SUM, 'mean': POOL_MEAN}.get(r['pool'])
            if pool is None:  # even_sum_odd_mean
                pool = POOL_SUM if f % 2 == 0 else POOL_MEAN
            tspec = r.get('tables', 'per_field')
            table = f % int(tspec['alias_mod']) if isinstance(tspec, dict) else f
            if f in onehot:
                feats.append(Feature(rows=rows, dim=dim, pool=pool, kind='onehot',
                                     coverage=float(_draw(rng, r['onehot_coverage'])), lmax=1, table=table))
            elif mh['kind'] == 'uniform':
                feats.append(Feature(rows=rows, dim=dim, pool=pool, kind='uniform', lo=int(mh['lo']), hi=int(mh['hi']),
                                     lmax=int(mh['hi']), table=table))
            else:
                mu = _draw(rng, mh['mu'])
                sigma = mu * mh['sigma_over_mu'] if 'sigma_over_mu' in mh else float(mh['sigma'])
                cov = float(_draw(rng, mh['coverage']))
                if 'lmax_over_mu' in mh:
                    lmax = int(round(mh['lmax_over_mu'] * mu))
                    if 'lmax_min' in mh:
                        lmax = max(int(mh['lmax_min']), lmax)
                else:
                    lmax = int(mh['lmax'])
                feats.append(Feature(rows=rows, dim=dim, pool=pool, kind=mh['kind'], mu=mu, sigma=sigma, coverage=cov,
                                     lmax=lmax, table=table))
        B = int(r['batch'])
    ntab = max(f.table for f in feats) + 1
    tables = [None] * ntab
    for f in feats:
        tables[f.table] = (f.rows, f.dim)
    return Model(name=name, features=feats, tables=tables, batch=B, seed=seed)


def custom_model(name: str, features: List[Feature], batch: int) -> Model:
    ntab = max(f.table for f in features) + 1
    tables = [None] * ntab
    for f in features:
        if tables[f.table] is not None and tables[f.table] != (f.rows, f.dim):
            raise ValueError('aliased features must share table shape')
        tables[f.table] = (f.rows, f.dim)
    return Model(name=name, features=features, tables=tables, batch=batch)


CONFIG_NAMES = ('tiny', 'medium', 'industrial', 'heavy', 'sharded1000', 'fig3')


def _name_key(name: str) -> int:
    return sum((i + 1) * ord(ch) for i, ch in enumerate(name))


# ---------------------------------------------------------------------------
# Batches: pooling factors and lookup IDs
# ---------------------------------------------------------------------------

def _lengths(rng, feat: Feature, B: int) -> np.ndarray:
    present = rng.random(B) < feat.coverage
    if feat.kind == 'onehot':
        L = np.ones(B, np.int64)
    elif feat.kind == 'fixed':
        L = np.full(B, int(feat.mu), np.int64)
    elif feat.kind == 'uniform':
        L = rng.integers(feat.lo, feat.hi + 1, size=B).astype(np.int64)
        return L  # U{lo..hi} already includes empty bags (tiny config)
    elif feat.kind == 'normal':
        L = np.clip(np.rint(rng.normal(feat.mu, feat.sigma, size=B)), 1, feat.lmax).astype(np.int64)
    elif feat.kind == 'lognormal':
        m = math.log(feat.mu) - 0.5 * feat.sigma ** 2
        L = np.clip(np.rint(np.exp(rng.normal(m, feat.sigma, size=B))), 1, feat.lmax).astype(np.int64)
    else:
        raise ValueError(feat.kind)
    return np.where(present, L, 0)


@dataclasses.dataclass
class Batch:
    indices: np.ndarray   # int32 [nnz]
    offsets: np.ndarray   # int32 [F*B + 1]
    B: int
    F: int

    @property
    def nnz(self) -> int:
        return int(self.offsets[-1])

    def lengths(self) -> np.ndarray:
        return np.diff(self.offsets.astype(np.int64)).reshape(self.F, self.B)


def make_batch(model: Model, batch_seed: int = 7, B: Optional[int] = None) -> Batch:
    """One synthetic batch (seed 7+i for the i-th batch)."""
    B = model.batch if B is None else int(B)
    rng = np.random.Generator(np.random.PCG64([model.seed, _name_key(model.name), batch_seed]))
    F = model.F
    lens = np.empty((F, B), np.int64)
    for f, feat in enumerate(model.features):
        lens[f] = _lengths(rng, feat, B)
    offsets = np.zeros(F * B + 1, np.int64)
    np.cumsum(lens.reshape(-1), out=offsets[1:])
    nnz = int(offsets[-1])
    if nnz >= 2 ** 31:
        raise ValueError('nnz exceeds int32 (reading C4)')
    indices = np.empty(nnz, np.int32)
    for f, feat in enumerate(model.features):
        a, b = int(offsets[f * B]), int(offsets[(f + 1) * B])
        if b > a:
            indices[a:b] = rng.integers(0, feat.rows, size=b - a, dtype=np.int64).astype(np.int32)
    return Batch(indices=indices, offsets=offsets.astype(np.int32), B=B, F=F)


def batch_from_lengths(lengths: np.ndarray, rows: List[int], seed: int = 0) -> Batch:
    """Hand-shaped batch: lengths[F][B] given, IDs uniform (for edge-case tests)."""
    lengths = np.asarray(lengths, np.int64)
    F, B = lengths.shape
    rng = np.random.Generator(np.random.PCG64(seed))
    offsets = np.zeros(F * B + 1, np.int64)
    np.cumsum(lengths.reshape(-1), out=offsets[1:])
    indices = np.empty(int(offsets[-1]), np.int32)
    for f in range(F):
        a, b = int(offsets[f * B]), int(offsets[(f + 1) * B])
        indices[a:b] = rng.integers(0, rows[f], size=b - a).astype(np.int32)
    return Batch(indices=indices, offsets=offsets.astype(np.int32), B=B, F=F)


# ---------------------------------------------------------------------------
# Table contents: counter-based hash (identical on CPU and CUDA)
# ---------------------------------------------------------------------------

_K1 = 0x7FEB352D
_K2 = 0x6C8E9CF5


def _mix32(x):
    """32-bit avalanche on a non-negative int64 tensor holding values < 2^32."""
    x = x ^ (x >> 16)
    x = (x * _K1) & M32
    x = x ^ (x >> 15)
    x = (x * _K2) & M32
    x = x ^ (x >> 16)
    return x


def table_rows(table_id: int, row_start: int, row_end: int, dim: int, mode: str = 'float',
               device='cpu', seed: int = MODEL_SEED):
    """Rows [row_start, row_end) of physical table ``table_id`` as a float32 torch tensor."""
    import torch
    return table_rows_at(table_id, torch.arange(row_start, row_end, dtype=torch.int64, device=device), dim, mode,
                         device, seed)


def table_rows_at(table_id: int, row_ids, dim: int, mode: str = 'float', device='cpu',
                  seed: int = MODEL_SEED):
    """Selected rows (any order, repeats allowed) of a physical table -- the same
    values make_table produces at those rows."""
    import torch
    r = torch.as_tensor(row_ids, dtype=torch.int64, device=device).reshape(-1)
    h0 = _mix32(torch.tensor(((table_id * 0x27D4EB2F) + (seed * 0x165667B1)) & M32, dtype=torch.int64,
                             device=device))
    h1 = _mix32((h0 ^ (r & M32)) & M32)
    c = torch.arange(dim, dtype=torch.int64, device=device)
    ck = (c * 0x61C88647) & M32
    h2 = _mix32((h1[:, None] + ck[None, :]) & M32)
    if mode == 'float':
        out = (h2 >> 8).to(torch.float64) * (2.0 ** -23) - 1.0
    elif mode == 'int':
        out = ((h2 >> 28) - 8).to(torch.float64)
    else:
        raise ValueError(mode)
    return out.to(torch.float32)


def make_table(table_id: int, rows: int, dim: int, mode: str = 'float', device='cpu',
               seed: int = MODEL_SEED, chunk_rows: Optional[int] = None):
    import torch
    out = torch.empty((rows, dim), dtype=torch.float32, device=device)
    if chunk_rows is None:
        chunk_rows = max(1, (1 << 25) // max(1, dim))
    for a in range(0, rows, chunk_rows):
        b = min(rows, a + chunk_rows)
        out[a:b] = table_rows(table_id, a, b, dim, mode, device, seed)
    return out


# ---------------------------------------------------------------------------
# Reduced-precision storage: the same seeded tables, stored
# as float16 / bfloat16 (round-to-nearest casts of the fp32 values) or as
# rowwise int8 (codes + per-row fp32 scale and bias, include/recflex.h).
# Encoding inputs only: the value of a stored element is defined (and
# computed for checking) by oracle_decode, not here.
# ---------------------------------------------------------------------------
STORAGE_DTYPES = ('f32', 'f16', 'bf16', 'i8', 'fp8')


def i8_row_bytes(dim: int) -> int:
    return (dim + 8 + 15) // 16 * 16


def table_rows_stored(table_id: int, row_ids, dim: int, dtype: str = 'f32', mode: str = 'float', device='cpu',
                      seed: int = MODEL_SEED):
    """Stored rows of a physical table: float32 / float16 / bfloat16 [n, dim],
    or uint8 [n, i8_row_bytes(dim)] for 'i8'.  'int' mode keeps every element
    an exact small integer in all storage types (i8: scale 1, integer bias)."""
    import torch
    if dtype == 'f32':
        return table_rows_at(table_id, row_ids, dim, mode, device, seed)
    if dtype in ('f16', 'bf16'):
        v = table_rows_at(table_id, row_ids, dim, mode, device, seed)
        return v.to(torch.float16 if dtype == 'f16' else torch.bfloat16)
    if dtype == 'fp8':
        # E4M3 codes (uint8) of the same values, rounded to nearest by the library
        # conversion; 'int' mode values (integers in [-8, 7]) are exact in E4M3
        v = table_rows_at(table_id, row_ids, dim, mode, device, seed)
        return v.to(torch.float8_e4m3fn).view(torch.uint8)
    if dtype != 'i8':
        raise ValueError(dtype)
    r = torch.as_tensor(row_ids, dtype=torch.int64, device=device).reshape(-1)
    n = r.numel()
    h0 = _mix32(torch.tensor(((table_id * 0x2545F491) + (seed * 0x9E3779B9) + 0x51ED27) & M32, dtype=torch.int64,
                             device=device))
    h1 = _mix32((h0 ^ (r & M32)) & M32)
    c = torch.arange(dim, dtype=torch.int64, device=device)
    h2 = _mix32((h1[:, None] + ((c * 0x61C88647) & M32)[None, :]) & M32)
    hs = _mix32((h1 + 0x3C6EF372) & M32)
    hb = _mix32((h1 + 0x7F4A7C15) & M32)
    if mode == 'float':
        q = (h2 >> 24) - 128                                             # [-128, 127]
        scale = ((hs >> 8).to(torch.float64) * 2.0 ** -24 + 1.0) * 2.0 ** -7  # [2^-7, 2^-6)
        bias = (hb >> 8).to(torch.float64) * 2.0 ** -23 - 1.0               # [-1, 1)
    elif mode == 'int':
        q = (h2 >> 28) - 8                                               # [-8, 7]
        scale = torch.ones(n, dtype=torch.float64, device=device)
        bias = ((hb >> 29) - 4).to(torch.float64)                         # [-4, 3]
    else:
        raise ValueError(mode)
    out = torch.zeros((n, i8_row_bytes(dim)), dtype=torch.uint8, device=device)
    out[:, :dim] = (q & 0xFF).to(torch.uint8)
    sb = torch.stack([scale.to(torch.float32), bias.to(torch.float32)], dim=1).contiguous()
    out[:, dim:dim + 8] = sb.view(torch.uint8).reshape(n, 8)
    return out


def make_table_stored(table_id: int, rows: int, dim: int, dtype: str = 'f32', mode: str = 'float', device='cpu',
                      seed: int = MODEL_SEED, chunk_rows: Optional[int] = None):
    """A whole physical table in storage type `dtype` (see table_rows_stored)."""
    import torch
    if dtype == 'f32':
        return make_table(table_id, rows, dim, mode, device, seed, chunk_rows)
    width = i8_row_bytes(dim) if dtype == 'i8' else dim
    tdt = {'f16': torch.float16, 'bf16': torch.bfloat16, 'i8': torch.uint8, 'fp8': torch.uint8}[dtype]
    out = torch.empty((rows, width), dtype=tdt, device=device)
    if chunk_rows is None:
        chunk_rows = max(1, (1 << 24) // max(1, dim))
    for a in range(0, rows, chunk_rows):
        b = min(rows, a + chunk_rows)
        out[a:b] = table_rows_stored(table_id, torch.arange(a, b, dtype=torch.int64, device=device), dim, dtype,
                                     mode, device, seed)
    return out


def row_bytes(dim: int, dtype: str = 'f32') -> int:
    """Algorithmic bytes of one stored row (C26 generalised): the element bytes,
    plus scale and bias for int8 (padding excluded)."""
    return {'f32': 4 * dim, 'f16': 2 * dim, 'bf16': 2 * dim, 'i8': dim + 8, 'fp8': dim}[dtype]


def make_tables(model: Model, mode: str = 'float', device='cpu'):
    """Physical tables of a model (list indexed by table id)."""
    return [make_table(t, rows, dim, mode, device, model.seed) for t, (rows, dim) in enumerate(model.tables)]


# ---------------------------------------------------------------------------
# Byte accounting (C26): what the method must move per batch
# ---------------------------------------------------------------------------

def algorithmic_bytes(model: Model, batch: Batch, dtype: str = 'f32') -> dict:
    """indices + gathered rows + outputs (reading C26); offsets reported apart.
    Rows count their stored bytes (row_bytes: int8 = codes + scale + bias)."""
    F, B = batch.F, batch.B
    offs = batch.offsets.astype(np.int64)
    nnz_f = offs[np.arange(1, F + 1) * B] - offs[np.arange(0, F) * B]
    dims = np.asarray(model.dims, np.int64)
    rowb = np.asarray([row_bytes(int(d), dtype) for d in dims], np.int64)
    idx_b = 4 * int(nnz_f.sum())
    row_b = int((rowb * nnz_f).sum())
    out_b = 4 * B * int(dims.sum())
    off_b = 4 * (F * B + 1)
    return {'index': idx_b, 'rows': row_b, 'out': out_b, 'offsets': off_b,
            'total': idx_b + row_b + out_b}
