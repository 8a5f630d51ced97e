"""Python face of the C ABI: a Plan object over torch tensors.

torch supplies device memory and streams only; every call below marshals
pointers into librecflex.so (include/recflex.h) and the work runs in its CUDA
kernels.  Names follow the C entry points (recflex_forward -> Plan.forward, ...).
"""
from __future__ import annotations

import ctypes
import json
from typing import List, Optional, Sequence

import torch

from . import _lib
from ._lib import check, lib

POOL_SUM = 0
POOL_MEAN = 1

# table row storage types (recflex_dtype_t)
DTYPES = {'f32': 0, 'f16': 1, 'bf16': 2, 'i8': 3, 'fp8': 4}
DTYPE_NAMES = {v: k for k, v in DTYPES.items()}


def dtype_code(dt) -> int:
    return DTYPES[dt] if isinstance(dt, str) else int(dt)


def i8_row_bytes(dim: int) -> int:
    """RECFLEX_I8_ROW_BYTES: d int8 codes + fp32 scale + fp32 bias, padded to 16 bytes."""
    return (dim + 8 + 15) // 16 * 16


def check_table(t: torch.Tensor, dim: int, dtype) -> None:
    """The tensor layout recflex_forward expects for a table of this dim / dtype."""
    code = dtype_code(dtype)
    want = {0: (torch.float32, dim), 1: (torch.float16, dim), 2: (torch.bfloat16, dim),
            3: (torch.uint8, i8_row_bytes(dim)), 4: (torch.uint8, dim)}[code]
    tdt = torch.uint8 if (code == 4 and t.dtype == torch.float8_e4m3fn) else t.dtype  # fp8: codes as uint8 or e4m3fn
    if not (t.is_cuda and tdt == want[0] and t.is_contiguous() and t.dim() == 2 and t.shape[1] == want[1]):
        raise ValueError(f'table: need contiguous CUDA {want[0]} [rows, {want[1]}] for dim {dim} '
                         f'dtype {DTYPE_NAMES[code]}, got {t.dtype} {tuple(t.shape)}')


def catalog():
    """List of dicts describing every catalog entry (schedule templates)."""
    out = []
    for i in range(lib.recflex_catalog_size()):
        ci = _lib.CatalogInfo()
        check(lib.recflex_catalog_info(i, ctypes.byref(ci)), 'recflex_catalog_info')
        out.append(dict(id=i, family=('group', 'block', 'flat', 'warp')[ci.family], G=ci.group, VEC=ci.vec, C=ci.cols,
                        U=ci.unroll, dtype=DTYPE_NAMES[ci.dtype]))
    return out


def occupancy_check(k: int, device: int = 0):
    a, r, s = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
    check(lib.recflex_occupancy_check(device, k, ctypes.byref(a), ctypes.byref(r), ctypes.byref(s)),
          'recflex_occupancy_check')
    return dict(active_blocks=a.value, registers=r.value, local_bytes=s.value)


def _stream_ptr(stream):
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def _dptr(t: torch.Tensor, dtype, name):
    if not t.is_cuda:
        raise ValueError(f'{name} must be a CUDA tensor')
    if t.dtype != dtype:
        raise TypeError(f'{name} must be {dtype}, got {t.dtype}')
    if not t.is_contiguous():
        raise ValueError(f'{name} must be contiguous')
    return ctypes.c_void_p(t.data_ptr())


class Plan:
    """recflex_plan_create / recflex_destroy around a list of feature specs.

    specs: sequence of dicts with keys rows, dim, pool, mean_len, max_len, coverage
    and optionally dtype ('f32' default, 'f16', 'bf16', 'i8' -- see check_table).
    """

    def __init__(self, specs: Sequence[dict], max_batch: int, device: int = 0):
        F = len(specs)
        arr = (_lib.FeatureSpec * F)()
        for i, s in enumerate(specs):
            arr[i].num_rows = int(s['rows'])
            arr[i].dim = int(s['dim'])
            arr[i].pool = int(s.get('pool', POOL_SUM))
            arr[i].mean_len = float(s.get('mean_len', 1.0))
            arr[i].max_len = float(s.get('max_len', 1.0))
            arr[i].coverage = float(s.get('coverage', 1.0))
            arr[i].dtype = dtype_code(s.get('dtype', 0))
        self._h = ctypes.c_void_p()
        check(lib.recflex_plan_create(arr, F, int(max_batch), int(device), ctypes.byref(self._h)),
              'recflex_plan_create')
        self.F = F
        self.dims = [int(s['dim']) for s in specs]
        self.dtypes = [dtype_code(s.get('dtype', 0)) for s in specs]
        self.d_tot = sum(self.dims)
        self.max_batch = int(max_batch)
        self.device = int(device)
        self._tables_key = None
        self._tables_arr = None

    @classmethod
    def from_model(cls, model, max_batch: Optional[int] = None, device: int = 0, dtype='f32') -> 'Plan':
        specs = [dict(rows=f.rows, dim=f.dim, pool=f.pool, mean_len=f.mean_len(), max_len=f.max_len(),
                      coverage=f.coverage, dtype=dtype) for f in model.features]
        return cls(specs, max_batch or model.batch, device)

    # -------------------------------------------------------------- lifecycle
    def close(self):
        if getattr(self, '_h', None) and self._h.value:
            lib.recflex_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # -------------------------------------------------------------- helpers
    def _tables(self, tables: Sequence[torch.Tensor]):
        if len(tables) != self.F:
            raise ValueError(f'expected {self.F} tables, got {len(tables)}')
        key = tuple(t.data_ptr() for t in tables)
        if key != self._tables_key:
            for f, t in enumerate(tables):
                try:
                    check_table(t, self.dims[f], self.dtypes[f])
                except ValueError as ex:
                    raise ValueError(f'table {f}: {ex}') from None
            self._tables_arr = (ctypes.c_void_p * self.F)(*key)
            self._tables_key = key
        return self._tables_arr

    # -------------------------------------------------------------- fusion compiler
    def compile(self, occupancies: Optional[Sequence[int]] = None) -> dict:
        """recflex_plan_compile: NVRTC-compile the plan-specialised fused kernel for the
        current schedules (at the plan's occupancy, or each k given); returns jit_info."""
        ks = [int(k) for k in occupancies] if occupancies else []
        arr = (ctypes.c_int32 * max(1, len(ks)))(*ks) if ks else None
        check(lib.recflex_plan_compile(self._h, arr, len(ks)), 'recflex_plan_compile')
        return self.jit_info(ks[0] if len(ks) == 1 else 0)

    def jit_info(self, k: int = 0) -> dict:
        ji = _lib.JitInfo()
        check(lib.recflex_jit_info(self._h, int(k), ctypes.byref(ji)), 'recflex_jit_info')
        return {n: getattr(ji, n) for n, _ in _lib.JitInfo._fields_}

    def set_jit(self, enable: bool) -> None:
        check(lib.recflex_set_jit(self._h, 1 if enable else 0), 'recflex_set_jit')

    @property
    def jit_enabled(self) -> bool:
        v = ctypes.c_int32()
        check(lib.recflex_get_jit(self._h, ctypes.byref(v)), 'recflex_get_jit')
        return bool(v.value)

    def select_kernel(self, indices: torch.Tensor, offsets: torch.Tensor, B: int, tables: Sequence[torch.Tensor],
                      reps: int = 7, stream=None) -> dict:
        """recflex_select_kernel: time the plan-specialised and the catalog kernel on this
        batch and keep the faster (part of the exported plan)."""
        j, c = ctypes.c_float(), ctypes.c_float()
        check(lib.recflex_select_kernel(self._h, _dptr(indices, torch.int32, 'indices'),
                                        _dptr(offsets, torch.int32, 'offsets'), int(B), self._tables(tables),
                                        int(reps), ctypes.byref(j), ctypes.byref(c), _stream_ptr(stream)),
              'recflex_select_kernel')
        return dict(jit_ms=j.value, catalog_ms=c.value, kernel='plan-specialised' if self.jit_enabled else 'catalog')

    # -------------------------------------------------------------- task order (reading C35)
    ORDER_KINDS = ('feature', 'lpt', 'spt')  # RECFLEX_ORDER_*

    @property
    def task_order(self) -> List[int]:
        """recflex_get_task_order: position -> feature (the order tasks are claimed in)."""
        o = (ctypes.c_int32 * self.F)()
        check(lib.recflex_get_task_order(self._h, o), 'recflex_get_task_order')
        return list(o)

    @task_order.setter
    def task_order(self, order: Optional[Sequence[int]]):
        """recflex_set_task_order: a permutation of range(F), or None = feature order."""
        if order is not None and len(order) != self.F:
            raise ValueError('task order: need a permutation of range(F)')
        arr = None if order is None else (ctypes.c_int32 * self.F)(*[int(f) for f in order])
        check(lib.recflex_set_task_order(self._h, arr), 'recflex_set_task_order')

    def set_column_order(self, follow_task_order: bool):
        """recflex_set_column_order: concatenate the pooled outputs in task order (True) or
        feature order (False, default)."""
        check(lib.recflex_set_column_order(self._h, 1 if follow_task_order else 0), 'recflex_set_column_order')

    @property
    def columns(self) -> List[int]:
        """recflex_get_columns: first output column of every feature."""
        c = (ctypes.c_int64 * self.F)()
        check(lib.recflex_get_columns(self._h, c), 'recflex_get_columns')
        return list(c)

    # -------------------------------------------------------------- L2 policy (reading C36)
    L2_POLICIES = ('default', 'evict_first', 'evict_last', 'keep_l1')  # RECFLEX_L2_*

    @property
    def l2_policy(self) -> List[int]:
        """recflex_get_l2_policy: every feature's L2 eviction priority (0/1/2)."""
        o = (ctypes.c_int32 * self.F)()
        check(lib.recflex_get_l2_policy(self._h, o), 'recflex_get_l2_policy')
        return list(o)

    @l2_policy.setter
    def l2_policy(self, policy: Optional[Sequence[int]]):
        if policy is not None and len(policy) != self.F:
            raise ValueError('l2 policy: one value per feature')
        arr = None if policy is None else (ctypes.c_int32 * self.F)(*[int(v) for v in policy])
        check(lib.recflex_set_l2_policy(self._h, arr), 'recflex_set_l2_policy')

    def l2_policy_heuristic(self, l2_bytes: int = 126 * 2 ** 20) -> List[int]:
        o = (ctypes.c_int32 * self.F)()
        check(lib.recflex_l2_policy_heuristic(self._h, int(l2_bytes), o), 'recflex_l2_policy_heuristic')
        return list(o)

    TASK_SIZES = ('x1', 'x1/2', 'x2')  # recflex_select_task_size

    def select_task_size(self, indices: torch.Tensor, offsets: torch.Tensor, B: int,
                         tables: Sequence[torch.Tensor], reps: int = 7, stream=None) -> dict:
        """recflex_select_task_size: every feature's per-task size x1, x1/2, x2 timed, the fastest kept."""
        chosen = ctypes.c_int32()
        ms = (ctypes.c_float * 3)()
        check(lib.recflex_select_task_size(self._h, _dptr(indices, torch.int32, 'indices'),
                                           _dptr(offsets, torch.int32, 'offsets'), int(B), self._tables(tables),
                                           int(reps), ctypes.byref(chosen), ms, _stream_ptr(stream)),
              'recflex_select_task_size')
        return dict(task_size=self.TASK_SIZES[chosen.value], ms={k: ms[i] for i, k in enumerate(self.TASK_SIZES)})

    L2_CANDIDATES = ('none', 'heuristic', 'evict_last_only')  # recflex_select_l2_policy

    def select_l2_policy(self, indices: torch.Tensor, offsets: torch.Tensor, B: int,
                         tables: Sequence[torch.Tensor], reps: int = 7, l2_bytes: int = 126 * 2 ** 20,
                         stream=None) -> dict:
        """recflex_select_l2_policy: time no hints / the heuristic / its evict_last part, keep the fastest."""
        chosen = ctypes.c_int32()
        ms = (ctypes.c_float * 3)()
        check(lib.recflex_select_l2_policy(self._h, _dptr(indices, torch.int32, 'indices'),
                                           _dptr(offsets, torch.int32, 'offsets'), int(B), self._tables(tables),
                                           int(reps), int(l2_bytes), ctypes.byref(chosen), ms, _stream_ptr(stream)),
              'recflex_select_l2_policy')
        return dict(l2=self.L2_CANDIDATES[chosen.value], ms={k: ms[i] for i, k in enumerate(self.L2_CANDIDATES)})

    def task_order_heuristic(self, kind: str) -> List[int]:
        o = (ctypes.c_int32 * self.F)()
        check(lib.recflex_task_order_heuristic(self._h, self.ORDER_KINDS.index(kind), o),
              'recflex_task_order_heuristic')
        return list(o)

    def select_task_order(self, indices: torch.Tensor, offsets: torch.Tensor, B: int,
                          tables: Sequence[torch.Tensor], reps: int = 7, stream=None) -> dict:
        """recflex_select_task_order: time every heuristic order on this batch, keep the fastest."""
        chosen = ctypes.c_int32()
        ms = (ctypes.c_float * len(self.ORDER_KINDS))()
        check(lib.recflex_select_task_order(self._h, _dptr(indices, torch.int32, 'indices'),
                                            _dptr(offsets, torch.int32, 'offsets'), int(B), self._tables(tables),
                                            int(reps), ctypes.byref(chosen), ms, _stream_ptr(stream)),
              'recflex_select_task_order')
        return dict(order=self.ORDER_KINDS[chosen.value], ms={k: ms[i] for i, k in enumerate(self.ORDER_KINDS)})

    # -------------------------------------------------------------- hot path
    def forward(self, indices: torch.Tensor, offsets: torch.Tensor, B: int, tables: Sequence[torch.Tensor],
                out: Optional[torch.Tensor] = None, stream=None) -> torch.Tensor:
        """recflex_forward: pooled [B, D_tot] float32 (async on `stream`)."""
        if out is None:
            out = torch.empty((B, self.d_tot), dtype=torch.float32, device=offsets.device)
        if out.shape != (B, self.d_tot) or out.dtype != torch.float32 or not out.is_contiguous():
            raise ValueError('out must be contiguous float32 [B, D_tot]')
        if offsets.numel() != self.F * B + 1:
            raise ValueError('offsets must have F*B+1 entries')
        tarr = self._tables(tables)
        idx_ptr = _dptr(indices, torch.int32, 'indices') if indices.numel() else ctypes.c_void_p(offsets.data_ptr())
        check(lib.recflex_forward(self._h, idx_ptr, _dptr(offsets, torch.int32, 'offsets'), int(B),
                                  tarr, _dptr(out, torch.float32, 'out'), _stream_ptr(stream)),
              'recflex_forward')
        return out

    def forward_routed(self, indices: torch.Tensor, offsets: torch.Tensor, B: int, tables: Sequence[torch.Tensor],
                       dst_ptrs: Sequence[int], rows_per_dst: int, dst_stride: int, col_base: int, stream=None):
        """recflex_forward_routed: pooled rows stored straight into destination buffers
        (device pointers, e.g. IPC-mapped peers): the fused all-to-all epilogue."""
        if offsets.numel() != self.F * B + 1:
            raise ValueError('offsets must have F*B+1 entries')
        tarr = self._tables(tables)
        darr = (ctypes.c_void_p * len(dst_ptrs))(*[int(p) for p in dst_ptrs])
        idx_ptr = _dptr(indices, torch.int32, 'indices') if indices.numel() else ctypes.c_void_p(offsets.data_ptr())
        check(lib.recflex_forward_routed(self._h, idx_ptr, _dptr(offsets, torch.int32, 'offsets'), int(B), tarr, darr,
                                         len(dst_ptrs), int(rows_per_dst), int(dst_stride), int(col_base),
                                         _stream_ptr(stream)), 'recflex_forward_routed')

    def forward_exchange(self, indices: torch.Tensor, offsets: torch.Tensor, B: int, tables: Sequence[torch.Tensor],
                         world: int, rank: int, rows_per_dst: int, dst_stride: int, col_base: int,
                         dst0: Sequence[int], dst1: Sequence[int], flags: Sequence[int], local_flags: int,
                         stream=None) -> int:
        """recflex_forward_exchange: routed forward into double-buffered destinations with a
        device-side completion signal (no host barrier); returns the buffer index (0/1) this
        step wrote -- see include/recflex.h for the lifetime rule."""
        if offsets.numel() != self.F * B + 1:
            raise ValueError('offsets must have F*B+1 entries')
        tarr = self._tables(tables)
        key = (tuple(dst0), tuple(dst1), tuple(flags))
        if getattr(self, '_xkey', None) != key:
            W = int(world)
            self._xarrs = [(ctypes.c_void_p * W)(*[int(p) for p in dst0]), (ctypes.c_void_p * W)(*[int(p) for p in dst1]),
                           (ctypes.c_void_p * W)(*[int(p) for p in flags])]
            self._xkey = key
        x = _lib.Exchange()
        x.world, x.rank, x.rows_per_dst, x.dst_stride, x.col_base = (int(world), int(rank), int(rows_per_dst),
                                                                      int(dst_stride), int(col_base))
        x.dst[0] = ctypes.cast(self._xarrs[0], ctypes.c_void_p)
        x.dst[1] = ctypes.cast(self._xarrs[1], ctypes.c_void_p)
        x.flags = ctypes.cast(self._xarrs[2], ctypes.c_void_p)
        x.local_flags = int(local_flags)
        idx_ptr = _dptr(indices, torch.int32, 'indices') if indices.numel() else ctypes.c_void_p(offsets.data_ptr())
        bi = ctypes.c_int32()
        check(lib.recflex_forward_exchange(self._h, idx_ptr, _dptr(offsets, torch.int32, 'offsets'), int(B), tarr,
                                           ctypes.byref(x), ctypes.byref(bi), _stream_ptr(stream)),
              'recflex_forward_exchange')
        return bi.value

    def forward_host(self, indices: torch.Tensor, offsets: torch.Tensor, B: int, tables: Sequence[torch.Tensor],
                     out: torch.Tensor, stream=None) -> torch.Tensor:
        """recflex_forward_host: host (pinned) int32 inputs -> host float32 out [B, D_tot]; blocking."""
        for name, t, dt in (('indices', indices, torch.int32), ('offsets', offsets, torch.int32),
                            ('out', out, torch.float32)):
            if t.is_cuda or t.dtype != dt or not t.is_contiguous():
                raise ValueError(f'{name} must be a contiguous host {dt} tensor')
        tarr = self._tables(tables)
        check(lib.recflex_forward_host(self._h, ctypes.c_void_p(indices.data_ptr()), int(indices.numel()),
                                       ctypes.c_void_p(offsets.data_ptr()), int(B), tarr,
                                       ctypes.c_void_p(out.data_ptr()), _stream_ptr(stream)),
              'recflex_forward_host')
        return out

    def forward_host_batches(self, batches: Sequence[tuple], tables: Sequence[torch.Tensor],
                             outs: Sequence[torch.Tensor], stream=None):
        """recflex_forward_host_batches: [(indices, offsets, B)] host (pinned) int32 -> host float32
        outs[i] [B_i, D_tot]; H2D / forward / D2H of consecutive batches overlapped; blocking."""
        n = len(batches)
        if len(outs) != n:
            raise ValueError('one output per batch')
        for i, ((ind, off, B), out) in enumerate(zip(batches, outs)):
            for name, t, dt in (('indices', ind, torch.int32), ('offsets', off, torch.int32),
                                ('out', out, torch.float32)):
                if t.is_cuda or t.dtype != dt or not t.is_contiguous():
                    raise ValueError(f'batch {i}: {name} must be a contiguous host {dt} tensor')
            if off.numel() != self.F * B + 1 or out.shape != (B, self.d_tot):
                raise ValueError(f'batch {i}: offsets must hold F*B+1 entries, out [B, D_tot]')
        tarr = self._tables(tables)
        P = ctypes.c_void_p
        check(lib.recflex_forward_host_batches(
            self._h, n, (P * n)(*[b[0].data_ptr() for b in batches]),
            (ctypes.c_int64 * n)(*[b[0].numel() for b in batches]), (P * n)(*[b[1].data_ptr() for b in batches]),
            (ctypes.c_int32 * n)(*[int(b[2]) for b in batches]), tarr, (P * n)(*[o.data_ptr() for o in outs]),
            _stream_ptr(stream)), 'recflex_forward_host_batches')
        return outs

    # -------------------------------------------------------------- backward (NEXT #4)
    def backward(self, indices: torch.Tensor, offsets: torch.Tensor, B: int, grad: torch.Tensor,
                 targets: Sequence[torch.Tensor], scale: float = 1.0, stream=None):
        """recflex_backward: targets[f][id] += scale * w * grad[s][col_f:] for every lookup
        (dense table gradients with zeroed targets and scale 1; SGD with targets = tables,
        scale = -lr).  targets: F contiguous CUDA float32 [rows_f, d_f]."""
        if offsets.numel() != self.F * B + 1:
            raise ValueError('offsets must have F*B+1 entries')
        if grad.shape != (B, self.d_tot):
            raise ValueError(f'grad must be [B, D_tot] = [{B}, {self.d_tot}]')
        if len(targets) != self.F:
            raise ValueError(f'expected {self.F} targets')
        for f, t in enumerate(targets):
            check_table(t, self.dims[f], 0)
        tarr = (ctypes.c_void_p * self.F)(*[t.data_ptr() for t in targets])
        idx_ptr = _dptr(indices, torch.int32, 'indices') if indices.numel() else ctypes.c_void_p(offsets.data_ptr())
        check(lib.recflex_backward(self._h, idx_ptr, _dptr(offsets, torch.int32, 'offsets'), int(B),
                                   _dptr(grad, torch.float32, 'grad'), tarr, float(scale), _stream_ptr(stream)),
              'recflex_backward')

    def sgd_step(self, indices: torch.Tensor, offsets: torch.Tensor, B: int, grad: torch.Tensor,
                 tables: Sequence[torch.Tensor], lr: float, stream=None):
        """One fused SGD update of float32 tables: T -= lr * dLoss/dT (recflex_backward, scale = -lr)."""
        self.backward(indices, offsets, B, grad, tables, scale=-float(lr), stream=stream)

    # -------------------------------------------------------------- tuner
    def tune(self, batches: Sequence[tuple], tables: Sequence[torch.Tensor], occupancies: Optional[List[int]] = None,
             reps: int = 7, pad_waves: int = 4, max_candidates: int = 0, verbose: bool = False, guard: bool = True,
             refine: bool = False, separate: bool = False, stage2_catalog: bool = False, tail: bool = True,
             isolated: bool = False, select_order: bool = True, select_l2: bool = True,
             select_task_size: bool = True, switch_margin: float = 0.0, position_balance: bool = False,
             stream=None) -> dict:
        """recflex_tune_ex over historical batches [(indices, offsets, B), ...]."""
        N = len(batches)
        idx_arr = (ctypes.c_void_p * N)(*[b[0].data_ptr() for b in batches])
        off_arr = (ctypes.c_void_p * N)(*[b[1].data_ptr() for b in batches])
        bs_arr = (ctypes.c_int32 * N)(*[int(b[2]) for b in batches])
        opt = _lib.TuneOptions()
        if occupancies:
            opt.num_occupancies = len(occupancies)
            for i, k in enumerate(occupancies):
                opt.occupancies[i] = int(k)
        opt.reps = reps
        opt.pad_waves = pad_waves
        opt.max_candidates = max_candidates
        opt.verbose = 1 if verbose else 0
        opt.skip_guard = 0 if guard else 1
        opt.refine = 1 if refine else 0
        opt.local_mode = 1 if separate else (2 if isolated else 0)
        opt.stage2_catalog = 1 if stage2_catalog else 0
        opt.no_tail = 0 if tail else 1
        opt.keep_order = 0 if select_order else 1
        opt.keep_l2 = 0 if select_l2 else 1
        opt.keep_task_size = 0 if select_task_size else 1
        opt.switch_margin = float(switch_margin)
        opt.position_balance = 1 if position_balance else 0
        st = _lib.TuneStats()
        check(lib.recflex_tune_ex(self._h, N, idx_arr, off_arr, bs_arr, self._tables(tables), _stream_ptr(stream),
                                  ctypes.byref(opt), ctypes.byref(st)), 'recflex_tune_ex')
        return dict(local_launches=st.local_launches, global_launches=st.global_launches,
                    local_evals=st.local_evals, global_evals=st.global_evals, guard_evals=st.guard_evals,
                    guard_won=bool(st.guard_won), refine_evals=st.refine_evals, refine_gain=st.refine_gain,
                    best_occupancy=st.best_occupancy, best_ms=st.best_ms, tune_seconds=st.tune_seconds,
                    two_stage_ms=st.two_stage_ms, incoming_ms=st.incoming_ms, jit_compiles=st.jit_compiles,
                    compile_seconds=st.compile_seconds, refine_seconds=st.refine_seconds,
                    task_order=self.ORDER_KINDS[st.task_order] if st.task_order >= 0 else None,
                    l2_policy=self.L2_CANDIDATES[st.l2_policy] if st.l2_policy >= 0 else None,
                    task_size=self.TASK_SIZES[st.task_size] if st.task_size >= 0 else None)

    # -------------------------------------------------------------- schedules
    def get_schedule(self, f: int) -> dict:
        s = _lib.Schedule()
        k = ctypes.c_int32()
        check(lib.recflex_get_schedule(self._h, f, ctypes.byref(s), ctypes.byref(k)), 'recflex_get_schedule')
        return dict(sched_id=s.sched_id, part=s.part, per_block=s.per_block, static_blocks=s.static_blocks)

    def set_schedule(self, f: int, sched_id: int, part: int = 0, per_block: int = 256, static_blocks: int = 0):
        """static_blocks > 0: the paper's static thread mapping with that many allocated tasks."""
        s = _lib.Schedule(int(sched_id), int(part), int(per_block), int(static_blocks))
        check(lib.recflex_set_schedule(self._h, f, ctypes.byref(s)), 'recflex_set_schedule')

    @property
    def occupancy(self) -> int:
        k = ctypes.c_int32()
        check(lib.recflex_get_occupancy(self._h, ctypes.byref(k)), 'recflex_get_occupancy')
        return k.value

    @occupancy.setter
    def occupancy(self, k: int):
        check(lib.recflex_set_occupancy(self._h, int(k)), 'recflex_set_occupancy')

    # -------------------------------------------------------------- introspection
    def debug_task_map(self, offsets: torch.Tensor, B: int, ranges: bool = False, stream=None):
        """block_start[F+1] over the task order (entry e = feature task_order[e]) and, with
        ranges, every task's [s0, s1) (lookup-partitioned features; else (-1, -1))."""
        bs = (ctypes.c_int32 * (self.F + 1))()
        if not ranges:
            check(lib.recflex_debug_task_map(self._h, _dptr(offsets, torch.int32, 'offsets'), int(B), bs, None, 0,
                                             _stream_ptr(stream)), 'recflex_debug_task_map')
            return list(bs), None
        check(lib.recflex_debug_task_map(self._h, _dptr(offsets, torch.int32, 'offsets'), int(B), bs, None, 0,
                                         _stream_ptr(stream)), 'recflex_debug_task_map')
        total = bs[self.F]
        rg = (ctypes.c_int32 * max(2, 2 * total))()
        check(lib.recflex_debug_task_map(self._h, _dptr(offsets, torch.int32, 'offsets'), int(B), bs, rg,
                                         max(2, 2 * total), _stream_ptr(stream)), 'recflex_debug_task_map')
        return list(bs), [(rg[2 * t], rg[2 * t + 1]) for t in range(total)]

    def task_slots(self, f: int) -> int:
        """recflex_get_task_slots: task-range slots reserved for feature f (reading C12)."""
        v = ctypes.c_int32()
        check(lib.recflex_get_task_slots(self._h, int(f), ctypes.byref(v)), 'recflex_get_task_slots')
        return v.value

    def debug_task_need(self) -> List[int]:
        """recflex_debug_task_need: tasks every feature NEEDED in the last map (before a static
        mapping folds them onto its allocated tasks)."""
        nd = (ctypes.c_int32 * self.F)()
        check(lib.recflex_debug_task_need(self._h, nd), 'recflex_debug_task_need')
        return list(nd)

    def validate(self, indices: torch.Tensor, offsets: torch.Tensor, B: int, stream=None) -> int:
        """Returns the raw status (0 ok, 1 invalid offsets, 5 index out of range)."""
        ip = ctypes.c_void_p(indices.data_ptr()) if indices.numel() else ctypes.c_void_p(offsets.data_ptr())
        return int(lib.recflex_validate(self._h, ip, _dptr(offsets, torch.int32, 'offsets'), int(B),
                                        _stream_ptr(stream)))

    def export(self) -> dict:
        n = ctypes.c_size_t()
        check(lib.recflex_plan_export(self._h, None, 0, ctypes.byref(n)), 'recflex_plan_export')
        buf = ctypes.create_string_buffer(n.value)
        check(lib.recflex_plan_export(self._h, buf, n.value, ctypes.byref(n)), 'recflex_plan_export')
        return json.loads(buf.value.decode())

    def import_(self, state: dict):
        check(lib.recflex_plan_import(self._h, json.dumps(state).encode()), 'recflex_plan_import')

    def set_profiling(self, enable: bool):
        check(lib.recflex_set_profiling(self._h, 1 if enable else 0), 'recflex_set_profiling')

    def kernel_times(self, reset: bool = True) -> dict:
        a, b, n = ctypes.c_double(), ctypes.c_double(), ctypes.c_int64()
        check(lib.recflex_get_kernel_times(self._h, ctypes.byref(a), ctypes.byref(b), ctypes.byref(n),
                                           1 if reset else 0), 'recflex_get_kernel_times')
        return dict(map_ms=a.value, fused_ms=b.value, forwards=n.value)


def shard_concat(recv: torch.Tensor, dims_per_rank: Sequence[int], rows: int, out: torch.Tensor, stream=None):
    """recflex_shard_concat: [W chunks of rows x d_i] -> [rows, sum d_i]."""
    W = len(dims_per_rank)
    dims = (ctypes.c_int32 * W)(*[int(d) for d in dims_per_rank])
    check(lib.recflex_shard_concat(_dptr(recv, torch.float32, 'recv'), W, int(rows), dims,
                                   _dptr(out, torch.float32, 'out'), _stream_ptr(stream)), 'recflex_shard_concat')
    return out


class DeviceBuffer:
    """A float32 [rows, cols] buffer from the library's own cudaMalloc (so its
    CUDA-IPC handle maps at offset 0), viewed as a torch tensor."""

    def __init__(self, rows: int, cols: int, device: int = 0):
        self.ptr = ctypes.c_void_p()
        nbytes = max(4, rows * cols * 4)
        check(lib.recflex_device_alloc(nbytes, device, ctypes.byref(self.ptr)), 'recflex_device_alloc')
        self.__cuda_array_interface__ = {'shape': (rows, cols), 'typestr': '<f4', 'data': (self.ptr.value, False),
                                         'version': 3, 'strides': None}
        self.tensor = torch.as_tensor(self, device=torch.device('cuda', device))

    def close(self):
        if self.ptr and self.ptr.value:
            lib.recflex_device_free(self.ptr)
            self.ptr = ctypes.c_void_p()


def ipc_handle(t) -> bytes:
    """64-byte CUDA IPC handle of a DeviceBuffer (or a tensor that starts its allocation)."""
    ptr = t.ptr.value if isinstance(t, DeviceBuffer) else t.data_ptr()
    buf = ctypes.create_string_buffer(64)
    check(lib.recflex_ipc_get_handle(ctypes.c_void_p(ptr), buf), 'recflex_ipc_get_handle')
    return buf.raw


def ipc_open(handle: bytes) -> int:
    p = ctypes.c_void_p()
    check(lib.recflex_ipc_open_handle(ctypes.create_string_buffer(handle, 64), ctypes.byref(p)),
          'recflex_ipc_open_handle')
    return int(p.value)


def ipc_close(ptr: int):
    check(lib.recflex_ipc_close(ctypes.c_void_p(ptr)), 'recflex_ipc_close')


def l2_flush(buf: torch.Tensor, stream=None):
    check(lib.recflex_l2_flush(ctypes.c_void_p(buf.data_ptr()), buf.numel() * buf.element_size(),
                               _stream_ptr(stream)), 'recflex_l2_flush')


class KJTDist:
    """recflex_kjt_dist_* : the table-wise input distribution's two device
    passes around the caller's alltoallv (include/recflex.h).

    owner[f] = rank owning feature f; this object is rank `rank`'s view with
    `local_batch` samples per rank.  pack/unpack take and fill caller-owned
    int32 CUDA tensors (no allocation inside the library)."""

    def __init__(self, owner: Sequence[int], world: int, rank: int, local_batch: int, device: int = 0):
        F = len(owner)
        arr = (ctypes.c_int32 * F)(*[int(o) for o in owner])
        self._h = ctypes.c_void_p()
        check(lib.recflex_kjt_dist_create(F, arr, int(world), int(rank), int(local_batch), int(device),
                                          ctypes.byref(self._h)), 'recflex_kjt_dist_create')
        self.F, self.world, self.rank, self.local_batch = F, int(world), int(rank), int(local_batch)
        sl = (ctypes.c_int32 * world)()
        rl = (ctypes.c_int32 * world)()
        fr = ctypes.c_int32()
        check(lib.recflex_kjt_dist_sizes(self._h, sl, rl, ctypes.byref(fr)), 'recflex_kjt_dist_sizes')
        self.send_length_counts = list(sl)
        self.recv_length_counts = list(rl)
        self.num_owned = fr.value

    def close(self):
        if getattr(self, '_h', None) and self._h.value:
            lib.recflex_kjt_dist_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def pack(self, indices: torch.Tensor, offsets: torch.Tensor, send_lengths: torch.Tensor,
             send_indices: torch.Tensor, dest_counts: torch.Tensor, stream=None):
        """recflex_kjt_pack: local KJT -> destination-major lengths / IDs + per-destination ID counts."""
        if offsets.numel() != self.F * self.local_batch + 1:
            raise ValueError('offsets must have F*Bl+1 entries')
        if send_lengths.numel() != self.F * self.local_batch or dest_counts.numel() != self.world:
            raise ValueError('send_lengths must hold F*Bl, dest_counts W entries')
        if send_indices.numel() < indices.numel():
            raise ValueError('send_indices smaller than the local IDs')
        nul = ctypes.c_void_p(offsets.data_ptr())
        check(lib.recflex_kjt_pack(self._h, _dptr(indices, torch.int32, 'indices') if indices.numel() else nul,
                                   _dptr(offsets, torch.int32, 'offsets'),
                                   _dptr(send_lengths, torch.int32, 'send_lengths') if send_lengths.numel() else nul,
                                   _dptr(send_indices, torch.int32, 'send_indices') if send_indices.numel() else nul,
                                   _dptr(dest_counts, torch.int32, 'dest_counts'), _stream_ptr(stream)),
              'recflex_kjt_pack')

    def unpack(self, recv_lengths: torch.Tensor, recv_indices: torch.Tensor, indices_out: torch.Tensor,
               offsets_out: torch.Tensor, stream=None):
        """recflex_kjt_unpack: source-major received buffers -> owned features' KJT (global sample order)."""
        B = self.world * self.local_batch
        if recv_lengths.numel() != self.world * self.num_owned * self.local_batch:
            raise ValueError('recv_lengths must hold W*F_r*Bl entries')
        if offsets_out.numel() != self.num_owned * B + 1 or indices_out.numel() < recv_indices.numel():
            raise ValueError('offsets_out must hold F_r*B+1 entries, indices_out the received IDs')
        nul = ctypes.c_void_p(offsets_out.data_ptr())
        check(lib.recflex_kjt_unpack(self._h,
                                     _dptr(recv_lengths, torch.int32, 'recv_lengths') if recv_lengths.numel() else nul,
                                     _dptr(recv_indices, torch.int32, 'recv_indices') if recv_indices.numel() else nul,
                                     _dptr(indices_out, torch.int32, 'indices_out') if indices_out.numel() else nul,
                                     _dptr(offsets_out, torch.int32, 'offsets_out'), _stream_ptr(stream)),
              'recflex_kjt_unpack')


def jit_generate(sched_ids, dims, pools, k: int, dtypes=None):
    """recflex_jit_generate (no GPU needed): (source, variant_of_feature, num_variants)."""
    F = len(sched_ids)
    A = ctypes.c_int32 * F
    dt = A(*[dtype_code(d) for d in dtypes]) if dtypes is not None else None
    n = ctypes.c_size_t()
    nv = ctypes.c_int32()
    var = A()
    check(lib.recflex_jit_generate(A(*sched_ids), A(*dims), A(*pools), dt, F, int(k), None, 0, ctypes.byref(n),
                                   var, ctypes.byref(nv)), 'recflex_jit_generate')
    buf = ctypes.create_string_buffer(n.value + 1)
    check(lib.recflex_jit_generate(A(*sched_ids), A(*dims), A(*pools), dt, F, int(k), buf, n.value + 1, None, None,
                                   None), 'recflex_jit_generate')
    return buf.value.decode(), list(var), nv.value


def jit_compile_source(source: str):
    """recflex_jit_compile_source (no GPU needed): (cubin bytes, NVRTC log, cache_hit)."""
    n = ctypes.c_size_t()
    log = ctypes.create_string_buffer(1 << 16)
    hit = ctypes.c_int32()
    check(lib.recflex_jit_compile_source(source.encode(), None, 0, ctypes.byref(n), log, 1 << 16, ctypes.byref(hit)),
          'recflex_jit_compile_source')
    buf = ctypes.create_string_buffer(n.value)
    check(lib.recflex_jit_compile_source(source.encode(), buf, n.value, ctypes.byref(n), None, 0, None),
          'recflex_jit_compile_source')
    return buf.raw[:n.value], log.value.decode(errors='replace'), bool(hit.value)
