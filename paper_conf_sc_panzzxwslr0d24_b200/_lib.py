"""ctypes binding of include/recflex.h (librecflex.so).

Argument marshalling only: every step of the hot path runs in the library's
CUDA kernels.  There is no fallback -- if librecflex.so is missing or fails to
load, importing this module raises (build it with ``python -m
paper_conf_sc_panzzxwslr0d24_b200.build`` or ``__graft_entry__.build()``).
"""
from __future__ import annotations

import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get('RECFLEX_LIB') or os.path.join(HERE, 'lib', 'librecflex.so')

c_int32 = ctypes.c_int32
c_int64 = ctypes.c_int64
c_void_p = ctypes.c_void_p
P = ctypes.POINTER


class FeatureSpec(ctypes.Structure):
    _fields_ = [('num_rows', ctypes.c_int64), ('dim', ctypes.c_int32), ('pool', ctypes.c_int32),
                ('mean_len', ctypes.c_float), ('max_len', ctypes.c_float), ('coverage', ctypes.c_float),
                ('dtype', ctypes.c_int32)]


class Schedule(ctypes.Structure):
    _fields_ = [('sched_id', ctypes.c_int32), ('part', ctypes.c_int32), ('per_block', ctypes.c_int32),
                ('static_blocks', ctypes.c_int32)]


class CatalogInfo(ctypes.Structure):
    _fields_ = [('family', ctypes.c_int32), ('group', ctypes.c_int32), ('vec', ctypes.c_int32),
                ('cols', ctypes.c_int32), ('unroll', ctypes.c_int32), ('dtype', ctypes.c_int32)]


class TuneOptions(ctypes.Structure):
    _fields_ = [('num_occupancies', ctypes.c_int32), ('occupancies', ctypes.c_int32 * 8),
                ('reps', ctypes.c_int32), ('pad_waves', ctypes.c_int32), ('max_candidates', ctypes.c_int32),
                ('verbose', ctypes.c_int32), ('skip_guard', ctypes.c_int32), ('refine', ctypes.c_int32),
                ('local_mode', ctypes.c_int32), ('stage2_catalog', ctypes.c_int32), ('no_tail', ctypes.c_int32),
                ('keep_order', ctypes.c_int32), ('keep_l2', ctypes.c_int32), ('keep_task_size', ctypes.c_int32),
                ('switch_margin', ctypes.c_float), ('position_balance', ctypes.c_int32)]


class TuneStats(ctypes.Structure):
    _fields_ = [('local_launches', ctypes.c_int64), ('global_launches', ctypes.c_int64),
                ('local_evals', ctypes.c_int64), ('global_evals', ctypes.c_int64),
                ('guard_evals', ctypes.c_int64), ('guard_won', ctypes.c_int32),
                ('best_occupancy', ctypes.c_int32), ('best_ms', ctypes.c_double), ('tune_seconds', ctypes.c_double),
                ('refine_evals', ctypes.c_int64), ('refine_gain', ctypes.c_double),
                ('two_stage_ms', ctypes.c_double), ('incoming_ms', ctypes.c_double), ('jit_compiles', ctypes.c_int64),
                ('compile_seconds', ctypes.c_double), ('refine_seconds', ctypes.c_double),
                ('task_order', ctypes.c_int32), ('l2_policy', ctypes.c_int32), ('task_size', ctypes.c_int32)]


class JitInfo(ctypes.Structure):
    _fields_ = [('compiled', ctypes.c_int32), ('active', ctypes.c_int32), ('variants', ctypes.c_int32),
                ('registers', ctypes.c_int32), ('local_bytes', ctypes.c_int32), ('blocks_per_sm', ctypes.c_int32),
                ('smem_bytes', ctypes.c_int32), ('cache_hit', ctypes.c_int32), ('compile_ms', ctypes.c_float)]


class Exchange(ctypes.Structure):
    _fields_ = [('world', ctypes.c_int32), ('rank', ctypes.c_int32), ('rows_per_dst', ctypes.c_int32),
                ('dst_stride', ctypes.c_int32), ('col_base', ctypes.c_int32), ('dst', ctypes.c_void_p * 2),
                ('flags', ctypes.c_void_p), ('local_flags', ctypes.c_void_p)]


LOCAL_COST_FN = ctypes.CFUNCTYPE(None, c_void_p, c_int32, c_int32, P(ctypes.c_double))
GLOBAL_COST_FN = ctypes.CFUNCTYPE(ctypes.c_double, c_void_p, c_int32, P(c_int32))

OK = 0
STATUS = {0: 'RECFLEX_OK', 1: 'RECFLEX_ERR_INVALID_ARG', 2: 'RECFLEX_ERR_CUDA', 3: 'RECFLEX_ERR_OOM',
          4: 'RECFLEX_ERR_NOT_SUPPORTED', 5: 'RECFLEX_ERR_INDEX_OOB'}

# name -> (restype, argtypes); the same names as include/recflex.h
SIGNATURES = {
    'recflex_plan_create': (c_int32, [P(FeatureSpec), c_int32, c_int32, c_int32, P(c_void_p)]),
    'recflex_destroy': (None, [c_void_p]),
    'recflex_status_string': (ctypes.c_char_p, [c_int32]),
    'recflex_last_error': (ctypes.c_char_p, []),
    'recflex_forward': (c_int32, [c_void_p, c_void_p, c_void_p, c_int32, P(c_void_p), c_void_p, c_void_p]),
    'recflex_forward_host': (c_int32, [c_void_p, c_void_p, c_int64, c_void_p, c_int32, P(c_void_p), c_void_p,
                                       c_void_p]),
    'recflex_tune': (c_int32, [c_void_p, c_int32, P(c_void_p), P(c_void_p), P(c_int32), P(c_void_p), c_void_p]),
    'recflex_tune_ex': (c_int32, [c_void_p, c_int32, P(c_void_p), P(c_void_p), P(c_int32), P(c_void_p), c_void_p,
                                  P(TuneOptions), P(TuneStats)]),
    'recflex_two_stage_select': (c_int32, [c_int32, c_int32, P(c_int32), LOCAL_COST_FN, GLOBAL_COST_FN, c_void_p,
                                           P(c_int32), P(c_int32), P(c_int64), P(c_int64)]),
    'recflex_get_schedule': (c_int32, [c_void_p, c_int32, P(Schedule), P(c_int32)]),
    'recflex_set_schedule': (c_int32, [c_void_p, c_int32, P(Schedule)]),
    'recflex_set_occupancy': (c_int32, [c_void_p, c_int32]),
    'recflex_get_occupancy': (c_int32, [c_void_p, P(c_int32)]),
    'recflex_catalog_size': (c_int32, []),
    'recflex_catalog_info': (c_int32, [c_int32, P(CatalogInfo)]),
    'recflex_catalog_valid': (c_int32, [c_int32, c_int32]),
    'recflex_catalog_valid_dtype': (c_int32, [c_int32, c_int32, c_int32]),
    'recflex_occupancy_check': (c_int32, [c_int32, c_int32, P(c_int32), P(c_int32), P(c_int32)]),
    'recflex_debug_task_map': (c_int32, [c_void_p, c_void_p, c_int32, P(c_int32), P(c_int32), c_int64, c_void_p]),
    'recflex_validate': (c_int32, [c_void_p, c_void_p, c_void_p, c_int32, c_void_p]),
    'recflex_plan_export': (c_int32, [c_void_p, ctypes.c_char_p, ctypes.c_size_t, P(ctypes.c_size_t)]),
    'recflex_plan_import': (c_int32, [c_void_p, ctypes.c_char_p]),
    'recflex_set_profiling': (c_int32, [c_void_p, c_int32]),
    'recflex_get_kernel_times': (c_int32, [c_void_p, P(ctypes.c_double), P(ctypes.c_double), P(c_int64), c_int32]),
    'recflex_shard_concat': (c_int32, [c_void_p, c_int32, c_int32, P(c_int32), c_void_p, c_void_p]),
    'recflex_l2_flush': (c_int32, [c_void_p, ctypes.c_size_t, c_void_p]),
    'recflex_forward_routed': (c_int32, [c_void_p, c_void_p, c_void_p, c_int32, P(c_void_p), P(c_void_p), c_int32,
                                         c_int32, c_int32, c_int32, c_void_p]),
    'recflex_backward': (c_int32, [c_void_p, c_void_p, c_void_p, c_int32, c_void_p, P(c_void_p), ctypes.c_float,
                                   c_void_p]),
    'recflex_ipc_get_handle': (c_int32, [c_void_p, c_void_p]),
    'recflex_ipc_open_handle': (c_int32, [c_void_p, P(c_void_p)]),
    'recflex_ipc_close': (c_int32, [c_void_p]),
    'recflex_device_alloc': (c_int32, [ctypes.c_size_t, c_int32, P(c_void_p)]),
    'recflex_device_free': (c_int32, [c_void_p]),
    'recflex_forward_host_batches': (c_int32, [c_void_p, c_int32, P(c_void_p), P(c_int64), P(c_void_p), P(c_int32),
                                               P(c_void_p), P(c_void_p), c_void_p]),
    'recflex_kjt_dist_create': (c_int32, [c_int32, P(c_int32), c_int32, c_int32, c_int32, c_int32, P(c_void_p)]),
    'recflex_kjt_dist_destroy': (None, [c_void_p]),
    'recflex_kjt_dist_sizes': (c_int32, [c_void_p, P(c_int32), P(c_int32), P(c_int32)]),
    'recflex_kjt_pack': (c_int32, [c_void_p, c_void_p, c_void_p, c_void_p, c_void_p, c_void_p, c_void_p]),
    'recflex_kjt_unpack': (c_int32, [c_void_p, c_void_p, c_void_p, c_void_p, c_void_p, c_void_p]),
    'recflex_plan_compile': (c_int32, [c_void_p, P(c_int32), c_int32]),
    'recflex_forward_exchange': (c_int32, [c_void_p, c_void_p, c_void_p, c_int32, P(c_void_p), P(Exchange),
                                           P(c_int32), c_void_p]),
    'recflex_debug_task_need': (c_int32, [c_void_p, P(c_int32)]),
    'recflex_get_task_slots': (c_int32, [c_void_p, c_int32, P(c_int32)]),
    'recflex_jit_info': (c_int32, [c_void_p, c_int32, P(JitInfo)]),
    'recflex_set_jit': (c_int32, [c_void_p, c_int32]),
    'recflex_get_jit': (c_int32, [c_void_p, P(c_int32)]),
    'recflex_select_kernel': (c_int32, [c_void_p, c_void_p, c_void_p, c_int32, P(c_void_p), c_int32,
                                        P(ctypes.c_float), P(ctypes.c_float), c_void_p]),
    'recflex_set_task_order': (c_int32, [c_void_p, P(c_int32)]),
    'recflex_select_task_size': (c_int32, [c_void_p, c_void_p, c_void_p, c_int32, P(c_void_p), c_int32,
                                           P(c_int32), P(ctypes.c_float), c_void_p]),
    'recflex_get_task_order': (c_int32, [c_void_p, P(c_int32)]),
    'recflex_set_column_order': (c_int32, [c_void_p, c_int32]),
    'recflex_get_columns': (c_int32, [c_void_p, P(c_int64)]),
    'recflex_set_l2_policy': (c_int32, [c_void_p, P(c_int32)]),
    'recflex_get_l2_policy': (c_int32, [c_void_p, P(c_int32)]),
    'recflex_l2_policy_heuristic': (c_int32, [c_void_p, c_int64, P(c_int32)]),
    'recflex_select_l2_policy': (c_int32, [c_void_p, c_void_p, c_void_p, c_int32, P(c_void_p), c_int32, c_int64,
                                           P(c_int32), P(ctypes.c_float), c_void_p]),
    'recflex_task_order_heuristic': (c_int32, [c_void_p, c_int32, P(c_int32)]),
    'recflex_select_task_order': (c_int32, [c_void_p, c_void_p, c_void_p, c_int32, P(c_void_p), c_int32,
                                            P(c_int32), P(ctypes.c_float), c_void_p]),
    'recflex_set_jit_cache_dir': (c_int32, [ctypes.c_char_p]),
    'recflex_jit_generate': (c_int32, [P(c_int32), P(c_int32), P(c_int32), P(c_int32), c_int32, c_int32,
                                       ctypes.c_char_p, ctypes.c_size_t, P(ctypes.c_size_t), P(c_int32), P(c_int32)]),
    'recflex_jit_compile_source': (c_int32, [ctypes.c_char_p, c_void_p, ctypes.c_size_t, P(ctypes.c_size_t),
                                             ctypes.c_char_p, ctypes.c_size_t, P(c_int32)]),
}


class RecflexError(RuntimeError):
    def __init__(self, code, where=''):
        self.code = code
        detail = ''
        try:
            detail = lib.recflex_last_error().decode() if code == 2 else ''
        except Exception:
            pass
        super().__init__(f'{where}: {STATUS.get(code, code)}' + (f' [{detail}]' if detail else ''))


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f'{LIB_PATH} is missing: build the CUDA library first '
                          '(python -m paper_conf_sc_panzzxwslr0d24_b200.build); there is no fallback path')
    lib = ctypes.CDLL(LIB_PATH)
    for name, (res, args) in SIGNATURES.items():
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    return lib


lib = _load()

# Compiled plan-specialised kernels (recflex_plan_compile) are cached in-tree
# next to the library unless RECFLEX_JIT_CACHE names another directory.
JIT_CACHE = os.environ.get('RECFLEX_JIT_CACHE') or os.path.join(HERE, 'jit_cache')
lib.recflex_set_jit_cache_dir(JIT_CACHE.encode())


def check(code, where=''):
    if code != OK:
        raise RecflexError(code, where)


# thin same-name wrappers -------------------------------------------------------
def __getattr__(name):
    if name in SIGNATURES:
        return getattr(lib, name)
    raise AttributeError(name)
