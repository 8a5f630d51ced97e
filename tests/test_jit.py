"""The plan-specialised fused kernel generator (csrc/jit.cpp; the paper's fusion
compiler, §IV-B) on the CPU: NVRTC cross-compiles for sm_100a without a
GPU, so the generated source, its variant numbering and the compiled cubin are
checked here; launching it is covered by the -m gpu tests."""
import re

import pytest

from paper_conf_sc_panzzxwslr0d24_b200 import plan as P
from paper_conf_sc_panzzxwslr0d24_b200._lib import JIT_CACHE, check, lib


def _ids():
    cat = P.catalog()

    def find(family, G, VEC, C, U, dtype='f32'):
        for e in cat:
            if (e['family'], e['G'], e['VEC'], e['C'], e['U'], e['dtype']) == (family, G, VEC, C, U, dtype):
                return e['id']
        raise KeyError((family, G, VEC, C, U, dtype))
    return find


def test_generate_one_branch_per_variant():
    find = _ids()
    g32 = find('group', 32, 4, 1, 4)
    g2 = find('group', 2, 4, 1, 4)
    blk = find('block', 16, 8, 1, 4)
    # features: (entry, dim, pool); features 0 and 3 share a variant
    sched = [g32, g2, blk, g32, g32]
    dims = [128, 8, 128, 128, 128]
    pools = [0, 1, 0, 0, 1]
    src, var, nv = P.jit_generate(sched, dims, pools, 4)
    assert nv == 4
    assert var == [0, 1, 2, 0, 3]
    assert src.count('jit_dispatch') == 1 or 'jit_dispatch(int v' in src
    # one literal-argument call per variant, d / pool / row pitch compiled in
    assert len(re.findall(r'sched_(group|block|flat)<', src)) == 4
    assert 'sched_group<0, 32, 4, 1, 4>(x.table, 512u, 32, x.offs, x.idx, x.out, 128, 0,' in src
    assert 'sched_group<0, 2, 4, 1, 4>(x.table, 32u, 2, x.offs, x.idx, x.out, 8, 1,' in src
    assert 'return false || v == 2;' in src          # the BLOCK-family variant is CTA-synchronous
    assert '__launch_bounds__(recflex::kBlockThreads, 4) recflex_fused_jit_k4' in src
    assert '#define RECFLEX_JIT_STATIC 0' in src


def test_generate_rejects_invalid_entry():
    find = _ids()
    with pytest.raises(Exception):
        P.jit_generate([find('group', 32, 8, 1, 4)], [12], [0], 4)   # 8 floats per lane do not divide d = 12
    with pytest.raises(Exception):
        P.jit_generate([find('group', 4, 4, 1, 4)], [16], [0], 9)    # k outside 1..8


def test_compiles_for_sm100a_without_spills_at_k4(tmp_path):
    """A heavy-like plan (one GROUP G32 V4 U4 variant, d = 128) compiles with NVRTC
    for sm_100a and keeps everything in registers at the k = 4 cap (64 registers)."""
    find = _ids()
    src, _, _ = P.jit_generate([find('group', 32, 4, 1, 4)] * 3, [128] * 3, [0, 0, 0], 4)
    # an empty cache directory: a cache hit would return the cubin without the ptxas log
    check(lib.recflex_set_jit_cache_dir(str(tmp_path).encode()), 'recflex_set_jit_cache_dir')
    try:
        cubin, log, hit = P.jit_compile_source(src)
    finally:
        check(lib.recflex_set_jit_cache_dir(JIT_CACHE.encode()), 'recflex_set_jit_cache_dir')
    assert not hit
    assert cubin[:4] == b'\x7fELF'
    m = re.search(r'(\d+) bytes spill stores, (\d+) bytes spill loads', log)
    assert m and m.group(1) == '0' and m.group(2) == '0', log
    assert 'sm_100a' in log


def test_cache_hit_on_second_compile(tmp_path):
    find = _ids()
    P._lib.lib.recflex_set_jit_cache_dir(str(tmp_path).encode())
    try:
        src, _, _ = P.jit_generate([find('group', 8, 4, 1, 2)], [32], [1], 6)
        c1, _, hit1 = P.jit_compile_source(src)
        c2, _, hit2 = P.jit_compile_source(src)
        assert not hit1 and hit2 and c1 == c2
        assert len(list(tmp_path.glob('rfx_*.cubin'))) == 1
    finally:
        P._lib.lib.recflex_set_jit_cache_dir(P._lib.JIT_CACHE.encode())
