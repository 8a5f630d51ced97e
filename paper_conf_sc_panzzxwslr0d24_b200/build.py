"""Build librecflex.so (sm_100a) in-tree: nvcc for the kernels, g++ for the host
plan/tuner, linked against the static CUDA runtime so the library loads on a
machine without a GPU driver (symbols can be inspected; calls need a GPU).

    python -m paper_conf_sc_panzzxwslr0d24_b200.build [--force] [-j N]
"""
from __future__ import annotations

import argparse
import concurrent.futures as cf
import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, 'csrc')
OBJ = os.path.join(HERE, 'build_obj')
LIBDIR = os.path.join(HERE, 'lib')
LIB = os.path.join(LIBDIR, 'librecflex.so')
ROOT = os.path.dirname(HERE)
CUDA = os.environ.get('CUDA_HOME', '/usr/local/cuda')
NVCC = os.path.join(CUDA, 'bin', 'nvcc')

ARCH = ['-gencode', 'arch=compute_100a,code=sm_100a']
NVCC_FLAGS = ARCH + ['-O3', '-lineinfo', '-std=c++17', '-Xcompiler', '-fPIC,-O2', '-Xptxas', '-v',
                     '--expt-relaxed-constexpr', f'-I{ROOT}/include']
CXX_FLAGS = ['-O2', '-fPIC', '-std=c++17', '-Wall', f'-I{CUDA}/include', f'-I{ROOT}/include']


def _headers():
    return glob.glob(os.path.join(CSRC, '*.h')) + glob.glob(os.path.join(CSRC, '*.cuh')) + \
        [os.path.join(ROOT, 'include', 'recflex.h')]


def _stale(target, deps):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def _compile(src, force, objdir=OBJ, defines=()):
    os.makedirs(objdir, exist_ok=True)
    obj = os.path.join(objdir, os.path.basename(src) + '.o')
    if not force and not _stale(obj, [src] + _headers()):
        return obj, None
    if src.endswith('.cu'):
        cmd = [NVCC] + NVCC_FLAGS + [f'-D{d}' for d in defines] + ['-c', src, '-o', obj]
    else:
        cmd = ['g++'] + CXX_FLAGS + ['-c', src, '-o', obj]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f'compile failed: {" ".join(cmd)}\n{r.stdout}\n{r.stderr}')
    return obj, r.stderr


def build(force: bool = False, jobs: int = 0, verbose: bool = False, defines=(), variant: str = '') -> str:
    """Build lib/librecflex.so.  `variant` + `defines` build an experimental
    copy lib/variants/<variant>/librecflex.so (selected at run time with
    RECFLEX_LIB=<path>; development only)."""
    srcs = sorted(glob.glob(os.path.join(CSRC, '*.cu')) + glob.glob(os.path.join(CSRC, '*.cpp')))
    objdir = os.path.join(OBJ, variant) if variant else OBJ
    libdir = os.path.join(LIBDIR, 'variants', variant) if variant else LIBDIR
    lib = os.path.join(libdir, 'librecflex.so')
    jobs = jobs or min(16, os.cpu_count() or 4)
    objs = []
    logs = {}
    with cf.ThreadPoolExecutor(max_workers=jobs) as ex:
        futs = {ex.submit(_compile, s, force, objdir, tuple(defines)): s for s in srcs}
        for fu in cf.as_completed(futs):
            obj, log = fu.result()
            objs.append(obj)
            if log:
                logs[futs[fu]] = log
    os.makedirs(libdir, exist_ok=True)
    objs.sort()
    if force or _stale(lib, objs):
        tmp = lib + f'.tmp{os.getpid()}'
        cmd = [NVCC] + ARCH + ['-shared', '-cudart', 'static', '-o', tmp] + objs + ['-lpthread', '-ldl', '-lrt']
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f'link failed: {" ".join(cmd)}\n{r.stdout}\n{r.stderr}')
        os.replace(tmp, lib)
    if logs:
        with open(os.path.join(objdir, 'ptxas.log'), 'w') as fh:
            for k in sorted(logs):
                fh.write(f'== {os.path.basename(k)}\n{logs[k]}\n')
    if verbose:
        for k in sorted(logs):
            print(f'== {os.path.basename(k)}')
            print(logs[k])
    return lib


if __name__ == '__main__':
    ap = argparse.ArgumentParser()
    ap.add_argument('--force', action='store_true')
    ap.add_argument('-j', type=int, default=0)
    ap.add_argument('-v', action='store_true')
    ap.add_argument('-D', action='append', default=[], help='extra nvcc define (variant builds)')
    ap.add_argument('--variant', default='')
    a = ap.parse_args()
    print(build(a.force, a.j, a.v, a.D, a.variant))
    sys.exit(0)
