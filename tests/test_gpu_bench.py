"""bench.py's GPU arm end to end (small workload): the N = 1 line and the N = 2
line (torchrun, 2 ranks sharing cuda:0 over gloo -- test plumbing; the driver
runs N > 1 over NCCL on N GPUs) carry the contract's keys, the roofline of the
plan-specialised kernel, and at N > 1 the compute / exchange split with the
NVLink all-to-all bounds."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _line(stdout):
    lines = [ln for ln in stdout.splitlines() if ln.startswith('{')]
    assert len(lines) == 1, stdout[-3000:]
    return json.loads(lines[0])


def _port():
    s = socket.socket()
    s.bind(('127.0.0.1', 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_bench_n1_line():
    r = subprocess.run([sys.executable, os.path.join(ROOT, 'bench.py'), '--config', 'medium', '--steps', '5',
                        '--warmup', '3', '--no-heavy', '--cpu-seconds', '0.5', '--cpu-samples', '64'],
                       capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    d = _line(r.stdout)
    for k in ('metric', 'value', 'unit', 'n_gpus', 'steps', 'warmup', 'ms_per_step', 'higher_is_better', 'scaling',
              'dtype', 'config', 'roofline', 'e2e', 'gpu_launches', 'clocks', 'cpu_baseline'):
        assert k in d, k
    assert d['n_gpus'] == 1 and d['steps'] == 5 and d['value'] > 0 and d['scaling'] == 'strong'
    assert d['roofline']['kernel'].startswith('recflex_fused_jit_k')
    assert 0 < d['roofline']['frac'] and d['roofline']['peak'] > 0
    assert d['cpu_baseline']['cpu_model'] and d['cpu_baseline']['cores'] >= 1
    assert d['e2e']['h2d_bytes_per_step'] > 0 and d['e2e']['d2h_bytes_per_step'] > 0


@pytest.mark.parametrize('exchange', ['nccl', 'fused'])
def test_bench_two_ranks_one_gpu_line(exchange):
    env = dict(os.environ, RECFLEX_DIST_BACKEND='gloo', RECFLEX_BENCH_DEVICE='0')
    cmd = [sys.executable, '-m', 'torch.distributed.run', '--nnodes=1', '--nproc-per-node', '2', '--master-addr',
           '127.0.0.1', '--master-port', str(_port()), os.path.join(ROOT, 'bench.py'), '--gpus', '2', '--config',
           'medium', '--steps', '4', '--warmup', '3', '--exchange', exchange, '--no-e2e']
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    d = _line(r.stdout)
    assert d['n_gpus'] == 2 and d['config']['parallelism'] == 'tablewise2'
    mg = d['multi_gpu']
    for k in ('compute_ms_max_rank', 'step_ms_max_rank', 'exchange_ms_max_rank', 'nvlink'):
        assert k in mg, k
    nv = mg['nvlink']
    assert nv['a2a_bytes_max_rank'] > 0 and nv['serial_bound_ms'] >= nv['overlapped_bound_ms'] > 0
    assert d['roofline']['traffic'] is None or d['roofline']['traffic_source'].endswith('_w2_r0.json')
