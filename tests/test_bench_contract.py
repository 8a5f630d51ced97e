"""bench.py's driver contract on CPU: the reference arm (--impl reference, the
CPU oracle timed on the host) prints one JSON line with the required keys and
the same metric / unit / config as the GPU arm."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(*args):
    r = subprocess.run([sys.executable, os.path.join(ROOT, 'bench.py'), *args], capture_output=True, text=True,
                       timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith('{')]
    assert len(lines) == 1, r.stdout
    return json.loads(lines[0])


def test_reference_arm_json_line():
    d = _run('--impl', 'reference', '--config', 'tiny', '--steps', '2', '--warmup', '1', '--ref-samples', '32')
    for k in ('impl', 'metric', 'value', 'unit', 'n_gpus', 'steps', 'warmup', 'ms_per_step', 'higher_is_better',
              'scaling', 'vs_baseline', 'dtype', 'data', 'config', 'cpu_baseline', 'e2e'):
        assert k in d, k
    assert d['impl'] == 'reference' and d['unit'] == 'samples/s' and d['higher_is_better'] is True
    assert d['steps'] == 2 and d['warmup'] == 1 and d['n_gpus'] == 1 and d['value'] > 0
    assert d['config']['workload'] == 'tiny'
    with open(os.path.join(ROOT, 'BASELINE.json')) as fh:
        assert d['metric'] == json.load(fh)['metric']
    cb = d['cpu_baseline']
    assert cb['kind'] == 'oracle' and cb['cores'] >= 1 and cb['value'] == d['value'] and cb['sample']
    assert d['e2e']['h2d_bytes_per_step'] == 0 and d['e2e']['d2h_bytes_per_step'] == 0
    assert d['e2e']['value'] == d['value'] and d['e2e']['unit'] == d['unit']


def _free_port():
    import socket
    s = socket.socket()
    s.bind(('127.0.0.1', 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_reference_arm_under_torchrun_two_ranks():
    """N > 1 launch (torchrun, 2 ranks, gloo on CPU): rank 0 alone prints one line
    with n_gpus = 2 and the same workload config the GPU arm prints; rank 1 exits 0."""
    cmd = [sys.executable, '-m', 'torch.distributed.run', '--nnodes=1', '--nproc-per-node', '2',
           '--master-addr', '127.0.0.1', '--master-port', str(_free_port()), os.path.join(ROOT, 'bench.py'),
           '--impl', 'reference', '--gpus', '2', '--config', 'tiny', '--steps', '2', '--warmup', '1',
           '--ref-samples', '16']
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith('{')]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d['n_gpus'] == 2 and d['impl'] == 'reference'
    assert d['config']['parallelism'] == 'tablewise2'
    sys.path.insert(0, ROOT)
    import argparse

    import bench
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    args = argparse.Namespace(config='tiny', dtype='f32', batches=3)
    assert d['config'] == bench._workload_config(args, synth.make_model('tiny'), 2)
    assert d['scaling'] == 'strong'
