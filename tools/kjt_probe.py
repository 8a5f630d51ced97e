"""Dump a synthetic batch (KJT) for tools/kjt_probe.cu and run it.
    python tools/kjt_probe.py heavy [fixed]"""
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_panzzxwslr0d24_b200 import synth  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else 'heavy'
m = synth.make_model(cfg)
if len(sys.argv) > 2 and sys.argv[2] == 'fixed':
    feats = [synth.Feature(rows=10_000_000, dim=128, pool=0, kind='fixed', mu=100, lmax=100, table=f % 16)
             for f in range(100)]
    m = synth.custom_model('fixedL100', feats, 8192)
b = synth.make_batch(m, 7)
b.indices.tofile('/tmp/kjt_idx.bin')
b.offsets.tofile('/tmp/kjt_off.bin')
rows, dim = m.tables[0]
if os.environ.get('KJT_DUMP_ONLY'):
    sys.exit(0)
print(subprocess.run(['/tmp/kjt_probe', '/tmp/kjt_idx.bin', '/tmp/kjt_off.bin', str(m.F), str(b.B), str(rows),
                      str(len(m.tables))], capture_output=True, text=True).stdout)
