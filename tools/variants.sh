#!/bin/bash
# Compare library variants (lib/variants/*) on the same workload/plan.
# usage: tools/variants.sh "<bench args>" v1 v2 ...   (v = variant name or 'main')
args="$1"; shift
for v in "$@"; do
  if [ "$v" = main ]; then lib=paper_conf_sc_panzzxwslr0d24_b200/lib/librecflex.so; else lib=paper_conf_sc_panzzxwslr0d24_b200/lib/variants/$v/librecflex.so; fi
  RECFLEX_LIB=$lib timeout 600 python bench.py $args --no-e2e --no-cpu-baseline > gpurun_out/var_$v.log 2>&1
  tail -1 gpurun_out/var_$v.log | python -c "import json,sys
try:
  d=json.loads(sys.stdin.read()); r=d['roofline']; print('$v', d['config']['workload'], 'k', d['config']['occupancy'], 'ms %.3f'%d['ms_per_step'], 'fused frac %.3f'%r['frac'], 'GB/s %.0f'%r['achieved'])
except Exception as e: print('$v failed', e)"
done
