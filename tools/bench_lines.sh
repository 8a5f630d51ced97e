#!/bin/bash
# bench lines for a list of "config:dtype" pairs -> gpurun_out/bench_<config>_<dtype>.log + a summary line each
set -u
mkdir -p gpurun_out
for cd in "$@"; do
  c=${cd%%:*}; d=${cd##*:}
  timeout 900 python bench.py --config $c --dtype $d --steps 20 --warmup 5 > gpurun_out/bench_${c}_${d}.log 2>&1
  echo "bench $c $d rc=$?"
  tail -1 gpurun_out/bench_${c}_${d}.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print(d['config']['workload'], d['config']['table_dtype'], 'samples/s %.4g'%d['value'], 'ms %.3f'%d['ms_per_step'], 'eff GB/s %.0f'%d['effective_hbm_gbs'], 'fused frac %.3f'%r['frac'], 'k', d['config']['occupancy'], 'clk', d['clocks'])" 2>&1 | tail -1
done
