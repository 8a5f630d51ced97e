#!/bin/bash
# One GPU measurement round: parity tests, (re)tune, bench, optional ncu.
# usage: tools/round.sh [tests] [tune] [bench] [ncu]
set -u
mkdir -p gpurun_out configs/tuned
for what in "$@"; do
  case $what in
    tests) timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest=$?"; tail -4 gpurun_out/pytest_gpu.log ;;
    tune) for c in sharded1000 heavy; do timeout 900 python tools/tune_plan.py $c --ks 2,3,4,5,6,8 > gpurun_out/tune_$c.log 2>&1; echo "tune $c=$?"; tail -1 gpurun_out/tune_$c.log | cut -c1-300; cp gpurun_out/tuned/${c}_w1_r0.json configs/tuned/ 2>/dev/null; done ;;
    bench) for c in sharded1000 heavy; do timeout 900 python bench.py --config $c --steps 20 --warmup 5 > gpurun_out/bench_$c.log 2>&1; echo "bench $c=$?"; tail -1 gpurun_out/bench_$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print(d['config']['workload'], 'samples/s %.3g'%d['value'], 'ms %.3f'%d['ms_per_step'], 'eff GB/s %.0f'%d['effective_hbm_gbs'], 'fused frac %.3f'%r['frac'], 'k', d['config']['occupancy'], 'clk', d['clocks'])"; done ;;
    ncu) for c in sharded1000 heavy; do timeout 900 ncu --set full --clock-control none --import-source on -k regex:recflex_fused -s 2 -c 1 -o gpurun_out/prof_$c -f python bench.py --config $c --steps 2 --warmup 1 --profile-only > gpurun_out/ncu_$c.log 2>&1; echo "ncu $c=$?"; done ;;
  esac
done
