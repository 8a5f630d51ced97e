#!/bin/bash
# Retune + bench the reduced-precision plans and time the backward (after kernel changes).
set -u
mkdir -p gpurun_out/tuned
for cd in heavy:bf16 heavy:f16 heavy:i8 sharded1000:bf16; do
  c=${cd%%:*}; d=${cd##*:}
  timeout 900 python tools/tune_plan.py $c --dtype $d --ks 3,4,5,6,8 > gpurun_out/tune_${c}_$d.log 2>&1; echo "tune $c $d=$?"
  cp gpurun_out/tuned/${c}_${d}_w1_r0.json configs/tuned/ 2>/dev/null
done
bash tools/bench_lines.sh heavy:bf16 heavy:f16 heavy:i8 sharded1000:bf16
for c in heavy sharded1000; do timeout 600 python tools/bench_backward.py $c > gpurun_out/bwd_$c.log 2>&1; echo "bwd $c=$?"; tail -1 gpurun_out/bwd_$c.log; done
