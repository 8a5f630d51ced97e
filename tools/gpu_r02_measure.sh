#!/bin/bash
# round-2 measurement pass: bench line, ncu evidence, tuner study
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/bench_r02b.json 2> gpurun_out/bench_r02b.err; echo "bench=$?"
bash tools/ncu_r02.sh r02 industrial sharded1000 heavy medium
for c in medium industrial; do
  timeout 900 python tools/tune_plan.py $c --ks 3,4,5,6,7,8 --out gpurun_out/tuned_r02 > gpurun_out/tune_r02_$c.log 2>&1; echo "tune $c=$?"
done
