#!/bin/bash
# round-2 measurement pass: bench lines, ncu evidence, ablations
mkdir -p gpurun_out/r02
timeout 900 python bench.py > gpurun_out/r02/bench_default.json 2> gpurun_out/r02/bench_default.err; echo "bench default=$?"
for c in industrial medium fig3 heavy; do
  timeout 600 python bench.py --config $c --no-heavy > gpurun_out/r02/bench_$c.json 2> gpurun_out/r02/bench_$c.err; echo "bench $c=$?"
done
for d in bf16 f16 fp8 i8; do
  timeout 600 python bench.py --config heavy --dtype $d --no-heavy --no-cpu-baseline > gpurun_out/r02/bench_heavy_$d.json 2> gpurun_out/r02/bench_heavy_$d.err; echo "bench heavy $d=$?"
done
bash tools/ncu_r02.sh r02 industrial sharded1000 heavy medium
for a in "mapping --config industrial" "mapping --config sharded1000" "tuning --config medium" "tuning --config industrial" "swap --config sharded1000"; do
  set -- $a
  timeout 1500 python tools/ablations.py $a --out gpurun_out/r02/ablation_$1_$3.md > gpurun_out/r02/ablation_$1_$3.log 2>&1; echo "ablation $a=$?"
done
