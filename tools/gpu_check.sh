#!/bin/bash
mkdir -p gpurun_out/r02
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r02/bench_default2.json 2> gpurun_out/r02/bench_default2.err; echo "bench=$?"
for d in bf16 i8; do timeout 600 python bench.py --config heavy --dtype $d --no-heavy --no-cpu-baseline > gpurun_out/r02/bench_heavy_${d}2.json 2>&1; echo "bench $d=$?"; done
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "export or graph or exchange" 2>&1 | tail -2
