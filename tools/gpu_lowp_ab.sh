#!/bin/bash
for d in bf16 f16 i8 fp8; do timeout 600 python tools/jit_ab.py heavy --dtype $d 2>&1 | grep '^{' | cut -c1-260; done
timeout 600 python tools/jit_ab.py sharded1000 --dtype bf16 2>&1 | grep '^{' | cut -c1-260
timeout 900 python bench.py --no-heavy --no-cpu-baseline > gpurun_out/r02/bench_e2e_check.json 2>&1; tail -c 1500 gpurun_out/r02/bench_e2e_check.json | grep -o '"e2e": {[^}]*}'
