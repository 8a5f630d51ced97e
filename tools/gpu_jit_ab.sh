#!/bin/bash
# JIT vs catalog-kernel A/B on the tuned plans (tools/jit_ab.py), one config at a time
nvidia-smi --query-gpu=name,clocks.sm --format=csv
for c in "industrial --ks 6,5,4,3" "medium --ks 6,4,8" "sharded1000 --ks 4,3,5,6" "heavy --ks 4,3,5" "fig3 --ks 2,4"; do
  timeout 600 python tools/jit_ab.py $c 2>&1 | tail -8
done
