#!/bin/bash
for d in bf16 f16 i8 fp8; do timeout 600 python tools/jit_ab.py heavy --dtype $d 2>&1 | grep '^{' | cut -c1-200; done
timeout 600 python tools/jit_ab.py sharded1000 --dtype bf16 2>&1 | grep '^{' | cut -c1-200
timeout 900 python tools/latency_probe.py medium --onehot --base tuned --families group,flat --vs 8,4 --us 2 --spbs 16,32,64,128,256 --ks 4 --no-tuned 2>&1 | grep '^{'
