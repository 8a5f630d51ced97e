#!/bin/bash
# Re-tune the single-GPU plans with the round-2 tuner (tail-aware stage 1,
# stage 2 + guard on the plan-specialised kernel); outputs gpurun_out/tuned_r02b/
mkdir -p gpurun_out/tuned_r02b
for c in medium fig3 industrial sharded1000 heavy; do
  ks=3,4,5,6,7,8; [ $c = heavy ] && ks=3,4,5,6; [ $c = sharded1000 ] && ks=3,4,5,6
  timeout 1500 python tools/tune_plan.py $c --ks $ks --out gpurun_out/tuned_r02b > gpurun_out/tuned_r02b/$c.out 2>&1
  echo "$c rc=$? $(tail -1 gpurun_out/tuned_r02b/$c.out | cut -c1-400)"
done
