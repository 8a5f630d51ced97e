#!/bin/bash
# ncu evidence for the round-2 kernel (plan-specialised fused kernel):
#   tools/ncu_r02.sh <tag> <config> [<config> ...]
# per config: one `ncu --set full` capture of the fused kernel (3rd launch) and a
# launch list (gpu__time_duration of every recflex kernel of a short bench run)
tag=$1; shift
mkdir -p gpurun_out
for c in "$@"; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:recflex_fused -s 2 -c 1 \
      -o gpurun_out/prof_${tag}_$c -f python bench.py --config $c --steps 2 --warmup 1 --profile-only \
      > gpurun_out/ncu_${tag}_$c.log 2>&1
  echo "ncu $c=$?"
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:recflex -c 40 --csv \
      --log-file gpurun_out/launches_${tag}_$c.csv python bench.py --config $c --steps 4 --warmup 3 --profile-only \
      > gpurun_out/launches_${tag}_$c.log 2>&1
  echo "launches $c=$?"
done
