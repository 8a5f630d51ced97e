#!/bin/bash
# Is the stage-1 bias the kernel it measures in?  Two-stage vs incoming with stage 2 (and the
# guard) timed in the CATALOG kernel, i.e. the same kernel stage 1 co-executes candidates in.
mkdir -p gpurun_out/cat_study
for c in medium industrial; do
  timeout 1500 python tools/tune_plan.py $c --ks 3,4,5,6,7,8 --stage2-catalog --no-post --out gpurun_out/cat_study > gpurun_out/cat_study/${c}.log 2>&1
  echo "$c catalog rc=$? $(tail -1 gpurun_out/cat_study/${c}.log | python -c 'import sys,json; l=sys.stdin.read(); d=json.loads(l[l.index("{"):]); print("two_stage", round(d["two_stage_ms"],4), "incoming", round(d["incoming_ms"],4), "ratio", round(d["incoming_ms"]/d["two_stage_ms"],3), "k", d["best_occupancy"])' 2>/dev/null)"
done
