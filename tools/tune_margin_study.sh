#!/bin/bash
# Stage-1 switch margin (reading C38): two-stage result vs the incoming heuristic plan
# (both from stage 2 on the tuning batches; guard on so incoming_ms is measured)
mkdir -p gpurun_out/margin_study
for c in medium industrial sharded1000; do
  ks=3,4,5,6,7,8; [ $c = sharded1000 ] && ks=3,4,5,6
  for m in ${MARGINS:-0 0.03 0.08}; do
    timeout 1500 python tools/tune_plan.py $c --ks $ks --margin $m --no-post $EXTRA --out gpurun_out/margin_study/m$m > gpurun_out/margin_study/${c}_m$m.log 2>&1
    echo "$c margin=$m $EXTRA rc=$? $(tail -1 gpurun_out/margin_study/${c}_m$m.log | python -c 'import sys,json; l=sys.stdin.read(); d=json.loads(l[l.index("{"):]); print("two_stage", round(d["two_stage_ms"],4), "incoming", round(d["incoming_ms"],4), "ratio", round(d["incoming_ms"]/d["two_stage_ms"],3), "k", d["best_occupancy"], "s", round(d["tune_seconds"],1))' 2>/dev/null)"
  done
done
