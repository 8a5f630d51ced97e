#!/bin/bash
# Tuner fidelity study (Fig. 11 analog): two-stage result vs the incoming
# (heuristic) plan, with the paper's plain stage-1 cost and the tail-aware one.
mkdir -p gpurun_out/tune_study
for c in medium industrial sharded1000; do
  ks=3,4,5,6,7,8; [ $c = sharded1000 ] && ks=3,4,5,6
  for mode in ${MODES:-plain tail isolated}; do
    extra=""; [ $mode = plain ] && extra="--no-tail"; [ $mode = isolated ] && extra="--isolated"
    timeout 1200 python tools/tune_plan.py $c --ks $ks $extra --out gpurun_out/tune_study/$mode > gpurun_out/tune_study/${c}_$mode.log 2>&1
    echo "$c $mode rc=$? $(tail -1 gpurun_out/tune_study/${c}_$mode.log | python -c 'import sys,json; l=sys.stdin.read(); d=json.loads(l[l.index("{"):]); print("two_stage", round(d["two_stage_ms"],4), "incoming", round(d["incoming_ms"],4), "ratio", round(d["incoming_ms"]/d["two_stage_ms"],3), "k", d["best_occupancy"], "s", round(d["tune_seconds"],1), "compile_s", round(d["compile_seconds"],1))' 2>/dev/null)"
  done
done
