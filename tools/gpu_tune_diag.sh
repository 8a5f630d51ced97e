# Diagnosis of the plain two-stage result on industrial: is it slower than the heuristic
# in the catalog kernel too (stage 1 measures there), or only in the plan-specialised one?
mkdir -p gpurun_out/s3 gpurun_out/diag
timeout 1200 python tools/tune_plan.py industrial --no-guard --ks 4,5,6 --out gpurun_out/diag > gpurun_out/s3/diag_tune.log 2>&1; echo tune=$?
python - <<'PY'
import json
d = json.load(open('configs/tuned/industrial_w1_r0.json'))
d.pop('order', None); d.pop('columns', None)
json.dump(d, open('gpurun_out/diag/industrial_r01plan_featureorder.json', 'w'))
PY
for kern in "" "--catalog"; do
  timeout 600 python tools/plan_compare.py industrial $kern default gpurun_out/diag/industrial_w1_r0.json gpurun_out/diag/industrial_r01plan_featureorder.json
done
