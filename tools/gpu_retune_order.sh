# Re-tune sharded1000 / industrial starting from the order-selected plans (stage 2 runs
# under their task order and column layout; the guard keeps them if nothing is faster).
mkdir -p gpurun_out/s3 gpurun_out/retune
for c in sharded1000 industrial; do
  timeout 1200 python tools/tune_plan.py $c --from-tuned --out gpurun_out/retune --ks 2,3,4,5,6 > gpurun_out/s3/retune_$c.log 2>&1; echo tune $c=$?; tail -1 gpurun_out/s3/retune_$c.log | cut -c1-400
  timeout 600 python tools/plan_compare.py $c configs/tuned/${c}_w1_r0.json gpurun_out/retune/${c}_w1_r0.json
done
