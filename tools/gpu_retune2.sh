# Re-tune from the current plans with every stage (stage 1/2, guard, kernel, task size, order, L2)
mkdir -p gpurun_out/s3 gpurun_out/retune2
for c in industrial medium heavy; do
  timeout 1500 python tools/tune_plan.py $c --from-tuned --out gpurun_out/retune2 --ks 3,4,5,6,8 > gpurun_out/s3/retune2_$c.log 2>&1; echo tune $c=$?; tail -1 gpurun_out/s3/retune2_$c.log | cut -c1-250
  timeout 600 python tools/plan_compare.py $c configs/tuned/${c}_w1_r0.json gpurun_out/retune2/${c}_w1_r0.json | tail -3
done
