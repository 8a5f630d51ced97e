# Task order / column layout (reading C35): parity tests, order selection for
# the tuned plans under both column layouts, bench lines with the selected plans.
mkdir -p gpurun_out/s3 gpurun_out/tuned gpurun_out/tuned_cols
timeout 1200 python -m pytest tests/test_gpu_task_order.py -q -x > gpurun_out/s3/pytest_order.log 2>&1; echo pytest=$?; tail -3 gpurun_out/s3/pytest_order.log
rm -f gpurun_out/s3/select_order.jsonl
for c in sharded1000 industrial medium fig3; do
  timeout 600 python tools/select_order.py $c --columns feature >> gpurun_out/s3/select_order.jsonl 2>>gpurun_out/s3/select_order.err; echo sel $c=$?
  timeout 600 python tools/select_order.py $c --columns task-order --out gpurun_out/tuned_cols >> gpurun_out/s3/select_order.jsonl 2>>gpurun_out/s3/select_order.err; echo selcols $c=$?
done
cat gpurun_out/s3/select_order.jsonl
for c in sharded1000 industrial medium; do
  for v in tuned tuned_cols; do
    timeout 600 python bench.py --config $c --plan gpurun_out/$v/${c}_w1_r0.json --no-cpu-baseline --no-heavy > gpurun_out/s3/bench_${c}_$v.json 2> gpurun_out/s3/bench_${c}_$v.err
    python -c "import json,sys; d=json.loads(open('gpurun_out/s3/bench_${c}_$v.json').read().strip().splitlines()[-1]); print('$c $v', round(d['ms_per_step'],4), round(d['roofline']['frac'],4), d['impl_config']['task_order'], d['impl_config']['output_columns'][:10])"
  done
done
