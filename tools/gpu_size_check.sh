# task size (C37): test, selection (size -> order -> L2) for the w1 plans, bench
mkdir -p gpurun_out/s3 gpurun_out/tuned_sz
timeout 900 python -m pytest tests/test_gpu_task_order.py -k "task_size" -q -x > gpurun_out/s3/pytest_size.log 2>&1; echo pytest=$?; tail -2 gpurun_out/s3/pytest_size.log
rm -f gpurun_out/s3/select_size.jsonl
for c in sharded1000 industrial medium fig3 heavy; do
  timeout 900 python tools/select_order.py $c --task-size --out gpurun_out/tuned_sz >> gpurun_out/s3/select_size.jsonl 2>>gpurun_out/s3/select_size.err; echo sel $c=$?
done
cat gpurun_out/s3/select_size.jsonl
for c in sharded1000 industrial medium; do
  timeout 600 python bench.py --config $c --plan gpurun_out/tuned_sz/${c}_w1_r0.json --no-cpu-baseline --no-heavy > gpurun_out/s3/bench_${c}_sz.json 2> gpurun_out/s3/bench_${c}_sz.err
  python -c "import json; d=json.loads(open('gpurun_out/s3/bench_${c}_sz.json').read().strip().splitlines()[-1]); print('$c', round(d['ms_per_step'],4), round(d['roofline']['frac'],4), d['impl_config']['task_order'])"
done
