# L2 policy (C36): tests, selection for the w1 plans (order kept), bench
mkdir -p gpurun_out/s3 gpurun_out/tuned_l2
timeout 1200 python -m pytest tests/test_gpu_l2_policy.py tests/test_gpu_parity.py -k "l2 or policy or tuner_runs or export" -q -x > gpurun_out/s3/pytest_l2.log 2>&1; echo pytest=$?; tail -3 gpurun_out/s3/pytest_l2.log
rm -f gpurun_out/s3/select_l2.jsonl
for c in sharded1000 industrial heavy medium; do
  timeout 900 python tools/select_order.py $c --out gpurun_out/tuned_l2 >> gpurun_out/s3/select_l2.jsonl 2>>gpurun_out/s3/select_l2.err; echo sel $c=$?
done
cat gpurun_out/s3/select_l2.jsonl
for c in sharded1000 industrial; do
  timeout 600 python bench.py --config $c --plan gpurun_out/tuned_l2/${c}_w1_r0.json --no-cpu-baseline --no-heavy > gpurun_out/s3/bench_${c}_l2.json 2> gpurun_out/s3/bench_${c}_l2.err
  python -c "import json; d=json.loads(open('gpurun_out/s3/bench_${c}_l2.json').read().strip().splitlines()[-1]); print('$c', round(d['ms_per_step'],4), round(d['roofline']['frac'],4), d['impl_config']['task_order'])"
done
