mkdir -p gpurun_out/s3
timeout 1500 python -m pytest tests/test_gpu_task_order.py tests/test_gpu_tuned_plans.py tests/test_gpu_bench.py tests/test_gpu_parity.py -k "order or tuned or bench or full_size or rank_plans or export or tuner" -q -x > gpurun_out/s3/pytest_check_order.log 2>&1; echo pytest=$?; tail -3 gpurun_out/s3/pytest_check_order.log
timeout 900 python bench.py > gpurun_out/s3/bench_default_order.json 2> gpurun_out/s3/bench_default_order.err; echo bench=$?
python -c "import json; d=json.loads(open('gpurun_out/s3/bench_default_order.json').read().strip().splitlines()[-1]); print(d['ms_per_step'], d['roofline']['frac'], d['impl_config']['task_order'], d['heavy']['ms_per_step'], d['e2e']['value'])"
