# fill-kernel rewrite: parity of the task map / part-1 paths, bench, launch list, ncu of the fused kernel
mkdir -p gpurun_out/s3
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_task_order.py tests/test_gpu_tuned_plans.py -k "task_map or part1 or order or sharded1000 or fine_grained or tuner" -q -x > gpurun_out/s3/pytest_fill.log 2>&1; echo pytest=$?; tail -2 gpurun_out/s3/pytest_fill.log
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/s3/bench_fill.json 2> gpurun_out/s3/bench_fill.err; echo bench=$?
python -c "import json; d=json.loads(open('gpurun_out/s3/bench_fill.json').read().strip().splitlines()[-1]); r=d['roofline']; print(d['ms_per_step'], r['frac'], r['fused_ms'], r['map_ms'], d['heavy']['ms_per_step'])"
bash tools/ncu_r02.sh r02b sharded1000
grep -o '"recflex[^"]*","1","[0-9]*","([0-9, ]*)","([0-9, ]*)".*"ns","[0-9.]*"' gpurun_out/launches_r02b_sharded1000.csv | head -6 | awk -F'","' '{print $1, $NF}'
