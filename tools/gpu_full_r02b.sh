# Full round-2 verification: every GPU test, smoke(), the default bench line, ncu of the headline kernel
mkdir -p gpurun_out/s3
timeout 2400 python -m pytest tests -m gpu -q --durations=15 > gpurun_out/s3/pytest_gpu_full2.log 2>&1; echo pytest=$?; tail -3 gpurun_out/s3/pytest_gpu_full2.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s3/smoke.log 2>&1; echo smoke=$?; tail -1 gpurun_out/s3/smoke.log
timeout 900 python bench.py > gpurun_out/s3/bench_final2.json 2> gpurun_out/s3/bench_final2.err; echo bench=$?
python -c "import json; d=json.loads(open('gpurun_out/s3/bench_final2.json').read().strip().splitlines()[-1]); r=d['roofline']; print(d['ms_per_step'], d['value'], r['frac'], r['fused_ms'], d['heavy']['ms_per_step'], d['heavy']['pct_of_8tbs'], d['e2e']['value'], d['clocks'])"
bash tools/ncu_r02.sh r02d sharded1000
