# Final bench lines of every config (one GPU, default flags)
mkdir -p gpurun_out/s3/final
for spec in "industrial" "medium" "fig3" "heavy" "heavy --dtype bf16" "heavy --dtype f16" "heavy --dtype fp8" "heavy --dtype i8" "sharded1000 --dtype bf16"; do
  tag=$(echo $spec | tr ' ' '_' | sed 's/--dtype_//')
  timeout 900 python bench.py --config $spec --no-heavy --no-cpu-baseline > gpurun_out/s3/final/bench_$tag.json 2> gpurun_out/s3/final/bench_$tag.err
  python -c "import json; d=json.loads(open('gpurun_out/s3/final/bench_$tag.json').read().strip().splitlines()[-1]); r=d['roofline']; print('$tag', round(d['ms_per_step'],4), round(d['value']/1e6,3), round(d['effective_hbm_gbs']), round(d['pct_of_8tbs'],1), round(r['frac'],3), d['impl_config'].get('task_order'), d['impl_config']['kernel'][:20], d['clocks']['reasons'])"
done
