# measured partition refinement on the plan-specialised kernel (W = 8), then rank_sim of the result
mkdir -p gpurun_out/s3 gpurun_out/rebal8
timeout 2400 python tools/rebalance.py sharded1000 --world 8 --moves 8 --reps 8 --out gpurun_out/rebal8 > gpurun_out/s3/rebalance_w8.log 2>&1; echo rebalance=$?; tail -2 gpurun_out/s3/rebalance_w8.log | cut -c1-300
timeout 1200 python tools/rank_sim.py sharded1000 --worlds 8 --tuned-dir gpurun_out/rebal8 > gpurun_out/s3/rank_sim_rebal8.jsonl 2> gpurun_out/s3/rank_sim_rebal8.err; echo ranksim=$?
python -c "
import json
for l in open('gpurun_out/s3/rank_sim_rebal8.jsonl'):
    d=json.loads(l); print(d['world'], round(d['compute_ms_max'],4), round(d['compute_ms_min'],4), round(d['samples_per_s_serial']/1e6,2), round(d['samples_per_s_overlapped']/1e6,2), [round(x['ms'],3) for x in d['ranks']])
"
