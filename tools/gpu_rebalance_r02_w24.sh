for W in 2 4; do
mkdir -p gpurun_out/s3 gpurun_out/rebal$W
timeout 2400 python tools/rebalance.py sharded1000 --world $W --moves 8 --reps 8 --out gpurun_out/rebal$W > gpurun_out/s3/rebalance_w$W.log 2>&1; echo rebalance=$?; tail -2 gpurun_out/s3/rebalance_w8.log | cut -c1-300
timeout 1200 python tools/rank_sim.py sharded1000 --worlds $W --tuned-dir gpurun_out/rebal$W > gpurun_out/s3/rank_sim_rebal$W.jsonl 2> gpurun_out/s3/rank_sim_rebal$W.err; echo ranksim=$?
python -c "
import json
for l in open('gpurun_out/s3/rank_sim_rebal$W.jsonl'):
    d=json.loads(l); print(d['world'], round(d['compute_ms_max'],4), round(d['compute_ms_min'],4), round(d['samples_per_s_serial']/1e6,2), round(d['samples_per_s_overlapped']/1e6,2), [round(x['ms'],3) for x in d['ranks']])
"
done
