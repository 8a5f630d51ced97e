# L2 policy (C36) + order re-selection for the W = 2/4/8 rank plans, then rank_sim
mkdir -p gpurun_out/s3 gpurun_out/tuned_rl2
rm -f gpurun_out/s3/select_l2_ranks.jsonl
for W in 2 4 8; do timeout 1200 python tools/select_order.py sharded1000 --world $W --out gpurun_out/tuned_rl2 >> gpurun_out/s3/select_l2_ranks.jsonl 2>>gpurun_out/s3/select_l2_ranks.err; echo sel W$W=$?; done
timeout 1200 python tools/rank_sim.py sharded1000 --worlds 2,4,8 --tuned-dir gpurun_out/tuned_rl2 > gpurun_out/s3/rank_sim_l2.jsonl 2> gpurun_out/s3/rank_sim_l2.err; echo ranksim=$?
python -c "
import json
for l in open('gpurun_out/s3/rank_sim_l2.jsonl'):
    d=json.loads(l); print(d['world'], round(d['compute_ms_max'],4), round(d['compute_ms_min'],4), round(d['samples_per_s_serial']/1e6,2), round(d['samples_per_s_overlapped']/1e6,2))
"
