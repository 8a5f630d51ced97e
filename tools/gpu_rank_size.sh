# task size (C37) + order + L2 re-selection for the W = 2/4/8 rank plans, then rank_sim
mkdir -p gpurun_out/s3 gpurun_out/tuned_rsz
rm -f gpurun_out/s3/select_size_ranks.jsonl
for W in 2 4 8; do timeout 1500 python tools/select_order.py sharded1000 --world $W --task-size --out gpurun_out/tuned_rsz >> gpurun_out/s3/select_size_ranks.jsonl 2>>gpurun_out/s3/select_size_ranks.err; echo sel W$W=$?; done
timeout 1200 python tools/rank_sim.py sharded1000 --worlds 2,4,8 --tuned-dir gpurun_out/tuned_rsz > gpurun_out/s3/rank_sim_sz.jsonl 2> gpurun_out/s3/rank_sim_sz.err; echo ranksim=$?
python -c "
import json
for l in open('gpurun_out/s3/rank_sim_sz.jsonl'):
    d=json.loads(l); print(d['world'], round(d['compute_ms_max'],4), round(d['compute_ms_min'],4), round(d['samples_per_s_serial']/1e6,2), round(d['samples_per_s_overlapped']/1e6,2))
"
