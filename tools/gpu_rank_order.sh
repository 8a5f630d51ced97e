# Task order + task-order columns (C35) for the W = 2/4/8 rank plans, then the per-rank
# device times of rank_sim with the selected plans vs the current ones.
mkdir -p gpurun_out/s3 gpurun_out/tuned_cols
for W in 2 4 8; do timeout 900 python tools/select_order.py sharded1000 --world $W --columns task-order --out gpurun_out/tuned_cols >> gpurun_out/s3/select_order_ranks.jsonl 2>>gpurun_out/s3/select_order_ranks.err; echo sel W$W=$?; done
cp configs/tuned/sharded1000_w*_parts.json gpurun_out/tuned_cols/
timeout 1200 python tools/rank_sim.py sharded1000 --worlds 2,4,8 --tuned-dir gpurun_out/tuned_cols > gpurun_out/s3/rank_sim_cols.jsonl 2> gpurun_out/s3/rank_sim_cols.err; echo ranksim=$?
cat gpurun_out/s3/select_order_ranks.jsonl; cat gpurun_out/s3/rank_sim_cols.jsonl
