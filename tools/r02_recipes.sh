#!/bin/bash
# GPU recipes behind the round-2 task-order / L2 / task-size measurements
# (profiles/r02_task_order.md).  Run one step on a B200 with
#   gpurun -- 'bash tools/r02_recipes.sh <step>'
# Every step writes under gpurun_out/ (scratch); the numbers that count were copied
# into profiles/ and configs/tuned/.
set -u
step=${1:-help}
mkdir -p gpurun_out/s3
case $step in
  order-probe)    # layout vs claim order grid, + the ncu DRAM bytes of four of its runs
    for c in sharded1000 industrial; do timeout 600 python tools/order_probe.py $c; done
    M=dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_write_lookup_miss.sum
    for run in model layout_model+order_lpt layout_lpt+order_lpt layout_lpt+order_model; do
      ORDER_PROBE_ONLY=$run ORDER_PROBE_REPS=2 timeout 600 ncu --metrics $M --clock-control none -k regex:recflex_fused \
        -s 1 -c 1 --csv python tools/order_probe.py sharded1000 > gpurun_out/s3/ncu_order_$run.csv 2>&1
    done ;;
  l2-probe)       # per-feature L2 eviction priorities (reading C36)
    for c in sharded1000 industrial; do
      timeout 600 python tools/l2_probe.py $c --variants none,heuristic,first_only,last_only,all_first,all_last,l1_1mb,l1_4mb
    done ;;
  size-probe)     # task granularity (reading C37)
    timeout 900 python tools/task_size_probe.py sharded1000 --factors 1,2,4,8,16 --which reuse,all ;;
  select)         # task size -> order -> L2 selections for the 1-GPU plans (written to gpurun_out/tuned_sel)
    for c in sharded1000 industrial medium fig3 heavy; do
      timeout 900 python tools/select_order.py $c --task-size --out gpurun_out/tuned_sel
    done ;;
  select-ranks)   # the same for the W = 2/4/8 rank plans, then rank_sim on them
    for W in 2 4 8; do timeout 1500 python tools/select_order.py sharded1000 --world $W --task-size --out gpurun_out/tuned_sel; done
    cp configs/tuned/sharded1000_w*_parts.json gpurun_out/tuned_sel/
    timeout 1200 python tools/rank_sim.py sharded1000 --worlds 2,4,8 --tuned-dir gpurun_out/tuned_sel ;;
  rebalance)      # measured partition refinement on the plan-specialised kernel, then rank_sim
    for W in 2 4 8; do
      timeout 2400 python tools/rebalance.py sharded1000 --world $W --moves 8 --reps 8 --out gpurun_out/rebal$W
      timeout 1200 python tools/rank_sim.py sharded1000 --worlds $W --tuned-dir gpurun_out/rebal$W
    done ;;
  retune)         # re-tune from the shipped plans with every stage; compare on held-out timing
    for c in sharded1000 industrial medium heavy; do
      timeout 1500 python tools/tune_plan.py $c --from-tuned --out gpurun_out/retune
      timeout 600 python tools/plan_compare.py $c configs/tuned/${c}_w1_r0.json gpurun_out/retune/${c}_w1_r0.json
    done ;;
  verify)         # every GPU test, smoke(), the default bench line, ncu of the headline kernel
    timeout 2400 python -m pytest tests -m gpu -q --durations=15
    timeout 300 python -c "import __graft_entry__ as g; g.smoke()"
    timeout 900 python bench.py
    bash tools/ncu_r02.sh r02d sharded1000 ;;
  bench-all)      # one bench line per config / row type
    for spec in "industrial" "medium" "fig3" "heavy" "heavy --dtype bf16" "heavy --dtype f16" "heavy --dtype fp8" \
                "heavy --dtype i8" "sharded1000 --dtype bf16"; do
      timeout 900 python bench.py --config $spec --no-heavy --no-cpu-baseline | tail -1
    done ;;
  tuner-studies)  # stage-1 switch margin (C38), position balance (C39), catalog-kernel stage 2
    MARGINS="0 0.03 0.08" bash tools/tune_margin_study.sh
    MARGINS=0 EXTRA=--balance bash tools/tune_margin_study.sh
    bash tools/tune_catalog_study.sh ;;
  *) sed -n 2,6p "$0"; echo "steps: order-probe l2-probe size-probe select select-ranks rebalance retune verify bench-all tuner-studies" ;;
esac
