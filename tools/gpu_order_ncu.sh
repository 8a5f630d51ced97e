mkdir -p gpurun_out/s3
M=dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_write_lookup_miss.sum
for run in model layout_model+order_lpt layout_lpt+order_lpt layout_lpt+order_model; do
  ORDER_PROBE_ONLY=$run ORDER_PROBE_REPS=2 timeout 600 ncu --metrics $M --clock-control none -k regex:recflex_fused -s 1 -c 1 --csv python tools/order_probe.py sharded1000 > gpurun_out/s3/ncu_order_$run.csv 2>&1; echo $run=$?
done
