#!/bin/bash
# ncu launch list (every kernel with its device time) for one bench config
c=${1:-sharded1000}
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:recflex -c 40 --csv --log-file gpurun_out/launches_$c.csv python bench.py --config $c --steps 4 --warmup 3 --profile-only > gpurun_out/launches_$c.log 2>&1
echo "launches $c=$?"
