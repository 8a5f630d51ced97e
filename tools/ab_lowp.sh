#!/bin/bash
# A/B of library variants on the reduced-precision bench lines (tuned plans).
# usage: tools/ab_lowp.sh main <variant> ...
for v in "$@"; do
  if [ $v = main ]; then lib=paper_conf_sc_panzzxwslr0d24_b200/lib/librecflex.so; else lib=paper_conf_sc_panzzxwslr0d24_b200/lib/variants/$v/librecflex.so; fi
  for cd in heavy:bf16 heavy:fp8 heavy:i8 sharded1000:bf16; do
    c=${cd%%:*}; d=${cd##*:}
    RECFLEX_LIB=$lib timeout 600 python bench.py --config $c --dtype $d --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', '$c', '$d', round(d['ms_per_step'],3), 'k', d['config']['occupancy'])"
  done
done
