#!/bin/bash
# A/B of library variants on the fp32 bench configs (tuned plans).
# usage: tools/ab_fp32.sh main <variant> ...
for v in "$@"; do
  if [ $v = main ]; then lib=paper_conf_sc_panzzxwslr0d24_b200/lib/librecflex.so; else lib=paper_conf_sc_panzzxwslr0d24_b200/lib/variants/$v/librecflex.so; fi
  for c in sharded1000 heavy medium industrial; do
    RECFLEX_LIB=$lib timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', '$c', round(d['ms_per_step'],4), 'fused', round(d['roofline']['fused_ms'],4))"
  done
done
