#!/bin/bash
# A/B: heavy uniform sweep subset + sharded tuned bench for each variant
for v in "$@"; do
  if [ "$v" = main ]; then lib=paper_conf_sc_panzzxwslr0d24_b200/lib/librecflex.so; else lib=paper_conf_sc_panzzxwslr0d24_b200/lib/variants/$v/librecflex.so; fi
  echo "== $v"
  RECFLEX_LIB=$lib timeout 600 python tools/sweep.py heavy --ks 4,6 --ids 15,16,17 --parts 0 2>&1 | tail -3
done
for v in "$@"; do tools/variants.sh "--config sharded1000 --steps 10 --warmup 3" $v; tools/variants.sh "--config heavy --steps 10 --warmup 3" $v; done
