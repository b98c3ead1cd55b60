#!/bin/bash
# A/B: bench.py phase times for every build/variants/libsieve_*.so (and the default build)
for so in default build/variants/libsieve_*.so; do
  if [ "$so" = default ]; then unset SIEVE_LIB_PATH; else export SIEVE_LIB_PATH=$PWD/$so; fi
  timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>>gpurun_out/ab_err.log | python -c "
import json,sys
d=json.loads(sys.stdin.read())
ph={k: round(v['ms_per_step'],3) for k,v in d['phases'].items()}
print('$so', round(d['ms_per_step'],3), ph)"
done
