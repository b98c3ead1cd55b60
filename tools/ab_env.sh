#!/bin/bash
# A/B of one environment knob on the bench: VAR=SIEVE_KDE_OVH VALS="inf 32 64" [CFG=C5] [STEPS=10]
#   gpurun -- 'VAR=... VALS=... bash tools/ab_env.sh'   (gpurun_out/abenv_<VAR>_<val>_<cfg>.log)
mkdir -p gpurun_out
CFG=${CFG:-C4}
for v in $VALS; do
  env $VAR=$v timeout 600 python bench.py --config $CFG --steps ${STEPS:-10} --warmup 3 --no-e2e --no-cpu-baseline \
    --no-ncu-traffic > gpurun_out/abenv_${VAR}_${v}_${CFG}.log 2>&1
  echo "== $VAR=$v $CFG"; python tools/bench_summary.py gpurun_out/abenv_${VAR}_${v}_${CFG}.log
done
