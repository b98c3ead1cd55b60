#!/bin/bash
# one gpurun call: GPU parity tests, a short bench line and the host-side timing marks.
#   gpurun -- 'TAG=r02x bash tools/gpu_check.sh'     (outputs under gpurun_out/*_$TAG.*)
TAG=${TAG:-check}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q ${TESTS:-} > gpurun_out/pytest_$TAG.log 2>&1
SIEVE_HOST_TIMING=1 timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-ncu-traffic \
  > gpurun_out/ht_$TAG.log 2> gpurun_out/ht_$TAG.err
timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_$TAG.log 2>&1
if [ -n "$C5" ]; then
  timeout 900 python bench.py --config C5 --steps 2 --warmup 2 --no-e2e --no-cpu-baseline --no-ncu-traffic \
    > gpurun_out/bench_c5_$TAG.log 2>&1
fi
