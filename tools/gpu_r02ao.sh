mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_r02ao.log 2>&1
SIEVE_HOST_TIMING=1 timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/ht_r02ao.log 2> gpurun_out/ht_r02ao.err
timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_r02ao.log 2>&1
