mkdir -p gpurun_out
SIEVE_HOST_TIMING=1 timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_r02s_ht.log 2> gpurun_out/bench_r02s_ht.err
timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_r02s.log 2>&1
