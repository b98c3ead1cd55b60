mkdir -p gpurun_out
./tools/mb/mb_kde3 > gpurun_out/mb_kde3.log 2>&1
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/tests_r02c.log 2>&1; echo rc=$? >> gpurun_out/tests_r02c.log
SIEVE_HOST_TIMING=1 timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_r02c.log 2> gpurun_out/bench_r02c.err
