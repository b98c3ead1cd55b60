mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/tests_r02q.log 2>&1; echo rc=$? >> gpurun_out/tests_r02q.log
timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_r02q.log 2>&1
SIEVE_NO_DEVICE_TIERS=1 timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_r02q_nodt.log 2>&1
TAG=r02q bash tools/gpu_sanitize.sh
