mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/tests_r02m.log 2>&1; echo rc=$? >> gpurun_out/tests_r02m.log
timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_r02m.log 2>&1
timeout 1500 python bench.py --config C5 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_c5_r02m.log 2>&1
