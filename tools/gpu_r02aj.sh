mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_r02aj.log 2>&1
timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_r02aj.log 2>&1
timeout 900 python bench.py --config C5 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_c5_r02aj.log 2>&1
