mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_r02af.log 2>&1
timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_r02af.log 2>&1
