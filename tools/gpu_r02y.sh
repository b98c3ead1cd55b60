mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/tests_r02y.log 2>&1; echo rc=$? >> gpurun_out/tests_r02y.log
timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_r02y.log 2>&1
timeout 600 python tools/timeline.py --steps 3 > gpurun_out/timeline_r02y.log 2>&1
TAG=r02y bash tools/gpu_sanitize.sh
