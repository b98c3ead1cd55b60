mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/tests_r02u.log 2>&1; echo rc=$? >> gpurun_out/tests_r02u.log
timeout 900 python bench.py > gpurun_out/bench_r02u.log 2> gpurun_out/bench_r02u.err
TAG=r02u bash tools/gpu_sanitize.sh
