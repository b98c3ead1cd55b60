mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "boundaries" > gpurun_out/tests_r02l.log 2>&1; echo rc=$? >> gpurun_out/tests_r02l.log
TAG=r02l bash tools/gpu_sanitize.sh
timeout 1500 python bench.py --config C5 --steps 5 --warmup 3 --no-e2e > gpurun_out/bench_c5_r02l.log 2> gpurun_out/bench_c5_r02l.err
