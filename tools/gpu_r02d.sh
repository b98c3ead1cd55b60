mkdir -p gpurun_out
./tools/mb/mb_kde2 > gpurun_out/mb_kde2.log 2>&1
timeout 900 python -m pytest tests/test_gpu_allocator.py tests/test_gpu_multirank.py tests/test_gpu_parity.py -x -q > gpurun_out/tests_r02d.log 2>&1; echo rc=$? >> gpurun_out/tests_r02d.log
timeout 900 python bench.py > gpurun_out/bench_r02d.log 2> gpurun_out/bench_r02d.err
timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_r02d2.log 2>&1
