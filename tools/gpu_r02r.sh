mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -x -q > gpurun_out/tests_r02r.log 2>&1; echo rc=$? >> gpurun_out/tests_r02r.log
timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_r02r.log 2>&1
timeout 600 ncu --kernel-name k_moments --launch-skip 2 --launch-count 1 --set full --clock-control none -o gpurun_out/ncu_mom_r02r -f python bench.py --steps 1 --warmup 2 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/ncu_mom_r02r.log 2>&1
