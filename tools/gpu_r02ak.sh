mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "assign or C2 or C1" > gpurun_out/pytest_r02ak.log 2>&1
bash tools/ab_variants.sh > gpurun_out/ab_r02al.log 2>&1
timeout 900 python bench.py --config C5 --steps 2 --warmup 2 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_c5_r02ak.log 2>&1
