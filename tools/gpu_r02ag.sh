mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_r02ag.log 2>&1
timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_r02ag.log 2>&1
timeout 600 ncu --kernel-name regex:"k_kde$|k_kde<" --kernel-name-base demangled --launch-skip 8 --launch-count 1 --set full --import-source on --clock-control none -o gpurun_out/ncu_kde_r02ag -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/ncu_kde_r02ag.log 2>&1
