mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/tests_r02k.log 2>&1; echo rc=$? >> gpurun_out/tests_r02k.log
bash tools/ab_variants.sh > gpurun_out/ab_r02k.log 2>&1
timeout 600 ncu --kernel-name k_moments --launch-skip 2 --launch-count 1 --set full --import-source on --clock-control none -o gpurun_out/ncu_mom_r02k -f python bench.py --steps 1 --warmup 2 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/ncu_mom_r02k.log 2>&1
