mkdir -p gpurun_out
timeout 600 ncu --kernel-name regex:"k_assign" --launch-skip 1 --launch-count 1 --set full --import-source on --clock-control none -o gpurun_out/ncu_assign_r02ah -f python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/ncu_assign_r02ah.log 2>&1
