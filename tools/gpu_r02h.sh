mkdir -p gpurun_out
./tools/mb/cub_yardstick > gpurun_out/cub_yardstick.log 2>&1
bash tools/ab_variants.sh > gpurun_out/ab_r02h.log 2>&1
timeout 900 ncu --kernel-name regex:"k_cell_hist|k_cell_scatter|k_assign|k_t3_scatter|k_moments$" --launch-skip 0 --launch-count 6 --set full --import-source on --clock-control none -o gpurun_out/ncu_stream_r02h -f python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/ncu_stream_r02h.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_r02h.log 2> gpurun_out/bench_r02h.err
