mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/tests_r02j.log 2>&1; echo rc=$? >> gpurun_out/tests_r02j.log
timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_r02j.log 2>&1
SIEVE_HOST_TIMING=1 timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_r02j_ht.log 2> gpurun_out/bench_r02j_ht.err
timeout 900 ncu --kernel-name regex:"k_cell_hist|k_cell_scatter|k_assign" --launch-skip 18 --launch-count 3 --set full --import-source on --clock-control none -o gpurun_out/ncu_cell_r02j -f python bench.py --steps 1 --warmup 2 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/ncu_cell_r02j.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_r02j.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/launches_r02j.log 2>&1
