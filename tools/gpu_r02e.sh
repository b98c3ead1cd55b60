mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/tests_r02e.log 2>&1; echo rc=$? >> gpurun_out/tests_r02e.log
timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_r02e.log 2>&1
SIEVE_CELL_RADIX=1 timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_r02e_radix.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_r02e.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/launches_r02e.log 2>&1
