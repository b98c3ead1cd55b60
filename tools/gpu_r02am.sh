mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/bench_full_r02am.log 2> gpurun_out/bench_full_r02am.err
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_r02am.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/launches_r02am.log 2>&1
