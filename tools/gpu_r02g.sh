mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/tests_r02g.log 2>&1; echo rc=$? >> gpurun_out/tests_r02g.log
bash tools/ab_variants.sh > gpurun_out/ab_r02g.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_r02g.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/launches_r02g.log 2>&1
