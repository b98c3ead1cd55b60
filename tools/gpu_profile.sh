#!/bin/bash
# one gpurun call: the full bench line, the ncu launch list of the same command, ncu --set full of
# the dominant kernel and of pass A / pass B, and the CUPTI device timeline.
#   gpurun -- 'TAG=r02x bash tools/gpu_profile.sh'
TAG=${TAG:-prof}
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/bench_full_$TAG.log 2> gpurun_out/bench_full_$TAG.err
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  --csv --log-file gpurun_out/launches_$TAG.csv \
  python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/launches_$TAG.log 2>&1
timeout 600 ncu --kernel-name regex:"k_kde$|k_kde<" --kernel-name-base demangled --launch-skip 8 --launch-count 1 \
  --set full --import-source on --clock-control none -o gpurun_out/ncu_kde_$TAG -f \
  python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/ncu_kde_$TAG.log 2>&1
timeout 600 ncu --kernel-name regex:"k_moments$|k_assign" --launch-skip 2 --launch-count 2 --set full \
  --import-source on --clock-control none -o gpurun_out/ncu_stream_$TAG -f \
  python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/ncu_stream_$TAG.log 2>&1
timeout 600 python tools/timeline.py --steps 3 > gpurun_out/timeline_$TAG.log 2>&1
