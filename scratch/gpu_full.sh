#!/bin/bash
# one gpurun call: full GPU tests, smoke, the default bench line, the ncu launch list and
# --set full captures of the KDE and the streaming kernels (round tag $TAG)
TAG=${TAG:-r01}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/tests_$TAG.log 2>&1; echo tests_rc=$? >> gpurun_out/tests_$TAG.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
timeout 600 python bench.py > gpurun_out/bench_$TAG.log 2>&1
if [ -z "$NO_NCU" ]; then
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
  python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/launches_$TAG.log 2>&1
timeout 900 ncu --kernel-name k_kde --launch-skip 8 --launch-count 2 --set full --import-source on --clock-control none \
  -o gpurun_out/prof_kde_$TAG -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/prof_kde_$TAG.log 2>&1
timeout 900 ncu --kernel-name regex:"k_moments$|k_t3_compact|k_cellkey|k_os_pass|k_cell_offsets|k_assign|k_valleys|k_part_stats" --launch-skip 60 --launch-count 12 --set full --clock-control none \
  -o gpurun_out/prof_stream_$TAG -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/prof_stream_$TAG.log 2>&1
fi
