set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q -k "widepaths or fullsize or c5" > gpurun_out/tests_r02b_new.log 2>&1; echo rc=$? >> gpurun_out/tests_r02b_new.log
bash tools/ab_variants.sh > gpurun_out/ab_r02b.log 2>&1
timeout 600 ncu --kernel-name regex:"k_kde$|k_kde<" --kernel-name-base demangled --launch-skip 8 --launch-count 1 --set full --import-source on --clock-control none -o gpurun_out/ncu_kde_r02b -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_kde_r02b.log 2>&1
timeout 600 ncu --kernel-name regex:"k_moments$|k_assign" --launch-skip 4 --launch-count 2 --set full --import-source on --clock-control none -o gpurun_out/ncu_stream_r02b -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_stream_r02b.log 2>&1
