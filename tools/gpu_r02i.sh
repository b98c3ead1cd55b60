mkdir -p gpurun_out
for so in default build/variants/libsieve_mmtest.so; do
  if [ "$so" = default ]; then unset SIEVE_LIB_PATH; tag=default; else export SIEVE_LIB_PATH=$PWD/$so; tag=$(basename $so .so); fi
  timeout 300 ncu --kernel-name k_moments --launch-count 3 --metrics gpu__time_duration.sum,dram__bytes_read.sum --clock-control none python bench.py --steps 1 --warmup 2 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/mm_$tag.log 2>&1
done
unset SIEVE_LIB_PATH
timeout 900 ncu --kernel-name regex:"k_cell_hist|k_cell_scatter|k_assign|k_t3_scatter|k_moments$|k_part_stats|k_valleys" --launch-skip 0 --launch-count 9 --set full --import-source on --clock-control none -o gpurun_out/ncu_stream_r02i -f python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/ncu_stream_r02i.log 2>&1
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/tests_r02i.log 2>&1; echo rc=$? >> gpurun_out/tests_r02i.log
