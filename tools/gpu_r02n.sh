mkdir -p gpurun_out
bash tools/ab_variants.sh > gpurun_out/ab_r02n.log 2>&1
for so in default build/variants/libsieve_asc128.so; do
  if [ "$so" = default ]; then unset SIEVE_LIB_PATH; tag=default; else export SIEVE_LIB_PATH=$PWD/$so; tag=$(basename $so .so); fi
  timeout 1500 python bench.py --config C5 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/c5_$tag.log 2>&1
done
