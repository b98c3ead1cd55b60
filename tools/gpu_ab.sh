#!/bin/bash
# one gpurun call: parity tests on the default build, A/B bench of every variant, ncu of k_kde
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q ${TESTS:-} > gpurun_out/ab_tests.log 2>&1; echo tests_rc=$? >> gpurun_out/ab_tests.log
bash tools/ab_variants.sh > gpurun_out/ab.log 2>&1
if [ -n "$NCU" ]; then
  for so in default $NCU_VARIANTS; do
    if [ "$so" = default ]; then unset SIEVE_LIB_PATH; tag=default; else export SIEVE_LIB_PATH=$PWD/$so; tag=$(basename $so .so); fi
    timeout 600 ncu --kernel-name regex:"$NCU" --kernel-name-base demangled --launch-skip ${NCU_SKIP:-8} --launch-count 1 --set full --import-source on --clock-control none \
      -o gpurun_out/ncu_$tag -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_$tag.log 2>&1
  done
fi
