#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over tools/sanitize_run.py (round tag $TAG)
TAG=${TAG:-r02}
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  extra=""
  [ "$tool" = memcheck ] && extra=""
  [ "$tool" = racecheck ] && extra="--racecheck-report all"
  timeout 1500 compute-sanitizer --tool $tool $extra --target-processes all --print-limit 50 \
    python tools/sanitize_run.py > gpurun_out/sanitize_${tool}_$TAG.log 2>&1
  echo "rc=$?" >> gpurun_out/sanitize_${tool}_$TAG.log
done
