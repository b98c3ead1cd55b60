mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/tests_r02v.log 2>&1; echo rc=$? >> gpurun_out/tests_r02v.log
