mkdir -p gpurun_out
timeout 600 python tools/timeline.py --steps 3 > gpurun_out/timeline_r02w.log 2>&1
