mkdir -p gpurun_out
SIEVE_HOST_TIMING=1 timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-ncu-traffic > gpurun_out/bench_r02o_ht.log 2> gpurun_out/bench_r02o_ht.err
cuobjdump -res-usage paper_conf_ispass_naderantahanse23_b200/libsieve.so > gpurun_out/resusage.txt 2>&1
