# ncu --set full captures of the top kernels (one launch each) for the Set-B bench step
K=${1:-k_ntt}
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"$K" -s 12 -c ${2:-4} -o gpurun_out/prof_full python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full.log 2>&1
tail -3 gpurun_out/ncu_full.log
