NEO_KLSS_REC=tc timeout 600 python -m pytest tests/test_gpu_klss.py -x -q 2>&1 | tail -1
timeout 600 python -m pytest tests/test_gpu_klss.py -x -q 2>&1 | tail -1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_klss_recover" -s 1 -c 1 -o gpurun_out/prof_klss3 python tools/klss_profile.py 1 > gpurun_out/ncu_klss.log 2>&1
python tools/ncu_summary.py gpurun_out/prof_klss3.ncu-rep
