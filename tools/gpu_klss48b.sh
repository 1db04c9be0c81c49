set -x
timeout 1200 python -m pytest tests/test_gpu_klss.py -q -x 2>&1 | tail -5
for b in 1 8; do timeout 300 python tools/klss_profile.py $b 48; done
