set -x
for b in 1 8; do timeout 300 python tools/klss_profile.py $b 48; done
timeout 300 python tools/klss_profile.py 1 36
