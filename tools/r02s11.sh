timeout 600 python -m pytest tests/test_scan_gpu.py -q -p no:cacheprovider 2>&1 | tail -1
for m in 144 222 375; do for T in 3072 2572; do for sc in 0 ""; do
  SW_DEBUG_PLAN=1 SW_SCAN=$sc timeout 120 python tools/profile_long.py $m $T 3 C2 2>&1 | grep -E "scan items|GCUPS" | tail -2 | sed "s/^/[m=$m T=$T scan=$sc] /"
done; done; done
SW_PROBE_EXTRA=64000,60000 SW_DEBUG_PLAN=1 timeout 120 python tools/profile_long.py 567 3072 3 C2 "SW_LONG_MODE=t" 2>&1 | grep -E "scan items|GCUPS" | tail -2 | sed "s/^/[outlier 567] /"
SW_PROBE_EXTRA=64000,60000 SW_SCAN=0 timeout 120 python tools/profile_long.py 567 3072 3 C2 "SW_LONG_MODE=t" 2>&1 | grep -E "GCUPS" | tail -1 | sed "s/^/[outlier 567 scan=0] /"
