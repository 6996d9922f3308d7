mkdir -p gpurun_out/s7
timeout 600 python -m pytest tests/test_scan_gpu.py -q -p no:cacheprovider 2>&1 | tail -1
for sc in 0 1; do SW_SCAN=$sc timeout 120 python tools/profile_long.py 567 0 3 C2 "SW_LONG_MODE=t" top:2 2>&1 | tail -1 | sed "s/^/[top pair scan=$sc] /"; done
for m in 144 567 1500; do for T in 3072 2572; do for sc in 0 ""; do
  SW_DEBUG_PLAN=1 SW_SCAN=$sc timeout 120 python tools/profile_long.py $m $T 3 C2 2>&1 | grep -E "scan items|GCUPS" | tail -2 | sed "s/^/[m=$m T=$T scan=$sc] /"
done; done; done
