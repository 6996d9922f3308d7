# row scan: outlier pair (two 64k/60k sequences added to C2's long set) and the top pair alone
mkdir -p gpurun_out/s6
timeout 600 python -m pytest tests/test_scan_gpu.py -x -q -p no:cacheprovider 2>&1 | tail -2
for T in 3072 2072 1172; do for sc in 0 ""; do
  SW_PROBE_EXTRA=64000,60000 SW_DEBUG_PLAN=1 SW_SCAN=$sc timeout 120 python tools/profile_long.py 567 $T 3 C2 "SW_LONG_MODE=t" 2>&1 | grep -E "scan items|GCUPS" | tail -2 | sed "s/^/[outlier T=$T scan=$sc] /"
done; done
for sc in 0 1; do SW_SCAN=$sc timeout 120 python tools/profile_long.py 567 0 3 C2 "SW_LONG_MODE=t" top:2 2>&1 | tail -1 | sed "s/^/[top pair scan=$sc] /"; done
for sc in 0 ""; do SW_SCAN=$sc timeout 120 python tools/profile_long.py 567 3072 3 C2 2>&1 | tail -1 | sed "s/^/[C2 T=3072 scan=$sc] /"; done
