mkdir -p gpurun_out/s2
for sc in 0 1; do for top in top:2 top:8; do
  SW_SCAN=$sc timeout 120 python tools/profile_long.py 567 0 3 C2 "SW_LONG_MODE=t" $top 2>&1 | tail -1 | sed "s/^/[scan=$sc $top] /"
done; done > gpurun_out/s2/top.txt 2>&1
cat gpurun_out/s2/top.txt
SW_SCAN=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_scan_pair -c 1 -o gpurun_out/s2/scan_top2 -f python tools/profile_long.py 567 0 1 C2 "SW_LONG_MODE=t" top:2 > gpurun_out/s2/ncu.log 2>&1
tail -2 gpurun_out/s2/ncu.log
