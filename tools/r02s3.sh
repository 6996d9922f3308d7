mkdir -p gpurun_out/s3
for T in 3072 2572 2072 1572; do
  for sc in 0 ""; do
    SW_DEBUG_PLAN=1 SW_SCAN=$sc timeout 120 python tools/profile_long.py 567 $T 3 C2 2>&1 | grep -E "scan items|GCUPS" | tail -2 | sed "s/^/[scan=$sc] /"
  done
done > gpurun_out/s3/long.txt 2>&1
for m in 567; do for sc in 0 ""; do
  SW_DEBUG_PLAN=1 SW_SCAN=$sc timeout 120 python tools/profile_long.py $m 3073 3 C3 2>&1 | grep -E "scan items|GCUPS" | tail -2 | sed "s/^/[C3 scan=$sc] /"
done; done >> gpurun_out/s3/long.txt 2>&1
cat gpurun_out/s3/long.txt
