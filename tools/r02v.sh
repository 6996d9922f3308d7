timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 180 --timeout-method thread -x 2>&1 | tail -5 > gpurun_out/r02v_tests.txt
for pk in 0 1; do
  for m in 144 567; do timeout 60 python tools/profile_long.py $m 3073 3 C3 "SW_T_PACKED=$pk" | tail -1 | sed "s/^/[packed=$pk] /"; done
  for T in 3072 1172 512 0; do timeout 90 python tools/profile_long.py 567 $T 3 C2 "SW_T_PACKED=$pk" | tail -1 | sed "s/^/[packed=$pk] /"; done
done > gpurun_out/r02v_perf.txt 2>&1
