for b in 0 32 128; do
  SW_LIB=build/bk$b/libsw_b200.so SW_SCAN=1 timeout 120 python tools/profile_long.py 567 0 3 C2 "SW_LONG_MODE=t" top:2 2>&1 | tail -1 | sed "s/^/[backoff=$b top pair] /"
  SW_LIB=build/bk$b/libsw_b200.so timeout 120 python tools/profile_long.py 144 3072 3 C2 2>&1 | tail -1 | sed "s/^/[backoff=$b C2 144 T3072] /"
done
