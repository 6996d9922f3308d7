for m in 144 375 567 729; do for T in 3072 2572 2072; do for sc in 0 ""; do
  SW_DEBUG_PLAN=1 SW_SCAN=$sc timeout 120 python tools/profile_long.py $m $T 3 C2 2>&1 | grep -E "scan items|GCUPS" | tail -2 | sed "s/^/[m=$m T=$T scan=$sc] /"
done; done; done
