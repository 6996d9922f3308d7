for f in 0 4 2 6 7; do
  for m in 567 144; do
    timeout 40 python tools/profile_long.py $m 3073 3 C3 "SW_T_PACK_FLAGS=$f" 2>&1 | tail -1 | sed "s/^/[flags $f m=$m] /"
    echo "[flags $f m=$m] rc=$?"
  done
done > gpurun_out/r02u.txt 2>&1
for f in 0 4 7; do timeout 40 python tools/profile_long.py 567 3072 3 C2 "SW_T_PACK_FLAGS=$f" 2>&1 | tail -1 | sed "s/^/[flags $f C2 T3072] /"; done >> gpurun_out/r02u.txt 2>&1
