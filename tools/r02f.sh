set -x
for sel in top:2 top:4 top:8 top:16 top:32 drop:32 drop:64 ""; do
  python tools/profile_long.py 567 3072 3 C2 "" "$sel" | tail -1 | sed "s/^/[$sel] /"
  python tools/profile_long.py 567 3072 3 C2 "SW_T_GANG=0:0" "$sel" | tail -1 | sed "s/^/[nogang $sel] /"
done > gpurun_out/r02f_sel.txt 2>&1
for g in 4:2 4:4 4:8 6:4 8:2 8:4 3:8 2:16 5:6; do
  python tools/profile_long.py 567 3072 3 C2 "SW_T_GANG=$g" | tail -1 | sed "s/^/[gang $g T3072] /"
  python tools/profile_long.py 567 2572 3 C2 "SW_T_GANG=$g" | tail -1 | sed "s/^/[gang $g T2572] /"
done > gpurun_out/r02f_gang.txt 2>&1
