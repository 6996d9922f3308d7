set -x
for m in 144 567 1500 2504; do
  for g in "SW_T_GANG=8:1" "SW_T_GANG=8:1;SW_T_GANG_CHAIN2=0"; do python tools/profile_long.py $m 3072 3 C2 "$g" top:2 | tail -1 | sed "s/^/[$g] /"; done
  python tools/profile_long.py $m 3072 2 C2 "SW_T_GANG=0:0;SW_T_TEAM=1" top:2 | tail -1 | sed "s/^/[team1 nogang] /"
done > gpurun_out/r02i_var.txt 2>&1
