# T-mode team-size grid on C3 (all long): SW_T_TEAM x SW_T_BIG for given query lengths.
#   bash tools/tmode_grid.sh "144 567" > gpurun_out/tgrid.txt
for m in $1; do for w in 2 4 8; do for big in 16 1000000; do
  echo "m=$m W=$w big=$big $(SW_LONG_MODE=t SW_T_TEAM=$w SW_T_BIG=$big python tools/profile_one.py $m 0 2 C3 | tail -1)"
done; done; done
