for m in 144 567; do for c2 in 0 1; do
SW_DEBUG_GANG_TIMES=1 python tools/profile_long.py $m 3072 2 C2 "SW_T_GANG=8:1;SW_T_GANG_CHAIN2=$c2" top:2 > gpurun_out/r02j_m${m}_c$c2.txt 2>&1
done; done
