for lib in build/old/libsw_b200.so ""; do
  for m in 144 567; do SW_LIB=$lib timeout 60 python tools/profile_long.py $m 3073 3 C3 | tail -1 | sed "s|^|[lib=$lib] |"; done
  for T in 3072 1172 512; do SW_LIB=$lib timeout 90 python tools/profile_long.py 567 $T 3 C2 | tail -1 | sed "s|^|[lib=$lib] |"; done
  SW_LIB=$lib SW_T_PACKED=0 timeout 60 python tools/profile_long.py 567 3072 3 C2 | tail -1 | sed "s|^|[lib=$lib packed0] |"
done > gpurun_out/r02w.txt 2>&1
