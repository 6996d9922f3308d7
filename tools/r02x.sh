for lib in build/old/libsw_b200.so ""; do
  for m in 144 567; do SW_LIB=$lib timeout 60 python tools/profile_long.py $m 3073 3 C3 | tail -1 | sed "s|^|[lib=$lib] |"; done
  for T in 3072 1172 512; do SW_LIB=$lib timeout 90 python tools/profile_long.py 567 $T 3 C2 | tail -1 | sed "s|^|[lib=$lib] |"; done
done > gpurun_out/r02x.txt 2>&1
for pk in 0 1; do for T in 3072 1172 512 0; do SW_T_PACKED=$pk timeout 90 python tools/profile_long.py 567 $T 3 C2 | tail -1 | sed "s|^|[packed=$pk] |"; done; done >> gpurun_out/r02x.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 180 --timeout-method thread -x 2>&1 | tail -3 >> gpurun_out/r02x.txt
