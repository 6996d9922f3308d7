for lib in build/old/libsw_b200.so build/v1/libsw_b200.so build/v2/libsw_b200.so; do
  echo "== $lib"
  SW_DEBUG_PLAN=1 SW_LIB=$lib timeout 300 python tools/query_sweep.py 3072 1500,5478 2>&1 | grep -E "tune m|gcups"
done
