# ncu --set full of the main k_search launch, new build vs build/old (SW_FORCE_MENU pins the entry).
#   bash tools/ncu_ab.sh TAG "m:menu m:menu ..."
TAG=$1; O=gpurun_out/$TAG; mkdir -p $O
for mm in $2; do
  m=${mm%%:*}; menu=${mm##*:}
  for v in new old; do
    lib=""; [ $v = old ] && lib=build/old/libsw_b200.so
    SW_LIB=$lib SW_FORCE_MENU=$menu timeout 900 ncu --set full --clock-control none --import-source on \
      -k regex:k_search -c 1 -o $O/${v}_m$m -f python tools/profile_one.py $m 3072 1 > $O/${v}_m$m.log 2>&1
    tail -1 $O/${v}_m$m.log
  done
done
