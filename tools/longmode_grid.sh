# long-sequence path: T-mode vs team mode on C3 (all long) per query length.
#   bash tools/longmode_grid.sh "567 1500 5478"
for m in $1; do for mode in t team default; do
  if [ $mode = default ]; then r=$(python tools/profile_one.py $m 0 2 C3 | tail -1); else r=$(SW_LONG_MODE=$mode python tools/profile_one.py $m 0 2 C3 | tail -1); fi
  echo "mode=$mode $r"
done; done
