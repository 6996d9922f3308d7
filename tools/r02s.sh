for f in 0 4 1 2 7; do
  for rep in 1 2; do
  SW_T_PACK_FLAGS=$f timeout 60 python -m pytest tests/test_parity_gpu.py -q -p no:cacheprovider -x -k "threshold_invariance or tmode_gangs_repeated or auto_threshold" 2>&1 | tail -1 | sed "s/^/[flags $f] /"
  done
done > gpurun_out/r02s.txt 2>&1
