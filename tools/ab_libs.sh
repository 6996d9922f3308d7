# Query sweep (C2, T=3072) for several library builds, interleaved twice.
#   bash tools/ab_libs.sh TAG "lens" lib1.so lib2.so ...
TAG=$1; LENS=$2; shift 2
O=gpurun_out/$TAG; mkdir -p $O
for i in 1 2; do
  for lib in "$@"; do
    SW_REPS=3 SW_LIB=$lib timeout 300 python tools/query_sweep.py 3072 $LENS | sed "s|^|$lib |"
  done
done > $O/qsweep.txt 2>&1
cat $O/qsweep.txt
