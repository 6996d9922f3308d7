# A/B of the short path (group kernels) against build/old/libsw_b200.so, then the GPU parity tests.
#   bash tools/ab_short.sh TAG
TAG=${1:-abs}
O=gpurun_out/$TAG; mkdir -p $O
for i in 1 2; do
  SW_REPS=3 SW_LIB=build/old/libsw_b200.so timeout 300 python tools/query_sweep.py 3072 144,375,729,1500,5478 | sed 's/^/old /'
  SW_REPS=3 timeout 300 python tools/query_sweep.py 3072 144,375,729,1500,5478 | sed 's/^/new /'
done > $O/qsweep.txt 2>&1
cat $O/qsweep.txt
timeout 1200 python -m pytest tests -m gpu -x -q -p no:cacheprovider > $O/pytest.log 2>&1; tail -3 $O/pytest.log
