set -x
timeout 600 python -m pytest tests/test_parity_gpu.py -q -p no:cacheprovider -x -k "gangs or long_sequence or auto" 2>&1 | tail -3 > gpurun_out/r02l_tests.txt
Ts=$(python -c "print(','.join(str(t) for t in list(range(3072,1171,-100))+[1024,512,0,36000]))")
timeout 1200 python tools/sweep_threshold.py C2 567 $Ts > gpurun_out/r02l_sweep_c2_567.jsonl 2> gpurun_out/r02l_sweep.err
timeout 900 python tools/variance_sweep.py > gpurun_out/r02l_variance.jsonl 2> gpurun_out/r02l_variance.err
