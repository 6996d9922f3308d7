timeout 600 python -m pytest tests/test_scan_gpu.py -x -q -p no:cacheprovider 2>&1 | tail -3
timeout 600 python -m pytest tests/test_parity_gpu.py -x -q -p no:cacheprovider -k "gang or long" 2>&1 | tail -2
bash tools/r02s3.sh
