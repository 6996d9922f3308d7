timeout 600 python -m pytest tests/test_scan_gpu.py -x -q -p no:cacheprovider 2>&1 | grep -E "Error|error|assert|mismatch" | head -10
SW_SCAN=0 timeout 120 python tools/profile_long.py 567 3072 2 C2 2>&1 | tail -3
timeout 600 python -m pytest tests/test_parity_gpu.py -x -q -p no:cacheprovider -k "long or gang" 2>&1 | tail -3
