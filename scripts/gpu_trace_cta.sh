timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_exactness.py -q -x -k "fastid or search or stream or best or exact" 2>&1 | tail -2
