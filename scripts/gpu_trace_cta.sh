timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_exactness.py -q -x -k "ld or sym or pair or tri or general or cfg" 2>&1 | tail -1
