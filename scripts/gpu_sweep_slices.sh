timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
timeout 600 python scripts/sweep.py --M 128,1024,8192 --N 1000000 --K 2048,4096 2>&1 >/dev/null | tail -7
SNP_SEARCH_SLICES=0 timeout 600 python scripts/sweep.py --M 128,1024,8192 --N 1000000 --K 2048,4096 2>&1 >/dev/null | tail -7
