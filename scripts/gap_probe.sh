python scripts/gap_probe.py
SNP_DEBUG_NOSTORE=1 python scripts/gap_probe.py 2>&1 | head -1
