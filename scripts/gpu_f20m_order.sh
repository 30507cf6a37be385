#!/bin/bash
# FastID-20M general-kernel raster orders (SNP_GEMM_ORDER: 2 grouped (default), 1 lane-block-major,
# 0 column-block-major) on the configs[3] shape, counts of both ops (no best pass)
cat > /tmp/f20.py <<'PY'
import os, sys, torch
sys.path.insert(0, os.getcwd())
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
nq, nd, nbits = 1024, int(os.environ.get("ND", 20_000_000)), 8192
w = snp.snp_words(nbits)
D = torch.randint(-2**62, 2**62, (nd, w), dtype=torch.int64, device="cuda").view(torch.uint64)
Q = torch.randint(-2**62, 2**62, (nq, w), dtype=torch.int64, device="cuda").view(torch.uint64)
pd = snp.snp_row_popc(D, nbits)
outs = [torch.empty((nq, nd), dtype=torch.uint32, device="cuda") for _ in range(2)]
f = lambda: snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), counts=outs, best=False, popD=pd)
f(); torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(); f(); e1.record(); torch.cuda.synchronize()
print(os.environ.get("SNP_GEMM_ORDER", "2"), nd, round(e0.elapsed_time(e1), 2), "ms", snp.snp_last_kernel())
PY
for o in 2 1 0; do SNP_GEMM_ORDER=$o python /tmp/f20.py; done
