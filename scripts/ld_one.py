"""One LD r2 (+counts) call at MxM x K for ncu captures."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
m = int(os.environ.get("M", 32768)); nbits = int(os.environ.get("K", 16384))
A = torch.randint(-2**62, 2**62, (m, snp.snp_words(nbits)), dtype=torch.int64, device="cuda").view(torch.uint64)
r2 = torch.empty((m, m), dtype=torch.float32, device="cuda")
cnt = torch.empty((m, m), dtype=torch.uint32, device="cuda") if os.environ.get("COUNTS") else None
for _ in range(2):
    snp.snp_ld_r2(A, A, nbits, r2=r2, counts=cnt)
torch.cuda.synchronize()
