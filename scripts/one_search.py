"""One fused FastID search (for ncu captures): NQ queries x ND rows x NBITS, XOR + ANDNOT,
best matches (COUNTS=1 also writes the count matrices); database popcounts given."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_binderlp19_b200 as snp
nq, nd, nbits = (int(os.environ.get(k, d)) for k, d in (("NQ", 1), ("ND", 20_000_000), ("NBITS", 4096)))
torch.cuda.set_device(0)
w = snp.snp_words(nbits)
D = torch.randint(-2**62, 2**62, (nd, w), dtype=torch.int64, device="cuda").view(torch.uint64)
Q = torch.randint(-2**62, 2**62, (nq, w), dtype=torch.int64, device="cuda").view(torch.uint64)
pd = snp.snp_row_popc(D, nbits)
for _ in range(3):
    snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), counts=os.environ.get("COUNTS") == "1", popD=pd)
torch.cuda.synchronize()
print(snp.snp_last_kernel())
