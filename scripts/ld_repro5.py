import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import snpgen
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
m, nbits = int(os.environ.get("M", 24576)), 16384
A = torch.empty((m, snp.snp_words(nbits)), dtype=torch.uint64, device="cuda")
for r0 in range(0, m, 4096):
    gg = snpgen.ld_genotypes(1003, torch.arange(r0, min(m, r0 + 4096), device="cuda"), nbits, structure=True, xp="torch", device="cuda")
    snp.snp_pack(gg, out=A[r0:r0 + gg.shape[0]])
torch.cuda.synchronize()
r2, _, cnt = snp.snp_ld_r2(A, A, nbits, counts=True)
torch.cuda.synchronize()
print("ok")
