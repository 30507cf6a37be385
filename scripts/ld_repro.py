import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import snpgen
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
for m, nbits, structure, counts in [(4096, 16384, True, True), (4096, 16384, False, True), (8192, 16384, True, False), (32768, 16384, True, True)]:
    A = torch.empty((m, snp.snp_words(nbits)), dtype=torch.uint64, device="cuda")
    for r0 in range(0, m, 4096):
        r1 = min(m, r0 + 4096)
        snp.snp_pack(snpgen.ld_genotypes(1003, torch.arange(r0, r1, device="cuda"), nbits, structure=structure, xp="torch", device="cuda"), out=A[r0:r1])
    try:
        r2, _, c = snp.snp_ld_r2(A, A, nbits, counts=counts)
        torch.cuda.synchronize()
        print(m, nbits, structure, counts, "ok", snp.snp_last_kernel(), flush=True)
    except Exception as e:
        print(m, nbits, structure, counts, "FAIL", str(e)[:200], flush=True)
        break
