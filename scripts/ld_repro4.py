import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import snpgen
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
m, nbits, seed = int(os.environ.get("M", 32768)), 16384, 1003
A = torch.empty((m, snp.snp_words(nbits)), dtype=torch.uint64, device="cuda")
for r0 in range(0, m, 4096):
    gg = snpgen.ld_genotypes(seed, torch.arange(r0, r0 + 4096, device="cuda"), nbits, structure=True, xp="torch", device="cuda")
    snp.snp_pack(gg, out=A[r0:r0 + 4096])
torch.cuda.synchronize(); print("packed", flush=True)
for i in range(3):
    for variant in ("given", "ws"):
        try:
            if variant == "given":
                pa = snp.snp_row_popc(A, nbits)
                r2, _, cnt = snp.snp_ld_r2(A, A, nbits, popA=pa, popB=pa, counts=True)
            else:
                r2, _, cnt = snp.snp_ld_r2(A, A, nbits, counts=True)
            torch.cuda.synchronize()
            print(i, variant, "ok", snp.snp_last_kernel(), flush=True)
        except Exception as e:
            print(i, variant, "FAIL", str(e)[:150], flush=True)
            sys.exit(1)
