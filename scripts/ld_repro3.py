import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import snpgen
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
m, nbits = int(os.environ.get("M", 32768)), 16384
A = torch.empty((m, snp.snp_words(nbits)), dtype=torch.uint64, device="cuda")
for r0 in range(0, m, 4096):
    r1 = min(m, r0 + 4096)
    snp.snp_pack(snpgen.ld_genotypes(1003, torch.arange(r0, r1, device="cuda"), nbits, structure=os.environ.get("S", "1") == "1", xp="torch", device="cuda"), out=A[r0:r1])
torch.cuda.synchronize()
pa = snp.snp_row_popc(A, nbits)
op = os.environ.get("OP", "ld")
t0 = time.time()
try:
    if op == "ld":
        r2, _, c = snp.snp_ld_r2(A, A, nbits, popA=pa, popB=pa)
    else:
        c = snp.snp_ld_counts(A, A, nbits)
    torch.cuda.synchronize()
    print(m, op, "ok", time.time() - t0, flush=True)
except Exception as e:
    print(m, op, "FAIL after", time.time() - t0, "s:", str(e)[:120], flush=True)
