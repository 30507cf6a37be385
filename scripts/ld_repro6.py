import os, sys, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import snpgen
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
L = snp.lib()
rec = (ctypes.c_int * 8)()
L.snp_debug_gemm_watchdog(1, rec)
m, nbits = int(os.environ.get("M", 32768)), 16384
A = torch.empty((m, snp.snp_words(nbits)), dtype=torch.uint64, device="cuda")
for r0 in range(0, m, 4096):
    gg = snpgen.ld_genotypes(1003, torch.arange(r0, min(m, r0 + 4096), device="cuda"), nbits, structure=True, xp="torch", device="cuda")
    snp.snp_pack(gg, out=A[r0:r0 + gg.shape[0]])
torch.cuda.synchronize()
import time
for i in range(3):
    t0 = time.time()
    r2, _, cnt = snp.snp_ld_r2(A, A, nbits, counts=True)
    torch.cuda.synchronize()
    L.snp_debug_gemm_watchdog(1, rec)
    print(i, "done in", round(time.time() - t0, 3), "s; watchdog", list(rec), flush=True)
