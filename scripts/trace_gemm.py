"""Run one traced LD-32K call and print the pipeline timeline of CTA 0 (gemm_tc4)."""
import ctypes, os, sys
os.environ["SNP_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import snpgen
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
m, nbits = int(os.environ.get("M", 32768)), int(os.environ.get("NB", 16384))
A = torch.empty((m, snp.snp_words(nbits)), dtype=torch.uint64, device="cuda")
for r0 in range(0, m, 4096):
    r1 = min(m, r0 + 4096)
    snp.snp_pack(snpgen.ld_genotypes(1003, torch.arange(r0, r1, device="cuda"), nbits, xp="torch", device="cuda"), out=A[r0:r1])
r2 = torch.empty((m, m), dtype=torch.float32, device="cuda")
for _ in range(2):
    snp.snp_ld_r2(A, A, nbits, r2=r2)
torch.cuda.synchronize()
buf = (ctypes.c_longlong * (8 * 2048))()
snp.lib().snp_debug_gemm_trace(buf, 8 * 2048)
t = np.array(buf, dtype=np.int64).reshape(2048, 8)
nst = -(-nbits // 512)
ntiles = (-(-m // 128)) ** 2
tiles0 = -(-ntiles // 148)
nit = min(2048, tiles0 * nst)
t = t[:nit]
t0 = t[0, 0]
print("it   e_start  wait  lds  produce | mma_got(rel publish) commit   mma_at")
for it in list(range(0, 16)) + list(range(nit - 8, nit)):
    r = t[it] - t0
    print(f"{it:4d} {r[0]:8d} {t[it,1]-t[it,0]:5d} {t[it,2]-t[it,1]:5d} {t[it,3]-t[it,2]:7d} | {t[it,5]-t[it,3]:7d} {t[it,7]-t[it,5]:6d}  {r[5]:8d}")
v = slice(6, nit - 1)
print("median: exp wait", np.median(t[v, 1] - t[v, 0]), " lds", np.median(t[v, 2] - t[v, 1]), " produce", np.median(t[v, 3] - t[v, 2]),
      " mma issue interval", np.median(np.diff(t[6:nit, 5])), " mma got->commit", np.median(t[v, 7] - t[v, 5]),
      " publish->mma got", np.median(t[v, 5] - t[v, 3]))
iv = np.diff(t[:nit, 5])
print("mean MMA interval", iv.mean(), " max", iv.max(), " boundary stalls (interval at tile starts):",
      [int(iv[k * nst - 1]) for k in range(1, min(8, nit // nst))])
