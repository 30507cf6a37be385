"""Expander-side per-iteration trace of the CTA-pair kernel (build -DSNP_PROFILING -DGEMM_TRACE
-DGEMM_DEBUG_SKIP, run with SNP_TRACE=1 SNP_GEMM_X2=1): warp 0 of both CTAs of cluster 0, the
time waiting for the MMA to free the stage slot (empty) and for the packed stage (pfull)."""
import ctypes, os, sys
os.environ["SNP_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
nd, nbits = int(os.environ.get("ND", 16384)), int(os.environ.get("NBITS", 16384))
w = snp.snp_words(nbits)
A = torch.randint(-2**62, 2**62, (nd, w), dtype=torch.int64, device="cuda").view(torch.uint64)
B = A.clone()
for _ in range(2):
    snp.snp_ld_r2(A, B, nbits, counts=True)
torch.cuda.synchronize()
print("kernel", snp.snp_last_kernel())
buf = (ctypes.c_longlong * 16384)()
snp.lib().snp_debug_gemm_trace(buf, 16384)
t = np.array(buf, dtype=np.int64).reshape(2048, 8)[50:1500]
for c in (0, 1):
    u = t[:, 4 * c: 4 * c + 4].astype(np.float64)
    print(f"CTA {c}: per group-0 iteration (2 stages): interval {np.median(np.diff(u[:, 0])):.0f}  "
          f"wait empty {np.median(u[:, 1] - u[:, 0]):.0f}  wait pfull {np.median(u[:, 2] - u[:, 1]):.0f}  "
          f"arrive {np.median(u[:, 3] - u[:, 2]):.0f} cycles")
