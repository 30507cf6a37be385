"""Run one traced FastID-1M call and print the per-iteration pipeline latencies of CTA 0."""
import ctypes, os, sys
os.environ["SNP_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import snpgen
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
nq, nd, nbits = 64, 1_000_000, 4096
D = torch.empty((nd, snp.snp_words(nbits)), dtype=torch.uint64, device="cuda")
for r0 in range(0, nd, 65536):
    r1 = min(nd, r0 + 65536)
    snp.snp_pack(snpgen.fastid_db(1002, torch.arange(r0, r1, device="cuda"), nbits, xp="torch", device="cuda"), out=D[r0:r1])
q, _ = snpgen.fastid_queries(1002, nq, nd, nbits)
Q = snp.snp_pack(torch.from_numpy(q).cuda())
for _ in range(3):
    out = snp.snp_fastid(Q, D, nbits, "xor")
torch.cuda.synchronize()
buf = (ctypes.c_longlong * 8192)()
snp.lib().snp_debug_fastid_trace(buf, 8192)
t = np.array(buf, dtype=np.int64).reshape(1024, 8)
t0 = t[0, 0]
tiles0 = (-(-nd // 128) + 147) // 148
kb = 512
nit = tiles0 * (-(-nbits // kb))
t = t[:nit]
print("CTA0 iterations", nit)
print("it  exp_start  waited  produce  mma_issue-full_arrive   mma_t  fence  asm  gap")
for it in list(range(0, 24)) + list(range(nit - 12, nit)):
    r = t[it] - t0
    print(f"{it:4d} {r[0]:9d} {r[1]-r[0]:7d} {r[2]-r[1]:8d} {r[3]-r[2]:9d} {r[3]:9d} {r[4]-r[3]:5d} {r[5]-r[4]:5d}")
v = slice(8, nit - 1)
d = np.diff(t[8:nit, 3])
print("MMA issue interval: median", np.median(d), "mean", d.mean())
print("expander produce (after waits): median", np.median(t[v, 2] - t[v, 1]))
print("expander wait: median", np.median(t[v, 1] - t[v, 0]))
print("full arrive -> MMA issue: median", np.median(t[v, 3] - t[v, 2]))
print("MMA: fence", np.median(t[v, 4] - t[v, 3]), "asm", np.median(t[v, 5] - t[v, 4]),
      "asm-end -> next full-wait-done", np.median(t[9:nit, 3] - t[8:nit - 1, 5]))
