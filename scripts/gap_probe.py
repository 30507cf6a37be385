"""Back-to-back timing of library kernels vs host overhead (methodology probe)."""
import os, sys, time
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
out = torch.empty((nq, nd), dtype=torch.uint32, device="cuda")
def timeit(name, fn, n=20):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda._sleep(200_000_000)          # ~100 ms of GPU busy-wait: host queues everything meanwhile
    a.record()
    h0 = time.perf_counter()
    for _ in range(n): fn()
    h1 = time.perf_counter()
    b.record(); torch.cuda.synchronize()
    print(f"{name:30s} GPU {a.elapsed_time(b) / n * 1e3:9.1f} us/call   host {(h1 - h0) / n * 1e6:8.1f} us/call", flush=True)
timeit("fastid xor", lambda: snp.snp_fastid(Q, D, nbits, "xor", out=out))
timeit("fastid andnot", lambda: snp.snp_fastid(Q, D, nbits, "andnot", out=out))
timeit("fastid and", lambda: snp.snp_fastid(Q, D, nbits, "and", out=out))
