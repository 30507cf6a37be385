"""LD-32K cost breakdown: counts-only vs r2 epilogue vs expanders skipped (results invalid
when SNP_DEBUG_SKIP_EXPAND=1).  Timing with CUDA events, 3 warm-ups."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
m = int(os.environ.get("M", 32768)); nbits = int(os.environ.get("K", 16384))
w = snp.snp_words(nbits)
A = torch.randint(-2**62, 2**62, (m, w), dtype=torch.int64, device="cuda").view(torch.uint64)
r2 = torch.empty((m, m), dtype=torch.float32, device="cuda")
cnt = torch.empty((m, m), dtype=torch.uint32, device="cuda")
def t(fn, n=3):
    for _ in range(2): fn()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); s.record()
    for _ in range(n): fn()
    e.record(); torch.cuda.synchronize()
    return s.elapsed_time(e) / n
res = {}
res["counts"] = t(lambda: snp.snp_ld_counts(A, A, nbits, C=cnt))
res["r2"] = t(lambda: snp.snp_ld_r2(A, A, nbits, r2=r2))
res["r2+counts"] = t(lambda: snp.snp_ld_r2(A, A, nbits, r2=r2, counts=cnt))
cmp = m * m * nbits
print(json.dumps({k: {"ms": v, "TOPS": 2 * cmp / v / 1e9} for k, v in res.items()}), flush=True)
