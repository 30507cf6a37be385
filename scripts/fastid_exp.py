"""FastID-1M cost breakdown of the fused search kernel (CUDA-event timing, graph-free)."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
nq = int(os.environ.get("NQ", 64)); nd = int(os.environ.get("ND", 1_000_000)); nbits = int(os.environ.get("K", 4096))
w = snp.snp_words(nbits)
D = torch.randint(-2**62, 2**62, (nd, w), dtype=torch.int64, device="cuda").view(torch.uint64)
Q = torch.randint(-2**62, 2**62, (nq, w), dtype=torch.int64, device="cuda").view(torch.uint64)
outs = [torch.empty((nq, nd), dtype=torch.uint32, device="cuda") for _ in range(2)]
def t(fn, n=20):
    for _ in range(3): fn()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); s.record()
    for _ in range(n): fn()
    e.record(); torch.cuda.synchronize()
    return s.elapsed_time(e) / n
res = {}
pd = snp.snp_row_popc(D, nbits)
res["2ops counts+best popD"] = t(lambda: snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), counts=outs, best=True, popD=pd))
res["2ops best only popD"] = t(lambda: snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), counts=False, best=True, popD=pd))
res["2ops counts+best"] = t(lambda: snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), counts=outs, best=True))
res["2ops best only"] = t(lambda: snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), counts=False, best=True))
res["1op counts+best"] = t(lambda: snp.snp_fastid_search(Q, D, nbits, ("xor",), counts=outs[:1], best=True))
res["1op counts"] = t(lambda: snp.snp_fastid(Q, D, nbits, "xor", out=outs[0]))
res["1op counts popD"] = t(lambda: snp.snp_fastid(Q, D, nbits, "xor", out=outs[0], popD=pd))
res["1op best only"] = t(lambda: snp.snp_fastid_search(Q, D, nbits, ("xor",), counts=False, best=True))
res["2ops counts only popD"] = t(lambda: snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), counts=outs, best=False, popD=pd))
rd = nd * w * 8
print(json.dumps({k: {"us": 1e3 * v, "GBps_read_only": rd / v / 1e6} for k, v in res.items()}), flush=True)
