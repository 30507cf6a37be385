"""A/B timing of one FastID search shape (the bench's fused call by default) for the library
named by SNP_LIB_PATH: 20 calls captured in a CUDA graph, best of 5 replays, us per call."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
nq = int(os.environ.get("NQ", 64)); nd = int(os.environ.get("ND", 1_000_000)); nbits = int(os.environ.get("K", 4096))
counts = os.environ.get("COUNTS", "1") == "1"; nops = int(os.environ.get("NOPS", 2))
w = snp.snp_words(nbits) if os.environ.get("TIGHT") != "1" else (int(os.environ["LDW"]) if os.environ.get("LDW") else 2 * ((nbits + 127) // 128))   # TIGHT: 16-byte-granular rows
if os.environ.get("DATA", "random") == "snpgen":   # the bench's seeded genotype recipe
    import numpy as np
    import snpgen
    D = torch.empty((nd, w), dtype=torch.uint64, device="cuda")
    for r0 in range(0, nd, 32768):
        r1 = min(nd, r0 + 32768)
        snp.snp_pack(snpgen.fastid_db(7, torch.arange(r0, r1, device="cuda"), nbits, xp="torch", device="cuda"), out=D[r0:r1])
    q, _ = snpgen.fastid_queries(7, nq, nd, nbits)
    Q = snp.snp_pack(torch.from_numpy(np.ascontiguousarray(q)).cuda())
else:
    D = torch.randint(-2**62, 2**62, (nd, w), dtype=torch.int64, device="cuda").view(torch.uint64)
    Q = torch.randint(-2**62, 2**62, (nq, w), dtype=torch.int64, device="cuda").view(torch.uint64)
pd = snp.snp_row_popc(D, nbits)
ops = ("xor", "andnot")[:nops]
outs = [torch.empty((nq, nd), dtype=torch.uint32, device="cuda") for _ in ops] if counts else False
best = None if os.environ.get("NOBEST") == "1" else [(torch.empty(nq, dtype=torch.uint32, device="cuda"), torch.empty(nq, dtype=torch.int64, device="cuda")) for _ in ops]
ws = torch.zeros(snp.snp_fastid_search_workspace_bytes(nq, nd, nbits, len(ops)), dtype=torch.uint8, device="cuda")
call = lambda: snp.snp_fastid_search(Q, D, nbits, ops, counts=outs, best=best, ws=ws, popD=pd)
s = torch.cuda.Stream(); s.wait_stream(torch.cuda.current_stream())
with torch.cuda.stream(s):
    for _ in range(3): call()
torch.cuda.current_stream().wait_stream(s); torch.cuda.synchronize()
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g):
    for _ in range(20): call()
res = []
for _ in range(5):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); e0.record(); g.replay(); e1.record(); torch.cuda.synchronize()
    res.append(e0.elapsed_time(e1) / 20 * 1e3)
byt = (nd + nq) * w * 8 + (len(ops) * nq * nd * 4 if counts else 0)
lib = os.path.basename(os.environ.get("SNP_LIB_PATH", "libsnp.so"))
print(json.dumps({"lib": lib, "data": os.environ.get("DATA", "random"), "nq": nq, "nd": nd, "nbits": nbits, "ldw": w, "counts": counts, "best": best is not None, "kernel": snp.snp_last_kernel(),
                  "us_best": round(min(res), 2), "us_all": [round(x, 2) for x in res],
                  "hbm_frac": round(byt / (min(res) * 1e-6) / 6548.2e9, 4)}), flush=True)
if os.environ.get("CHECK") == "1" and best is not None:   # vs the CUDA-core variant of the same library
    ref = [(torch.empty(nq, dtype=torch.uint32, device="cuda"), torch.empty(nq, dtype=torch.int64, device="cuda")) for _ in ops]
    snp.snp_set_variant("popc")
    snp.snp_fastid_search(Q, D, nbits, ops, counts=False, best=ref, popD=pd)
    snp.snp_set_variant("auto")
    call(); torch.cuda.synchronize()
    ok = all(torch.equal(a[0], b[0]) and torch.equal(a[1], b[1]) for a, b in zip(best, ref))
    print(json.dumps({"lib": lib, "check_vs_popc": ok}), flush=True)
