"""LD step parts on one GPU (CUDA graphs of 20 reps, the L2 flush before each rep timed alone and
subtracted, as bench.py does): pack_popc alone, snp_ld_sym alone, the whole step."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_binderlp19_b200 as snp
import snpgen
torch.cuda.set_device(0)
m, nbits = int(os.environ.get("M", 2048)), int(os.environ.get("NBITS", 4096))
G = snpgen.ld_genotypes(1001, torch.arange(m, device="cuda"), nbits, structure=True, xp="torch", device="cuda")
w = snp.snp_words(nbits)
B = torch.empty((m, w), dtype=torch.uint64, device="cuda")
pop = torch.empty(m, dtype=torch.uint32, device="cuda")
nt = snp.snp_sym_tiles(m)
r2 = torch.empty((nt, 128, 128), dtype=torch.float32, device="cuda")
cnt = torch.empty((nt, 128, 128), dtype=torch.uint32, device="cuda")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
pack = lambda: snp.snp_pack_popc(G, nbits=nbits, out=B, popc=pop)
ld = lambda: snp.snp_ld_sym(B, nbits, popA=pop, r2=r2, counts=cnt)
def graph(fns, n=20, fl=True):
    s = torch.cuda.Stream(); s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for f in fns: f()
    torch.cuda.current_stream().wait_stream(s); torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(n):
            if fl: flush.add_(1)
            for f in fns: f()
    g.replay(); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(3):
        e0.record(); g.replay(); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1) * 1e3 / n)
    return min(ts)
f0 = graph([])
res = {"flush_us": f0}
for name, fns in (("pack_popc", [pack]), ("ld_sym", [ld]), ("step", [pack, ld])):
    res[name + "_us"] = round(graph(fns) - f0, 2)
    res[name + "_noflush_us"] = round(graph(fns, fl=False), 2)
res["kernel"] = snp.snp_last_kernel()
print(json.dumps(res))
