"""Where the FastID-1M bench step's time goes beyond the search kernel: CUDA-graph replays of
20 calls of (a) the search call, (b) pack(Q) + search, (c) (b) with event-record nodes at step
boundaries (the bench's step timing), (d) (c) with events around the search call too."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
nq, nd, nbits = 64, 1_000_000, 4096
w = snp.snp_words(nbits)
D = torch.randint(-2**62, 2**62, (nd, w), dtype=torch.int64, device="cuda").view(torch.uint64)
qb = torch.randint(0, 2, (nq, nbits), dtype=torch.uint8, device="cuda")
Q = torch.empty((nq, w), dtype=torch.uint64, device="cuda")
pd = snp.snp_row_popc(D, nbits)
outs = [torch.empty((nq, nd), dtype=torch.uint32, device="cuda") for _ in range(2)]
best = [(torch.empty(nq, dtype=torch.uint32, device="cuda"), torch.empty(nq, dtype=torch.int64, device="cuda")) for _ in range(2)]
ws = torch.zeros(snp.snp_fastid_search_workspace_bytes(nq, nd, nbits, 2), dtype=torch.uint8, device="cuda")
pack = lambda: snp.snp_pack(qb, nbits=nbits, out=Q)
search = lambda: snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), counts=outs, best=best, ws=ws, popD=pd)
mk = lambda: torch.cuda.Event(enable_timing=True, external=True)
def run(name, body, n=20):
    s = torch.cuda.Stream(); s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        body([torch.cuda.Event(enable_timing=True) for _ in range(4)])
    torch.cuda.current_stream().wait_stream(s); torch.cuda.synchronize()
    evs = [[mk() for _ in range(4)] for _ in range(n)]
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for i in range(n): body(evs[i])
    g.replay(); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    best_t = 1e9
    for _ in range(3):
        e0.record(); g.replay(); e1.record(); torch.cuda.synchronize()
        best_t = min(best_t, e0.elapsed_time(e1) / n * 1e3)
    ks = [ev[1].elapsed_time(ev[2]) * 1e3 for ev in evs] if body.__name__ == "d" else []
    print(json.dumps({"variant": name, "us_per_step": round(best_t, 2), **({"kernel_event_us": round(float(np.mean(ks)), 2)} if ks else {})}), flush=True)
def a(e): search()
def b(e): pack(); search()
def c(e):
    s = torch.cuda.current_stream(); e[0].record(s); pack(); search(); e[3].record(s)
def d(e):
    s = torch.cuda.current_stream(); e[0].record(s); pack(); e[1].record(s); search(); e[2].record(s); e[3].record(s)
for name, body in (("search", a), ("pack+search", b), ("pack+search, step events", c), ("pack+search, step+kernel events", d)):
    run(name, body)
