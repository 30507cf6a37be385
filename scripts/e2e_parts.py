"""Where the FastID-1M end-to-end step's time goes (eager public-API calls, 100 steps back to back):
device-only step, + query H2D, + per-array result D2H, + one merged D2H, + double-buffered H2D."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
nq, nd, nbits = 64, 1_000_000, 4096
w = snp.snp_words(nbits)
D = torch.randint(-2**62, 2**62, (nd, w), dtype=torch.int64, device="cuda").view(torch.uint64)
pd = snp.snp_row_popc(D, nbits)
qhost = torch.randint(0, 2, (nq, nbits), dtype=torch.uint8).pin_memory()
qdev = [torch.empty((nq, nbits), dtype=torch.uint8, device="cuda") for _ in range(2)]
Q = torch.empty((nq, w), dtype=torch.uint64, device="cuda")
outs = [torch.empty((nq, nd), dtype=torch.uint32, device="cuda") for _ in range(2)]
bi_all = torch.empty((2, nq), dtype=torch.int64, device="cuda")
bc_all = torch.empty((2, nq), dtype=torch.uint32, device="cuda")
best = [(bc_all[j], bi_all[j]) for j in range(2)]
res = torch.empty((2, nq), dtype=torch.int64).pin_memory()
resc = torch.empty((2, nq), dtype=torch.uint32).pin_memory()
ws = torch.zeros(snp.snp_fastid_search_workspace_bytes(nq, nd, nbits, 2), dtype=torch.uint8, device="cuda")
copy = torch.cuda.Stream()
ev_copied = [torch.cuda.Event() for _ in range(2)]
ev_packed = [torch.cuda.Event() for _ in range(2)]
def search():
    snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), counts=outs, best=best, ws=ws, popD=pd)
def run(mode, n=100):
    s = torch.cuda.current_stream()
    def one(i):
        if mode == "device":
            snp.snp_pack(qdev[0], nbits=nbits, out=Q); search(); return
        if mode in ("h2d", "h2d+d2h4", "h2d+d2h1"):
            qdev[0].copy_(qhost, non_blocking=True); snp.snp_pack(qdev[0], nbits=nbits, out=Q); search()
        if mode == "dbuf+d2h1":
            b = i % 2
            s.wait_event(ev_copied[b]); snp.snp_pack(qdev[b], nbits=nbits, out=Q); ev_packed[b].record(s)
            with torch.cuda.stream(copy):   # the next step's queries while this step searches
                nb = (i + 1) % 2
                copy.wait_event(ev_packed[nb])
                qdev[nb].copy_(qhost, non_blocking=True); ev_copied[nb].record(copy)
            search()
        if mode == "h2d+d2h4":
            for j in range(2):
                res[j].copy_(best[j][1], non_blocking=True); resc[j].copy_(best[j][0], non_blocking=True)
        if mode in ("h2d+d2h1", "dbuf+d2h1"):
            res.copy_(bi_all, non_blocking=True); resc.copy_(bc_all, non_blocking=True)
    for i in range(3): one(i)
    torch.cuda.synchronize()
    if mode == "dbuf+d2h1":   # prime buffer 0
        qdev[0].copy_(qhost); ev_copied[0].record(s); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for i in range(n): one(i)
    e1.record(s); torch.cuda.synchronize()
    print(json.dumps({"mode": mode, "us_per_step": round(e0.elapsed_time(e1) / n * 1e3, 2)}), flush=True)
for m in ("device", "h2d", "h2d+d2h4", "h2d+d2h1", "dbuf+d2h1"):
    run(m)
