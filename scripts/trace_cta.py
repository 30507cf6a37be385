"""Per-CTA timeline of one FastID search call (the bench's fused step): start, main-loop start
(after the query prologue) and end of every CTA, from a -DSNP_PROFILING build (SNP_TRACE=1)."""
import ctypes, os, sys
os.environ["SNP_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
nq = int(os.environ.get("NQ", 64)); nd = int(os.environ.get("ND", 1_000_000)); nbits = int(os.environ.get("K", 4096))
w = snp.snp_words(nbits)
D = torch.randint(-2**62, 2**62, (nd, w), dtype=torch.int64, device="cuda").view(torch.uint64)
Q = torch.randint(-2**62, 2**62, (nq, w), dtype=torch.int64, device="cuda").view(torch.uint64)
pd = snp.snp_row_popc(D, nbits)
outs = [torch.empty((nq, nd), dtype=torch.uint32, device="cuda") for _ in range(2)]
best = [(torch.empty(nq, dtype=torch.uint32, device="cuda"), torch.empty(nq, dtype=torch.int64, device="cuda")) for _ in range(2)]
ws = torch.zeros(snp.snp_fastid_search_workspace_bytes(nq, nd, nbits, 2), dtype=torch.uint8, device="cuda")
call = lambda: snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), counts=outs, best=best, ws=ws, popD=pd)
for _ in range(5): call()
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(); call(); e1.record(); torch.cuda.synchronize()
print("kernel", snp.snp_last_kernel(), "event ms", round(e0.elapsed_time(e1), 4))
ct = (ctypes.c_longlong * (4 * 1024))()
k1024 = os.environ.get("SNP_FASTID_KBITS", "1024") == "1024"
getattr(snp.lib(), "snp_debug_fastid_cta_times" + ("_k1024" if k1024 else ""))(ct, 4 * 1024)
c = np.array(ct, dtype=np.int64).reshape(1024, 4)[:148]
c = c[:, [0, 2, 3, 1]]   # entry, main loop, end, after griddepcontrol.wait
st = c[:, 0].min()
gdc = (c[:, 3] - c[:, 0]) / 1e3
pro = (c[:, 1] - c[:, 3]) / 1e3
end = (c[:, 2] - st) / 1e3
print(f"start spread {(c[:,0].max()-st)/1e3:.2f} us; griddepcontrol.wait min/med/max {gdc.min():.2f} {np.median(gdc):.2f} {gdc.max():.2f} us; "
      f"prologue min/med/max {pro.min():.2f} {np.median(pro):.2f} {pro.max():.2f} us")
print(f"end min/med/max {end.min():.2f} {np.median(end):.2f} {end.max():.2f} us")
ntiles = -(-nd // 128)
tiles = np.array([(ntiles - 1 - b) // 148 + 1 for b in range(148)])
for k in sorted(set(tiles)):
    sel = tiles == k
    print(f"CTAs with {k} tiles: {sel.sum()}, end med {np.median(end[sel]):.2f} us, per-tile {np.median((c[sel,2]-c[sel,1])/1e3/k):.3f} us")
byt = (nd + nq) * w * 8 + 2 * nq * nd * 4
print(f"alg bytes {byt/1e6:.1f} MB; at 6551 GB/s {byt/6551e3:.1f} us")
