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

ct = (ctypes.c_longlong * (3 * 148))()
snp.lib().snp_debug_fastid_cta_times(ct, 3 * 148)
c = np.array(ct, dtype=np.int64).reshape(148, 3)
st = c[:, 0].min()
print("CTA start spread (us):", (c[:, 0].max() - st) / 1e3, " prologue median (us):", np.median(c[:, 1] - c[:, 0]) / 1e3)
print("CTA end (us) min/median/max:", (c[:, 2].min() - st) / 1e3, np.median(c[:, 2] - st) / 1e3, (c[:, 2].max() - st) / 1e3)
ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
ev0.record(); snp.snp_fastid(Q, D, nbits, "xor", out=out); ev1.record(); torch.cuda.synchronize()
print("event-timed single call (ms):", ev0.elapsed_time(ev1))
# timing methodology check
g = torch.cuda.CUDAGraph()
side = torch.cuda.Stream(); side.wait_stream(torch.cuda.current_stream())
with torch.cuda.stream(side):
    snp.snp_fastid(Q, D, nbits, "xor", out=out)
torch.cuda.current_stream().wait_stream(side); torch.cuda.synchronize()
with torch.cuda.graph(g):
    snp.snp_fastid(Q, D, nbits, "xor", out=out)
for _ in range(3): g.replay()
torch.cuda.synchronize()
ev0.record()
for _ in range(20): g.replay()
ev1.record(); torch.cuda.synchronize()
print("20 back-to-back graph replays: per call (ms)", ev0.elapsed_time(ev1) / 20)
ev0.record()
for _ in range(20): snp.snp_fastid(Q, D, nbits, "xor", out=out)
ev1.record(); torch.cuda.synchronize()
print("20 back-to-back eager calls: per call (ms)", ev0.elapsed_time(ev1) / 20)
evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(20)]
for a, b in evs:
    a.record(); g.replay(); b.record()
torch.cuda.synchronize()
print("per-replay events (ms):", [round(a.elapsed_time(b), 4) for a, b in evs][:10])

lt = (ctypes.c_longlong * 128)()
snp.lib().snp_debug_fastid_launch_times(lt, 128)
L = np.array(lt, dtype=np.int64).reshape(64, 2)
L = L[L[:, 0] > 0]
L = L[np.argsort(L[:, 0])]
print("last launches: CTA0 run (us)", ((L[-8:, 1] - L[-8:, 0]) / 1e3).round(1).tolist())
print("              gap to next start (us)", ((L[-7:, 0] - L[-8:-1, 1]) / 1e3).round(1).tolist())
