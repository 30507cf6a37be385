"""Pipeline trace of CTA 0 of the fused FastID search (build with -DFASTID_TRACE2):
per stage it: expander [0] start, [4] after pfull wait, [1] after empty wait, [2] before
full arrive; MMA warp [3] before full wait, [5] after it."""
import ctypes, os, sys
os.environ["SNP_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
nq, nd, nbits = int(os.environ.get("NQ", 64)), int(os.environ.get("ND", 1_000_000)), int(os.environ.get("NBITS", 4096))
w = snp.snp_words(nbits) if os.environ.get("TIGHT") != "1" else (int(os.environ["LDW"]) if os.environ.get("LDW") else 2 * ((nbits + 127) // 128))
D = torch.randint(-2**62, 2**62, (nd, w), dtype=torch.int64, device="cuda").view(torch.uint64)
Q = torch.randint(-2**62, 2**62, (nq, w), dtype=torch.int64, device="cuda").view(torch.uint64)
pd = snp.snp_row_popc(D, nbits)
outs = [torch.empty((nq, nd), dtype=torch.uint32, device="cuda") for _ in range(2)]
mode = os.environ.get("MODE", "search")
for _ in range(3):
    if mode == "search":
        snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), counts=outs, best=True, popD=pd)
    elif mode == "bestonly":
        snp.snp_fastid_search(Q, D, nbits, ("xor",), counts=False, best=True, popD=pd)
    else:
        snp.snp_fastid(Q, D, nbits, "xor", out=outs[0])
torch.cuda.synchronize()
buf = (ctypes.c_longlong * 8192)()
SUF = "" if os.environ.get("SNP_FASTID_KBITS") == "512" else "_k1024"
getattr(snp.lib(), "snp_debug_fastid_trace" + SUF)(buf, 8192)
t = np.array(buf, dtype=np.int64).reshape(1024, 8)
nst = (nbits + (511 if SUF == "" else 1023)) // (512 if SUF == "" else 1024)
ntile = (nd + 127) // 128 // 148
nit = min(1024, ntile * nst)
t = t[:nit]
v = slice(16, nit - 8)
def med(x): return float(np.median(x))
print("mode", mode, "nq", nq, "nd", nd, "nbits", nbits)
print("expander: pfull wait", med(t[v, 4] - t[v, 0]), " empty wait", med(t[v, 1] - t[v, 4]),
      " produce", med(t[v, 2] - t[v, 1]), " iteration", med(np.diff(t[16:nit:4, 0])) if False else "")
print("  produce split: LDS+release", med(t[v, 6] - t[v, 1]), " expand+STTM issue", med(t[v, 7] - t[v, 6]),
      " wait::st", med(t[v, 2] - t[v, 7]))
print("MMA: wait for full", med(t[v, 5] - t[v, 3]), " full-arrive->MMA got", med(t[v, 5] - t[v, 2]),
      " MMA stage interval", med(np.diff(t[16:nit - 8, 5])), " mean", float(np.diff(t[16:nit - 8, 5]).mean()))
print("stage throughput (cycles/stage) over CTA:", (t[nit - 1, 5] - t[8, 5]) / (nit - 9))
for it in range(40, 56):
    r = t[it] - t[0, 0]
    print(it, r[0], r[4], r[1], r[2], "| mma", r[3], r[5])

eb = (ctypes.c_longlong * 1024)()
getattr(snp.lib(), "snp_debug_fastid_etrace" + SUF)(eb, 1024)
e = np.array(eb, dtype=np.int64).reshape(256, 4)[:min(ntile, 256)]
print("per tile (rel. cycles): MMA before acce wait | after | epilogue got accf | epilogue done")
for k in range(20, 30):
    print(k, *(e[k] - e[20, 0]))
print("tile: MMA acce wait", med(e[2:50, 1] - e[2:50, 0]), "mean", float((e[2:50, 1] - e[2:50, 0]).mean()),
      " epilogue busy (accf->done)", med(e[2:50, 3] - e[2:50, 2]), " tile interval (MMA)", med(np.diff(e[2:50, 1])))
for k in range(10, 16):
    print(k, e[k] - e[0, 0])

wb = (ctypes.c_longlong * 4096)()
snp.lib().snp_debug_fastid_wtrace(wb, 4096)
W = np.array(wb, dtype=np.int64).reshape(1024, 4)[:nit]
lag = W[v] - W[v].min(axis=1, keepdims=True)
print("per-warp full-arrive lag behind the group's first warp (median over stages), qa=0..3:",
      [float(np.median(lag[:, k])) for k in range(4)], " slowest-first spread median", float(np.median(lag.max(axis=1))))
print("MMA got stage - slowest warp arrive (median)", med(t[v, 5] - W[v].max(axis=1)))

w2 = (ctypes.c_longlong * 32768)()
snp.lib().snp_debug_fastid_wtrace2(w2, 32768)
X = np.array(w2, dtype=np.int64).reshape(1024, 4, 8)[:nit]
for k in range(4):
    Y = X[v, k]
    print(f"warp qa={k}: pfull wait {med(Y[:,4]-Y[:,0])}  empty wait {med(Y[:,1]-Y[:,4])}  LDS+release {med(Y[:,6]-Y[:,1])}"
          f"  expand+STTM {med(Y[:,7]-Y[:,6])}  wait::st {med(Y[:,2]-Y[:,7])}  start lag vs qa0 {med(Y[:,0]-X[v,0,0])}")
