"""configs[4] shape sweep: query rows M x database rows N x nbits, CUDA-core (popc) vs
tensor-core (tc) variant, one XOR op with per-query best (snp_fastid_search, best only:
no M x N count matrix, so every shape fits).  Random packed operands (timing only; parity
is the tests' job).  CUDA-event timing: 2 warm-ups, median of 5.  Shapes whose estimated
POPC time exceeds --max-popc-s are skipped for that variant (recorded as null).
Writes one JSON object per shape to stdout and a summary table to stderr."""
import argparse, json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_binderlp19_b200 as snp

ap = argparse.ArgumentParser()
ap.add_argument("--M", default="1,2,4,8,16,32,64,128,256,1024,4096,8192")
ap.add_argument("--N", default="1000000,4000000")
ap.add_argument("--K", default="2048,4096,8192,16384")
ap.add_argument("--max-popc-s", type=float, default=0.4)
ap.add_argument("--tight", action="store_true", help="packed rows of ceil(nbits/64) (even) words, no padding")
ap.add_argument("--counts", action="store_true", help="also write the count matrix (else best only)")
a = ap.parse_args()
torch.cuda.set_device(0)
POPC_RATE = 1.2e14          # comparisons/s, measured (~86% of the POPC pipe peak)

def timeit(fn, reps=5):
    for _ in range(2):
        fn()
    ts = []
    for _ in range(reps):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(); fn(); e.record(); torch.cuda.synchronize()
        ts.append(s.elapsed_time(e))
    ts.sort()
    return ts[len(ts) // 2]

rows = []
for K in [int(x) for x in a.K.split(",")]:
    w = snp.snp_words(K) if not a.tight else ((K + 63) // 64 + 1) // 2 * 2
    for N in [int(x) for x in a.N.split(",")]:
        D = torch.randint(-2**62, 2**62, (N, w), dtype=torch.int64, device="cuda").view(torch.uint64)
        pd = snp.snp_row_popc(D, K)
        for M in [int(x) for x in a.M.split(",")]:
            Q = torch.randint(-2**62, 2**62, (M, w), dtype=torch.int64, device="cuda").view(torch.uint64)
            rec = {"M": M, "N": N, "nbits": K, "cmp": M * N * K, "ldw": w, "counts": bool(a.counts),
                   "bytes": N * w * 8 + (M * N * 4 if a.counts else 0)}
            for v in ("tc", "popc"):
                if v == "popc" and M * N * K / POPC_RATE > a.max_popc_s:
                    rec[v + "_ms"] = None
                    continue
                snp.snp_set_variant(v)
                ws = torch.zeros(snp.snp_fastid_search_workspace_bytes(M, N, K, 1), dtype=torch.uint8, device="cuda")
                outc = [torch.empty((M, N), dtype=torch.uint32, device="cuda")] if a.counts else False
                ms = timeit(lambda: snp.snp_fastid_search(Q, D, K, ("xor",), counts=outc, best=True, ws=ws, popD=pd))
                rec[v + "_ms"] = ms
                rec[v + "_kernel"] = snp.snp_last_kernel()
                del ws
            snp.snp_set_variant("auto")
            t, p = rec["tc_ms"], rec["popc_ms"]
            rec["winner"] = "tc" if p is None or t <= p else "popc"
            rec["tc_cmp_per_s"] = M * N * K / (t / 1e3)
            print(json.dumps(rec), flush=True)
            rows.append(rec)
            del Q
        del D, pd
        torch.cuda.empty_cache()
print("M\\tN\\tnbits\\ttc_ms\\tpopc_ms\\twinner\\ttc Tcmp/s\\tbest GB/s", file=sys.stderr)
for r in rows:
    print(f"{r['M']}\t{r['N']}\t{r['nbits']}\t{r['tc_ms']:.3f}\t{r['popc_ms'] if r['popc_ms'] is None else round(r['popc_ms'], 3)}\t{r['winner']}\t{r['tc_cmp_per_s']/1e12:.0f}\t{r['bytes'] / min(x for x in (r['tc_ms'], r['popc_ms']) if x) / 1e6:.0f}", file=sys.stderr)
