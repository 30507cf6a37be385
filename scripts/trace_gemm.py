"""Per-tile pipeline trace of the general tcgen05 kernel, CTA 0 (build with -DSNP_PROFILING
-DGEMM_TRACE4, run with SNP_TRACE=1 and SNP_LIB_PATH at that build): many-query FastID search
(both ops' counts, the configs[3] shape on a smaller database) or LD.  Prints per tile: MMA
waiting for a free accumulator, the MMA stream, the MMA's waits for expanded stages, and the
epilogue's drain time."""
import ctypes, os, sys
os.environ["SNP_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
nq, nd, nbits = int(os.environ.get("NQ", 1024)), int(os.environ.get("ND", 2_000_000)), int(os.environ.get("NBITS", 8192))
w = snp.snp_words(nbits)
if os.environ.get("MODE") == "ldrows":   # LD of ND x ND SNPs in the row layout (r2 + counts)
    A = torch.randint(-2**62, 2**62, (nd, w), dtype=torch.int64, device="cuda").view(torch.uint64)
    B = A.clone()   # not aliased: the general (non-mirrored) layout
    for _ in range(2):
        r2, _, cnt = snp.snp_ld_r2(A, B, nbits, counts=True)
    nq = nd   # single: (nd/128)^2 tiles over 148 CTAs; pair: (nd/256)(nd/128) over 74 clusters
elif os.environ.get("MODE") == "ld":   # packed-triangle self-LD of ND SNPs (r2 + counts)
    A = torch.randint(-2**62, 2**62, (nd, w), dtype=torch.int64, device="cuda").view(torch.uint64)
    pa = snp.snp_row_popc(A, nbits)
    nt = snp.snp_sym_tiles(nd)
    r2 = torch.empty((nt, 128, 128), dtype=torch.float32, device="cuda")
    cnt = torch.empty((nt, 128, 128), dtype=torch.uint32, device="cuda")
    for _ in range(2):
        snp.snp_ld_sym(A, nbits, popA=pa, r2=r2, counts=cnt)
    nq = 128 * nt // ((nd + 127) // 128)   # so that the tile count below is the triangle's
else:
    D = torch.randint(-2**62, 2**62, (nd, w), dtype=torch.int64, device="cuda").view(torch.uint64)
    Q = torch.randint(-2**62, 2**62, (nq, w), dtype=torch.int64, device="cuda").view(torch.uint64)
    pd = snp.snp_row_popc(D, nbits)
    outs = [torch.empty((nq, nd), dtype=torch.uint32, device="cuda") for _ in range(2)]
    for _ in range(2):
        snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), counts=outs, best=False, popD=pd)
torch.cuda.synchronize()
print("kernel", snp.snp_last_kernel())
buf = (ctypes.c_longlong * 16384)()
snp.lib().snp_debug_gemm_trace(buf, 16384)
t = np.array(buf, dtype=np.int64).reshape(2048, 8)
ntl = int(((nd + 127) // 128) * ((nq + 127) // 128) / 148)
v = slice(4, min(ntl - 2, 2040))
med = lambda x: float(np.median(x))
print(f"tiles per CTA ~{ntl}")
print("MMA wait for free accumulator", med(t[v, 1] - t[v, 0]), "  MMA stream (acc free -> accf commit)", med(t[v, 2] - t[v, 1]),
      "  of which waiting for stages", med(t[v, 5]))
print("epilogue: accf seen -> acc drained (warp 0)", med(t[v, 4] - t[v, 3]), " (warp 7)", med(t[v, 7] - t[v, 6]),
      "  commit -> epilogue sees it", med(t[v, 3] - t[v, 2]))
print("tile interval (MMA commits)", med(np.diff(t[v, 2])))
