"""Per-CTA timeline of the LD GEMM (build with -DSNP_PROFILING -DGEMM_TRACE3, run with
SNP_LIB_PATH pointing at it): the LD step (pack_popc + snp_ld_sym) of configs[0] / [2];
prints, per event, the min / median / max over CTAs in us from the earliest CTA entry."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
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
def step():
    snp.snp_pack_popc(G, nbits=nbits, out=B, popc=pop)
    snp.snp_ld_sym(B, nbits, popA=pop, r2=r2, counts=cnt)
for _ in range(5):
    step()
torch.cuda.synchronize()
e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
e[0].record(); snp.snp_pack_popc(G, nbits=nbits, out=B, popc=pop); e[1].record()
snp.snp_ld_sym(B, nbits, popA=pop, r2=r2, counts=cnt); e[2].record(); torch.cuda.synchronize()
print(f"events: pack_popc {e[0].elapsed_time(e[1])*1e3:.1f} us, gemm {e[1].elapsed_time(e[2])*1e3:.1f} us")
step(); torch.cuda.synchronize()
buf = (ctypes.c_longlong * 8192)()
snp.lib().snp_debug_gemm_cta(buf, 8192)
grid = min(nt, 148)
t = np.array(buf, dtype=np.int64).reshape(1024, 8)[:grid, :7].astype(np.float64)
t0 = t[:, 0].min()
names = ["entry", "setup done", "gdc.wait done", "1st stage in", "1st acc ready", "last tile stored", "exit"]
for k, nm in enumerate(names):
    x = (t[:, k] - t0) / 1e3
    print(f"{nm:18s} min {x.min():7.2f}  med {np.median(x):7.2f}  max {x.max():7.2f} us")

b2 = (ctypes.c_longlong * 8192)()
snp.lib().snp_debug_gemm_cta2(b2, 8192)
u = np.array(b2, dtype=np.int64).reshape(1024, 8)[:grid, :4].astype(np.float64)
for k, nm in enumerate(["TMEM ld half 0", "block half 0 done", "TMEM ld half 1", "block half 1 done"]):
    x = (u[:, k] - t0) / 1e3
    print(f"{nm:18s} min {x.min():7.2f}  med {np.median(x):7.2f}  max {x.max():7.2f} us")
