"""bench-like LD-32K sequence with watchdog record mode (debug)."""
import os, sys, ctypes, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import snpgen
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
L = snp.lib()
rec = (ctypes.c_int * 8)()
mode = int(os.environ.get("WDMODE", "1"))
L.snp_debug_gemm_watchdog(mode, rec)
m, nbits = 32768, 16384
G = torch.empty((m, nbits), dtype=torch.uint8, device="cuda")
for r0 in range(0, m, 2048):
    G[r0:r0 + 2048] = snpgen.ld_genotypes(1003, torch.arange(r0, r0 + 2048, device="cuda"), nbits, structure=True, xp="torch", device="cuda")
B = torch.empty((m, snp.snp_words(nbits)), dtype=torch.uint64, device="cuda")
r2 = torch.empty((m, m), dtype=torch.float32, device="cuda")
cnt = torch.empty((m, m), dtype=torch.uint32, device="cuda")
ws = torch.empty(max(1, snp.snp_ld_workspace_bytes(m, m, nbits)), dtype=torch.uint8, device="cuda")
for i in range(6):
    t0 = time.time()
    snp.snp_pack(G, nbits=nbits, out=B)
    snp.snp_ld_r2(B, B, nbits, r2=r2, counts=cnt, ws=ws)
    try:
        torch.cuda.synchronize()
    except Exception as e:
        print(i, "FAIL", str(e)[:100], flush=True); break
    L.snp_debug_gemm_watchdog(mode, rec)
    print(i, round(time.time() - t0, 3), list(rec), flush=True)
