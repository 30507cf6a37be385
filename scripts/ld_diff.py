"""Debug: compare the tensor-core LD counts with the CUDA-core variant at full size."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import snpgen
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
m, nbits = int(os.environ.get("M", 32768)), int(os.environ.get("NB", 16384))
A = torch.empty((m, snp.snp_words(nbits)), dtype=torch.uint64, device="cuda")
for r0 in range(0, m, 4096):
    gg = snpgen.ld_genotypes(1003, torch.arange(r0, min(m, r0 + 4096), device="cuda"), nbits, structure=True, xp="torch", device="cuda")
    snp.snp_pack(gg, out=A[r0:r0 + gg.shape[0]])
snp.snp_set_variant("popc")
ref = snp.snp_ld_counts(A, A, nbits)
torch.cuda.synchronize()
snp.snp_set_variant("tc")
for trial in range(int(os.environ.get("T", 3))):
    mode = os.environ.get("MODE", "r2")
    if mode == "r2":
        r2, _, got = snp.snp_ld_r2(A, A, nbits, counts=True)
    else:
        got = snp.snp_ld_counts(A, A, nbits)
    torch.cuda.synchronize()
    bad = (got.view(torch.int32) != ref.view(torch.int32))
    nb = int(bad.sum().item())
    print(trial, mode, "kernel", snp.snp_last_kernel(), "mismatches", nb, flush=True)
    if nb:
        idx = bad.nonzero()
        tiles = torch.unique(idx[:, 0] // 128 * 100000 + idx[:, 1] // 128)
        print("  bad tiles:", tiles.numel(), "first", [(int(t) // 100000, int(t) % 100000) for t in tiles[:10]], flush=True)
        r, c = int(idx[0, 0]), int(idx[0, 1])
        print("  first bad", r, c, "got", int(got.view(torch.int32)[r, c]), "ref", int(ref.view(torch.int32)[r, c]), flush=True)
        # rows within tile / cols within tile distribution
        print("  row%128 hist", torch.bincount(idx[:, 0] % 128, minlength=128).nonzero().flatten()[:20].tolist(), flush=True)
        print("  col%128 hist", torch.bincount(idx[:, 1] % 128, minlength=128).nonzero().flatten()[:20].tolist(), flush=True)
