"""Diagnose the CTA-pair LD kernel on small shapes: mismatch pattern vs numpy."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
rng = np.random.default_rng(1)
for (m, n, nbits) in [(256, 128, 512), (256, 128, 64), (512, 256, 1024), (260, 300, 1500)]:
    ga = (rng.random((m, nbits)) < 0.3).astype(np.uint8)
    gb = (rng.random((n, nbits)) < 0.3).astype(np.uint8)
    A = snp.snp_pack(torch.from_numpy(ga).cuda()); B = snp.snp_pack(torch.from_numpy(gb).cuda())
    C = snp.snp_ld_counts(A, B, nbits).cpu().numpy().view(np.int32).astype(np.int64)
    ref = ga.astype(np.int64) @ gb.astype(np.int64).T
    bad = C != ref
    print(m, n, nbits, "kernel", snp.snp_last_kernel(), "bad", int(bad.sum()), "of", bad.size)
    if bad.any():
        rows = np.where(bad.any(1))[0]; cols = np.where(bad.any(0))[0]
        print("  bad rows", rows.min(), rows.max(), len(rows), " bad cols", cols.min(), cols.max(), len(cols))
        i, j = np.argwhere(bad)[0]
        print("  first", i, j, "got", C[i, j], "ref", ref[i, j])
        # is it some other pairing?  check C vs ref with column halves swapped / rows offset
        for name, alt in [("cols+64", np.roll(ref, -64, 1)), ("cols-64", np.roll(ref, 64, 1)),
                          ("rows+128", np.roll(ref, -128, 0)), ("2x", 2 * ref), ("0", 0 * ref)]:
            print("   match", name, float((C == alt)[bad].mean()))
        print("  C[0,:8]", C[0, :8], "ref", ref[0, :8]); print("  C[0,64:72]", C[0, 64:72], "ref", ref[0, 64:72])
        print("  C[128,:8]", C[128, :8], "ref", ref[128, :8])
