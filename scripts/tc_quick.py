"""Quick tcgen05-variant sanity check on a tiny shape (run under `timeout`)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle, snpgen
import paper_conf_ipps_binderlp19_b200 as snp

torch.cuda.set_device(0)
snp.snp_set_variant("tc")
for (m, n, nbits) in [(128, 64, 256), (130, 70, 300), (200, 300, 1000), (64, 1000, 4096)]:
    ga = snpgen.fastid_db(5, np.arange(m), nbits)
    gb = snpgen.fastid_db(6, np.arange(n), nbits)
    A = snp.snp_pack(torch.from_numpy(ga).cuda())
    B = snp.snp_pack(torch.from_numpy(gb).cuda())
    for op in ("and", "xor"):
        out = snp.snp_fastid(A, B, nbits, op)
        torch.cuda.synchronize()
        got = out.cpu().numpy().astype(np.int64)
        ref = oracle.counts(ga, gb, op).astype(np.int64)
        bad = (got != ref)
        print(m, n, nbits, op, "variant", snp.snp_last_variant(), "mismatches", int(bad.sum()), "of", bad.size,
              flush=True)
        if bad.any():
            i, j = np.argwhere(bad)[0]
            print("  first bad", i, j, "got", got[i, j], "ref", ref[i, j], "row0 got", got[0, :8], "ref", ref[0, :8])
