"""Quick tensor-core variant sanity check on small shapes (run under `timeout`)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle, snpgen
import paper_conf_ipps_binderlp19_b200 as snp

torch.cuda.set_device(0)
snp.snp_set_variant(os.environ.get("V", "tc"))
bad_total = 0
for (m, n, nbits) in [(128, 64, 256), (130, 70, 300), (200, 300, 1000), (64, 1000, 4096), (300, 129, 2049),
                      (1, 5000, 100), (64, 3000, 4097), (100, 2000, 777), (33, 40000, 256)]:
    ga = snpgen.fastid_db(5, np.arange(m), nbits)
    gb = snpgen.fastid_db(6, np.arange(n), nbits)
    A = snp.snp_pack(torch.from_numpy(ga).cuda())
    B = snp.snp_pack(torch.from_numpy(gb).cuda())
    for op in ("and", "xor", "andnot", "notand"):
        out = snp.snp_fastid(A, B, nbits, op)
        torch.cuda.synchronize()
        got = out.cpu().numpy().astype(np.int64)
        ref = oracle.counts(ga, gb, op).astype(np.int64)
        bad = (got != ref)
        bad_total += int(bad.sum())
        print(m, n, nbits, op, "variant", snp.snp_last_variant(), "mismatches", int(bad.sum()), "of", bad.size,
              flush=True)
        if bad.any():
            i, j = np.argwhere(bad)[0]
            print("  first bad", i, j, "got", got[i, j], "ref", ref[i, j], "row0 got", got[0, :8], "ref", ref[0, :8])
# exactness at long K: all-ones rows -> count = nbits
for nbits in (16384, 100000, 1 << 20):
    g = np.ones((130, nbits), np.uint8)
    A = snp.snp_pack(torch.from_numpy(g).cuda())
    out = snp.snp_fastid(A[:64], A, nbits, "and")
    torch.cuda.synchronize()
    ok = bool((out.cpu().numpy().astype(np.int64) == nbits).all())
    bad_total += 0 if ok else 1
    print("all-ones nbits", nbits, "exact", ok, out.cpu().numpy().astype(np.int64).ravel()[:3], flush=True)
print("TOTAL_BAD", bad_total)
