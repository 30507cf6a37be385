"""Tiny-shape pass over every kernel family and instantiation the dispatcher can select,
for compute-sanitizer (memcheck / racecheck / synccheck / initcheck).

    compute-sanitizer --tool memcheck python scripts/sanitize.py

Each call is checked against the oracle as well, so a run also proves the tiny shapes are
right under the sanitizer's serialisation.  Shapes are small (a few tiles, ragged tails)
because the tools slow kernels down by 10-1000x.  Kernel families exercised:
pack / pack_popc / row_popc / best; fastid_tc4 (64- and 32-wide query batches, popD given
and counted in-kernel, 1 op / 2 ops / runtime-coefficient ops, best and counts, the
accumulate instantiation); gemm_tc4 (LD r2+D'+counts, f3 symmetric, swapped two-op
many-query layout, counts accumulate); the CUDA-core POPC kernel; the kind::i8 kernel and
the CTA-pair kernel when SNP_TC_KIND=i8 / SNP_GEMM_X2=1 are set by the caller."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import snpgen  # noqa: E402
import paper_conf_ipps_binderlp19_b200 as snp  # noqa: E402

torch.cuda.set_device(0)
DEV = "cuda"


def dev(g):
    return torch.from_numpy(np.ascontiguousarray(g)).to(DEV)


def u32(t):
    return t.cpu().numpy().astype(np.uint32)


def check(name, got, ref):
    if not np.array_equal(got, ref):
        raise SystemExit(f"MISMATCH {name}")
    print("ok", name, flush=True)


def fastid_cases():
    # (nq, nd, nbits): 64-wide and 32-wide resident batches, ragged tiles and K tails
    for nq, nd, nbits in [(5, 300, 700), (64, 520, 1000), (20, 400, 7000), (3, 129, 64)]:
        db = snpgen.fastid_db(3, np.arange(nd), nbits)
        q, _ = snpgen.fastid_queries(3, nq, nd, nbits)
        D, Q = snp.snp_pack(dev(db)), snp.snp_pack(dev(q))
        pd = snp.snp_row_popc(D, nbits)
        for op in ("and", "xor", "andnot", "notand"):
            check(f"fastid {op} {nq}x{nd}x{nbits} k={snp.snp_last_kernel()}", u32(snp.snp_fastid(Q, D, nbits, op)),
                  oracle.counts(q, db, op))
        acc = snp.snp_fastid(Q, D, nbits, "xor")
        snp.snp_fastid(Q, D, nbits, "xor", out=acc, accumulate=True)
        check(f"fastid accumulate {nq}x{nd}", u32(acc), 2 * oracle.counts(q, db, "xor"))
        for pre in (None, pd):
            for ops in (("xor", "andnot"), ("xor",), ("and", "notand", "xor")):
                counts, best = snp.snp_fastid_search(Q, D, nbits, ops, popD=pre, index_base=3)
                for j, op in enumerate(ops):
                    ref = oracle.counts(q, db, op)
                    check(f"search {ops} {op} pre={pre is not None}", u32(counts[j]), ref)
                    rb, ri = oracle.best(ref, 3)
                    check(f"search best {op}", np.concatenate([u32(best[j][0]).astype(np.int64),
                                                               best[j][1].cpu().numpy()]),
                          np.concatenate([rb.astype(np.int64), ri]))


def ld_cases():
    for m, n, nbits, self_ld in [(300, 300, 1025, True), (130, 257, 700, False), (40, 300, 129, False)]:
        ga = snpgen.ld_genotypes(4, np.arange(m), nbits, structure=True)
        gb = ga if self_ld else snpgen.ld_genotypes(5, np.arange(n), nbits, structure=True)
        A = snp.snp_pack(dev(ga))
        B = A if self_ld else snp.snp_pack(dev(gb))
        r2, dp, cnt = snp.snp_ld_r2(A, B, nbits, dprime=True, counts=True)
        _, _, n_ref = oracle.ld(ga, gb)
        check(f"ld {m}x{n}x{nbits} self={self_ld} k={snp.snp_last_kernel()}", u32(cnt), n_ref)
        c = snp.snp_ld_counts(A, B, nbits)
        snp.snp_ld_counts(A, B, nbits, C=c, accumulate=True)
        check("ld_counts accumulate", u32(c), 2 * n_ref)
    # many-query search: general kernel, swapped two-op layout + best pass
    nq, nd, nbits = 80, 300, 5000
    db = snpgen.fastid_db(6, np.arange(nd), nbits)
    q, _ = snpgen.fastid_queries(6, nq, nd, nbits)
    counts, best = snp.snp_fastid_search(snp.snp_pack(dev(q)), snp.snp_pack(dev(db)), nbits, ("xor", "andnot"))
    for j, op in enumerate(("xor", "andnot")):
        check(f"many-query {op}", u32(counts[j]), oracle.counts(q, db, op))


def round2_kernels():
    # CUDA-core streaming FastID (nq <= 3 in AUTO, <= 4 forced), all ops + best, popD both ways
    for nq, nd, nbits in [(1, 700, 700), (3, 520, 1000), (2, 300, 64)]:
        db = snpgen.fastid_db(13, np.arange(nd), nbits)
        q, _ = snpgen.fastid_queries(13, nq, nd, nbits)
        D, Q = snp.snp_pack(dev(db)), snp.snp_pack(dev(q))
        for pre in (None, snp.snp_row_popc(D, nbits)):
            counts, best = snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot", "and"), popD=pre, index_base=1)
            for j, op in enumerate(("xor", "andnot", "and")):
                check(f"stream {op} {nq}x{nd}x{nbits} k={snp.snp_last_kernel()}", u32(counts[j]), oracle.counts(q, db, op))
    # packed-triangle self-LD (tensor TRI instantiation and CUDA-core), unpack
    for variant in ("auto", "popc"):
        snp.snp_set_variant(variant)
        g = snpgen.ld_genotypes(14, np.arange(300), 777, structure=True)
        A = snp.snp_pack(dev(g))
        r2, dp, cnt = snp.snp_ld_sym(A, 777, r2=True, dprime=True, counts=True)
        check(f"ld_sym {variant} k={snp.snp_last_kernel()}", u32(snp.snp_sym_unpack(cnt, 300)), oracle.ld(g, g)[2])
        _, _, c2 = snp.snp_ld_sym(A, 777, 1, 5, r2=False, counts=True)
        check(f"ld_sym range {variant}", u32(c2), u32(cnt[1:5]))
    snp.snp_set_variant("auto")
    # K-chunked long-profile search (<= 16 queries that do not fit the resident batch)
    nq, nd, nbits = 6, 600, 20000
    db = snpgen.fastid_db(15, np.arange(nd), nbits)
    q, _ = snpgen.fastid_queries(15, nq, nd, nbits)
    counts, _ = snp.snp_fastid_search(snp.snp_pack(dev(q)), snp.snp_pack(dev(db)), nbits, ("xor", "andnot"))
    check("kchunk xor", u32(counts[0]), oracle.counts(q, db, "xor"))
    # threshold list
    qi, cnt, idx, total = snp.snp_fastid_threshold(snp.snp_pack(dev(q)), snp.snp_pack(dev(db)), nbits, "xor",
                                                   tau=9000, capacity=nq * nd)
    ref = oracle.counts(q, db, "xor")
    check("threshold total", np.array([total]), np.array([int((ref <= 9000).sum())]))


def small_kernels():
    g = snpgen.fastid_db(8, np.arange(333), 1000)
    P, pc = snp.snp_pack_popc(dev(g))
    check("pack_popc words", P.cpu().numpy(), oracle.pack(g, snp.snp_words(1000)))
    check("pack_popc popc", u32(pc), oracle.row_popc(g))
    check("row_popc", u32(snp.snp_row_popc(P, 1000)), oracle.row_popc(g))
    c = (np.arange(7 * 300, dtype=np.uint32).reshape(7, 300) * 2654435761 % 97).astype(np.uint32)
    bc, bi = snp.snp_fastid_best(dev(c.view(np.int32)).view(torch.uint32), index_base=2)
    rb, ri = oracle.best(c, 2)
    check("best", np.concatenate([u32(bc).astype(np.int64), bi.cpu().numpy()]),
          np.concatenate([rb.astype(np.int64), ri]))


if __name__ == "__main__":
    small_kernels()
    if os.environ.get("SNP_TC_KIND") != "i8":
        fastid_cases()
        round2_kernels()
    ld_cases()
    snp.snp_set_variant("popc")
    small_kernels()
    ld_cases()
    snp.snp_set_variant("auto")
    torch.cuda.synchronize()
    print("SANITIZE-PASS-DONE")
