"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, element by element.

Integer outputs must be bit-exact; r2 / D' within 1e-6 relative of the fp64 oracle
and exactly 0 where the oracle is 0 (BASELINE.json north_star).  Inputs come from
snpgen (seeded); the oracle always sees the generator's unpacked bytes, never
anything the CUDA path produced.
"""
import os

import numpy as np
import pytest
import torch

import oracle
import snpgen

pytestmark = pytest.mark.gpu

DEV = "cuda"
VARIANTS = ["popc", "tc"]


@pytest.fixture(scope="module")
def snp(snplib):
    torch.cuda.set_device(0)
    yield snplib
    snplib.snp_set_variant("auto")


def _variant(snp, v):
    snp.snp_set_variant(v)


def to_dev(g):
    return torch.from_numpy(np.ascontiguousarray(g)).to(DEV)


def pack_dev(snp, g, ldw=None, garbage_seed=None):
    """snp_pack on device; optionally fill every padding bit with garbage."""
    nbits = g.shape[1]
    P = snp.snp_pack(to_dev(g), nbits=nbits, ldw=ldw)
    if garbage_seed is not None:
        rng = np.random.default_rng(garbage_seed)
        junk = torch.from_numpy(rng.integers(0, 2**63, size=tuple(P.shape), dtype=np.int64)).to(DEV)
        words = (nbits + 63) // 64
        pv = P.view(torch.int64)
        tail = nbits % 64
        if tail:
            keep = (1 << tail) - 1
            pv[:, words - 1] = (pv[:, words - 1] & keep) | (junk[:, words - 1] & ~keep)
        pv[:, words:] = junk[:, words:]
    return P


def u32(t):
    return t.cpu().numpy().astype(np.uint32)


# ------------------------------------------------------------------ a1 / a2

@pytest.mark.parametrize("nbits", [1, 63, 64, 65, 127, 129, 1000, 4095, 4097])
def test_pack_bit_exact(snp, nbits):
    rng = np.random.default_rng(nbits)
    g = (rng.random((37, nbits)) < 0.4).astype(np.uint8) * snpgen.random_bytes_nonzero((37, nbits), 1)
    ldw = snp.snp_words(nbits) + 2
    P = snp.snp_pack(to_dev(g), ldw=ldw)
    torch.cuda.synchronize()
    assert np.array_equal(P.cpu().numpy(), oracle.pack(g, ldw))


def test_pack_unaligned_rows(snp):
    rng = np.random.default_rng(5)
    nbits = 300
    big = (rng.random((20, nbits + 7)) < 0.5).astype(np.uint8)
    gd = to_dev(big)[:, 3:3 + nbits]          # odd offset and ldg = nbits + 7
    P = snp.snp_pack(gd, nbits=nbits)
    assert np.array_equal(P.cpu().numpy(), oracle.pack(big[:, 3:3 + nbits], snp.snp_words(nbits)))


@pytest.mark.parametrize("nbits", [1, 63, 64, 65, 1000, 4095, 4097, 16384])
@pytest.mark.parametrize("offset", [0, 3])
def test_pack_popc_fused(snp, nbits, offset):
    """a1 + a2 in one pass: packed words and row popcounts both equal the oracle's
    (offset 3 exercises the unaligned byte path; extra ldw words must come back zero)."""
    rows = 4100 if nbits <= 1000 else 70          # more rows than one grid-stride pass at small nbits
    rng = np.random.default_rng(nbits + offset)
    big = (rng.random((rows, nbits + offset)) < 0.3).astype(np.uint8) * \
        snpgen.random_bytes_nonzero((rows, nbits + offset), 2)
    g = big[:, offset:offset + nbits]
    ldw = snp.snp_words(nbits) + 2
    P, pc = snp.snp_pack_popc(to_dev(big)[:, offset:offset + nbits], nbits=nbits, ldw=ldw)
    torch.cuda.synchronize()
    assert np.array_equal(P.cpu().numpy(), oracle.pack(g, ldw))
    assert np.array_equal(u32(pc), oracle.row_popc(g))


def test_pack_popc_empty_and_errors(snp):
    g = torch.zeros((0, 64), dtype=torch.uint8, device=DEV)
    P, pc = snp.snp_pack_popc(g, nbits=64)
    assert P.shape[0] == 0 and pc.shape[0] == 0
    lib = snp.lib()
    g1 = torch.ones((2, 64), dtype=torch.uint8, device=DEV)
    out = torch.empty((2, 8), dtype=torch.uint64, device=DEV)
    assert lib.snp_pack_popc(g1.data_ptr(), 2, 64, 64, out.data_ptr(), 8, None, None) != 0   # popc NULL


@pytest.mark.parametrize("nbits", [1, 64, 65, 1000, 4097])
def test_row_popc_ignores_padding(snp, nbits):
    g = snpgen.fastid_db(7, np.arange(300), nbits)
    P = pack_dev(snp, g, garbage_seed=nbits)
    pc = snp.snp_row_popc(P, nbits)
    assert np.array_equal(u32(pc), oracle.row_popc(g))


# ------------------------------------------------------------------ a3 / a4 counts

SHAPES = [(1, 1, 1), (3, 700, 129), (64, 1000, 4096), (70, 513, 1000), (130, 300, 777),
          (257, 129, 2049)]


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("nq,nd,nbits", SHAPES)
def test_fastid_all_ops(snp, variant, nq, nd, nbits):
    db = snpgen.fastid_db(11, np.arange(nd), nbits)
    q, _ = snpgen.fastid_queries(11, nq, nd, nbits)
    D = pack_dev(snp, db, garbage_seed=1)
    Q = pack_dev(snp, q, garbage_seed=2)
    _variant(snp, variant)
    for op in ("and", "xor", "andnot", "notand"):
        try:
            out = snp.snp_fastid(Q, D, nbits, op)
        except snp.SnpError as e:
            if variant == "tc" and e.status == 2:
                pytest.skip("tc variant does not support this shape")
            raise
        assert np.array_equal(u32(out), oracle.counts(q, db, op)), (op, variant)
    _variant(snp, "auto")


@pytest.mark.parametrize("variant", VARIANTS)
def test_ld_counts_accumulate_and_selfld(snp, variant):
    nbits = 1500
    g = snpgen.ld_genotypes(21, np.arange(260), nbits, structure=True)
    _variant(snp, variant)
    try:
        A = pack_dev(snp, g, garbage_seed=3)
        C = snp.snp_ld_counts(A, A, nbits)              # self-LD, B aliases A
        ref = oracle.counts(g, g, "and")
        assert np.array_equal(u32(C), ref)
        # K split into two chunks with accumulate (paper's gamma += form)
        k1 = 640
        A1 = pack_dev(snp, g[:, :k1])
        A2 = pack_dev(snp, g[:, k1:])
        C2 = snp.snp_ld_counts(A1, A1, k1)
        snp.snp_ld_counts(A2, A2, nbits - k1, C=C2, accumulate=True)
        assert np.array_equal(u32(C2), ref)
    except snp.SnpError as e:
        if variant == "tc" and e.status == 2:
            pytest.skip("tc variant does not support this shape")
        raise
    finally:
        _variant(snp, "auto")


def test_leading_dimensions(snp):
    """ld > words for A, B and C (ldc > n) — only the first n columns are written."""
    nbits = 200
    ga = snpgen.fastid_db(31, np.arange(50), nbits)
    gb = snpgen.fastid_db(32, np.arange(90), nbits)
    A = pack_dev(snp, ga, ldw=12, garbage_seed=4)
    B = pack_dev(snp, gb, ldw=6, garbage_seed=5)
    Cbig = torch.full((50, 100), 0xDEAD, dtype=torch.int32, device=DEV).view(torch.uint32)
    snp.snp_fastid(A, B, nbits, "xor", out=Cbig[:, :90])
    c = u32(Cbig)
    assert np.array_equal(c[:, :90], oracle.counts(ga, gb, "xor"))
    assert (c[:, 90:] == 0xDEAD).all()


# ------------------------------------------------------------------ a5 LD r2 / D'

def check_r2(got, ref):
    got = got.astype(np.float64)
    zero = ref == 0
    assert (got[zero] == 0).all(), "must be exactly 0 where the oracle is 0"
    rel = np.abs(got[~zero] - ref[~zero]) / np.abs(ref[~zero])
    assert rel.size == 0 or rel.max() <= 1e-6, rel.max()


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("m,n,nbits", [(200, 200, 300), (130, 257, 4096), (1, 5, 7), (300, 129, 1025)])
def test_ld_r2_dprime(snp, variant, m, n, nbits):
    ga = snpgen.ld_genotypes(41, np.arange(m), nbits, structure=True)
    gb = snpgen.ld_genotypes(41, np.arange(n) + 50, nbits, structure=True)
    A = pack_dev(snp, ga, garbage_seed=6)
    B = pack_dev(snp, gb, garbage_seed=7)
    _variant(snp, variant)
    try:
        r2, dp, cnt = snp.snp_ld_r2(A, B, nbits, dprime=True, counts=True)
    except snp.SnpError as e:
        if variant == "tc" and e.status == 2:
            pytest.skip("tc variant does not support this shape")
        raise
    finally:
        _variant(snp, "auto")
    r2_ref, dp_ref, n_ref = oracle.ld(ga, gb)
    assert np.array_equal(u32(cnt), n_ref)
    check_r2(r2.cpu().numpy(), r2_ref)
    check_r2(dp.cpu().numpy(), dp_ref)


def test_ld_r2_with_given_popcounts(snp):
    nbits = 513
    g = snpgen.ld_genotypes(43, np.arange(150), nbits, structure=True)
    A = pack_dev(snp, g)
    pa = snp.snp_row_popc(A, nbits)
    r2, _, _ = snp.snp_ld_r2(A, A, nbits, popA=pa, popB=pa)
    check_r2(r2.cpu().numpy(), oracle.ld(g, g)[0])


# ------------------------------------------------------------------ a6 best

def test_best_ties_and_base(snp):
    rng = np.random.default_rng(8)
    c = rng.integers(0, 4, size=(33, 20001)).astype(np.uint32)
    ct = torch.from_numpy(c.view(np.int32)).to(DEV).view(torch.uint32)
    b, i = snp.snp_fastid_best(ct, index_base=123456789)
    rb, ri = oracle.best(c, 123456789)
    assert np.array_equal(u32(b), rb) and np.array_equal(i.cpu().numpy(), ri)
    # unaligned row starts (ldo odd) and nd = 0
    sub = ct[:, 1:]
    b, i = snp.snp_fastid_best(sub)
    rb, ri = oracle.best(c[:, 1:])
    assert np.array_equal(u32(b), rb) and np.array_equal(i.cpu().numpy(), ri)
    b, i = snp.snp_fastid_best(ct[:, :0])
    assert (i.cpu().numpy() == -1).all() and (u32(b) == 0xFFFFFFFF).all()


# ------------------------------------------------------------------ BASELINE configs

def _gen_dev_fastid(seed, nd, nbits, chunk=65536):
    """Full DB generated on device in row chunks and packed by snp_pack."""
    import paper_conf_ipps_binderlp19_b200 as snp
    D = torch.empty((nd, snp.snp_words(nbits)), dtype=torch.uint64, device=DEV)
    for r0 in range(0, nd, chunk):
        r1 = min(nd, r0 + chunk)
        g = snpgen.fastid_db(seed, torch.arange(r0, r1, device=DEV), nbits, xp="torch", device=DEV)
        snp.snp_pack(g, out=D[r0:r1])
    return D


def _sample_cols(n, tile, k, seed):
    rng = np.random.default_rng(seed)
    s = set(rng.integers(0, n, size=k).tolist())
    for b in range(tile, n, tile * 97):
        s.update([b - 1, b, b + 1])
    s.update([0, 1, n - 2, n - 1])
    return np.array(sorted(x for x in s if 0 <= x < n))


@pytest.mark.parametrize("variant", ["auto", "popc"])
def test_cfg2_fastid_1m_sampled(snp, variant):
    """configs[1]: 64 queries x 1,000,000 profiles x 4,096 SNPs, XOR and ANDNOT,
    the launch configuration bench.py times; sampled DB rows vs the oracle, planted
    matches found, best == numpy min/argmin of the produced counts."""
    nq, nd, nbits, seed = 64, 1_000_000, 4096, 1002
    D = _gen_dev_fastid(seed, nd, nbits)
    q, plan = snpgen.fastid_queries(seed, nq, nd, nbits)
    Q = snp.snp_pack(to_dev(q))
    cols = _sample_cols(nd, 128, 600, 9)
    dbs = snpgen.fastid_db(seed, cols, nbits)
    _variant(snp, variant)
    try:
        for op in ("xor", "andnot"):
            out = snp.snp_fastid(Q, D, nbits, op)
            got = u32(out.view(torch.int32)[:, torch.from_numpy(cols).to(DEV)])
            assert np.array_equal(got, oracle.counts(q, dbs, op)), op
            if op == "xor":
                b, i = snp.snp_fastid_best(out)
                full = out.cpu().numpy().astype(np.uint32)
                assert np.array_equal(u32(b), full.min(1))
                assert np.array_equal(i.cpu().numpy(), full.argmin(1))
                for qi, (kind, js, flips) in enumerate(plan):
                    if kind == "copy":
                        assert full[qi, js[0]] == len(flips) and u32(b)[qi] <= len(flips)
            del out
    finally:
        _variant(snp, "auto")


def test_cfg1_ld_full(snp):
    """configs[0]: LD 2,048 SNPs x 4,096 samples, counts + r2 + D', full oracle."""
    m, nbits = 2048, 4096
    g = snpgen.ld_genotypes(1001, np.arange(m), nbits, structure=True)
    A = snp.snp_pack(to_dev(g))
    r2, dp, cnt = snp.snp_ld_r2(A, A, nbits, dprime=True, counts=True)
    r2_ref, dp_ref, n_ref = oracle.ld(g, g)
    assert np.array_equal(u32(cnt), n_ref)
    check_r2(r2.cpu().numpy(), r2_ref)
    check_r2(dp.cpu().numpy(), dp_ref)


def test_cfg3_ld_32k_sampled_rows(snp):
    """configs[2]: LD 32,768 x 32,768 SNPs x 16,384 samples (counts + r2); sampled
    rows including tile boundaries vs the oracle over all columns."""
    m, nbits, seed = 32768, 16384, 1003
    A = torch.empty((m, snp.snp_words(nbits)), dtype=torch.uint64, device=DEV)
    for r0 in range(0, m, 4096):
        gg = snpgen.ld_genotypes(seed, torch.arange(r0, r0 + 4096, device=DEV), nbits,
                                 structure=True, xp="torch", device=DEV)
        snp.snp_pack(gg, out=A[r0:r0 + 4096])
    r2, _, cnt = snp.snp_ld_r2(A, A, nbits, counts=True)
    rows = np.array([0, 1, 127, 128, 4095, 4096, 20000, m - 1])
    ga = snpgen.ld_genotypes(seed, rows, nbits, structure=True)
    gall = np.concatenate([snpgen.ld_genotypes(seed, np.arange(r0, r0 + 1024), nbits, structure=True)
                           for r0 in range(0, m, 1024)])
    r2_ref, _, n_ref = oracle.ld(ga, gall)
    ridx = torch.from_numpy(rows).to(DEV)
    assert np.array_equal(u32(cnt.view(torch.int32)[ridx]), n_ref)
    check_r2(r2[ridx].cpu().numpy(), r2_ref)


@pytest.mark.parametrize("mode", ["counts", "r2"])
def test_cfg3_ld_32k_full_cross_variant(snp, mode):
    """Race detector at full configs[2] size: every one of the 2^30 LD counts of the
    tensor-core kernel equals the CUDA-core kernel's (itself oracle-checked above).
    This is a consistency property over all elements, complementing the sampled
    oracle parity; repeated three times because pipeline races are intermittent."""
    m, nbits = 32768, 16384
    A = torch.empty((m, snp.snp_words(nbits)), dtype=torch.uint64, device=DEV)
    for r0 in range(0, m, 4096):
        gg = snpgen.ld_genotypes(1003, torch.arange(r0, r0 + 4096, device=DEV), nbits,
                                 structure=True, xp="torch", device=DEV)
        snp.snp_pack(gg, out=A[r0:r0 + 4096])
    _variant(snp, "popc")
    ref = snp.snp_ld_counts(A, A, nbits).view(torch.int32)
    _variant(snp, "tc")
    try:
        for _ in range(3):
            if mode == "counts":
                got = snp.snp_ld_counts(A, A, nbits)
            else:
                _, _, got = snp.snp_ld_r2(A, A, nbits, counts=True)
            assert snp.snp_last_kernel().startswith("tc_mxf4")
            assert int((got.view(torch.int32) != ref).sum().item()) == 0
            del got
    finally:
        _variant(snp, "auto")


def test_cfg2_fastid_full_cross_variant(snp):
    """Same race check for the FastID kernel at configs[1] size, all 6.4e7 outputs, XOR."""
    nq, nd, nbits, seed = 64, 1_000_000, 4096, 1002
    D = _gen_dev_fastid(seed, nd, nbits)
    q, _ = snpgen.fastid_queries(seed, nq, nd, nbits)
    Q = snp.snp_pack(to_dev(q))
    _variant(snp, "popc")
    ref = snp.snp_fastid(Q, D, nbits, "xor").view(torch.int32)
    _variant(snp, "tc")
    try:
        for _ in range(3):
            got = snp.snp_fastid(Q, D, nbits, "xor")
            assert snp.snp_last_kernel() == "fastid_mxf4"
            assert int((got.view(torch.int32) != ref).sum().item()) == 0
    finally:
        _variant(snp, "auto")


# ------------------------------------------------------------------ f1 fused search

ALL_OPS = ("and", "xor", "andnot", "notand")
# > 64 queries: 64-query slices of the fused kernel up to 4096 bits (a7), above that the
# general kernel (two ops per pass) + best pass
SEARCH_SHAPES = [(1, 4, 1), (3, 700, 129), (33, 1000, 4096), (64, 2000, 777), (64, 300, 100),
                 (70, 513, 1000), (130, 300, 2049), (100, 3000, 5000),
                 (20, 3000, 8000), (32, 700, 9000),   # <= 32 queries at > 6500 bits: 32-wide kernel
                 (50, 1200, 7000)]                    # 33..64 queries there: two 32-query slices


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("nq,nd,nbits", SEARCH_SHAPES)
@pytest.mark.parametrize("pre", [False, True], ids=["popD_inkernel", "popD_given"])
def test_search_all_ops_counts_and_best(snp, variant, nq, nd, nbits, pre):
    db = snpgen.fastid_db(31, np.arange(nd), nbits)
    q, _ = snpgen.fastid_queries(31, nq, nd, nbits)
    D = pack_dev(snp, db, garbage_seed=5)
    Q = pack_dev(snp, q, garbage_seed=6)
    popD = snp.snp_row_popc(D, nbits) if pre else None
    _variant(snp, variant)
    try:
        counts, best = snp.snp_fastid_search(Q, D, nbits, ALL_OPS, counts=True, best=True, index_base=7,
                                             popD=popD)
        for j, op in enumerate(ALL_OPS):
            ref = oracle.counts(q, db, op)
            assert np.array_equal(u32(counts[j]), ref), (op, variant)
            rb, ri = oracle.best(ref, 7)
            assert np.array_equal(u32(best[j][0]), rb), op
            assert np.array_equal(best[j][1].cpu().numpy(), ri), op
        # best only (no count matrix written), two ops, chunked composition for big nq
        _, best2 = snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), counts=False, best=True, popD=popD)
        for j, op in enumerate(("xor", "andnot")):
            rb, ri = oracle.best(oracle.counts(q, db, op))
            assert np.array_equal(u32(best2[j][0]), rb) and np.array_equal(best2[j][1].cpu().numpy(), ri)
    finally:
        _variant(snp, "auto")


def test_search_stream_dispatch(snp):
    """a7 (profiles/round2/head/sweep/sweep_few.txt): AUTO streams 1-2 queries on the CUDA
    cores, 3 queries only above 12,288 SNPs; the tensor kernel takes 3+ queries otherwise."""
    for nq, nbits, want in ((1, 4096, "popc_stream"), (2, 2048, "popc_stream"), (3, 4096, "fastid_mxf4"),
                            (3, 16384, "popc_stream"), (4, 16384, "fastid_mxf4")):
        db = snpgen.fastid_db(5, np.arange(1000), nbits)
        q, _ = snpgen.fastid_queries(5, nq, 1000, nbits)
        _, best = snp.snp_fastid_search(pack_dev(snp, q), pack_dev(snp, db), nbits, ("xor",), counts=False)
        assert snp.snp_last_kernel() == want, (nq, nbits, snp.snp_last_kernel())
        rb, ri = oracle.best(oracle.counts(q, db, "xor"))
        assert np.array_equal(u32(best[0][0]), rb) and np.array_equal(best[0][1].cpu().numpy(), ri)


def test_search_kernel_choice(snp):
    for nq, nbits in ((32, 8192), (20, 9000)):   # the 32-wide resident-query kernel
        db = snpgen.fastid_db(4, np.arange(2048), nbits)
        q, _ = snpgen.fastid_queries(4, nq, 2048, nbits)
        snp.snp_fastid_search(pack_dev(snp, q), pack_dev(snp, db), nbits)
        assert snp.snp_last_kernel() == "fastid_mxf4", (nq, nbits)
    nbits, nd = 4096, 4096
    db = snpgen.fastid_db(3, np.arange(nd), nbits)
    q, _ = snpgen.fastid_queries(3, 64, nd, nbits)
    snp.snp_fastid_search(pack_dev(snp, q), pack_dev(snp, db), nbits)
    assert snp.snp_last_kernel() == "fastid_mxf4"


@pytest.mark.parametrize("nq", [40, 100])
def test_search_ties_lowest_index_across_ctas(snp, nq):
    """Many exact ties spread over every CTA, warp and lane quarter: the merged best
    must be the lowest database index (reading R4), for counts and best-only.  nq = 40
    runs the FastID kernel, nq = 100 the general kernel's fused two-op best."""
    nbits, nd = 1000, 200_000
    base = snpgen.fastid_db(41, np.arange(13), nbits)
    idx = (np.arange(nd) * 7 + 3) % 13                # row j = base[idx[j]]
    db = base[idx]
    q = base[np.arange(nq) % 13].copy()
    q[::5, :3] ^= 1                                   # some queries have no exact copy
    D = pack_dev(snp, db)
    Q = pack_dev(snp, q)
    for variant in ("auto", "popc"):
        _variant(snp, variant)
        try:
            for counts in (True, False):
                c, best = snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot", "and"), counts=counts,
                                                index_base=1 << 33)
                for j, op in enumerate(("xor", "andnot", "and")):
                    ref = oracle.counts(q, base, op)[:, idx]     # = counts vs every db row
                    rb, ri = oracle.best(ref, 1 << 33)
                    assert np.array_equal(u32(best[j][0]), rb), (variant, op)
                    assert np.array_equal(best[j][1].cpu().numpy(), ri), (variant, op)
        finally:
            _variant(snp, "auto")


@pytest.mark.parametrize("counts", ["both", "first"])
def test_search_general_kernel_best(snp, counts):
    """Many-query search on the general tcgen05 kernel (swapped layout: > 64 queries above
    4096 bits; both ops' counts from one pass, best matches by best.cu).  Exact ties spread
    over every CTA / lane quarter / ragged last tile must give the lowest index; counts and
    bests vs the oracle.  counts="first": op 0 stored, op 1 best-only (chunked path)."""
    nbits, nd, nq = 4500, 20_000, 100
    base = snpgen.fastid_db(47, np.arange(29), nbits)
    idx = (np.arange(nd) * 11 + 5) % 29
    db = base[idx]
    q = base[np.arange(nq) % 29].copy()
    q[::7, :5] ^= 1
    D = pack_dev(snp, db)
    Q = pack_dev(snp, q)
    ops = ("xor", "andnot")
    c = True if counts == "both" else [torch.empty((nq, nd), dtype=torch.uint32, device=DEV), None]
    got, best = snp.snp_fastid_search(Q, D, nbits, ops, counts=c, index_base=3)
    assert snp.snp_last_kernel() in ("tc_mxf4", "popc"), snp.snp_last_kernel()
    for j, op in enumerate(ops):
        ref = oracle.counts(q, base, op)[:, idx]
        if got[j] is not None:
            assert np.array_equal(u32(got[j]), ref), op
        rb, ri = oracle.best(ref, 3)
        assert np.array_equal(u32(best[j][0]), rb), op
        assert np.array_equal(best[j][1].cpu().numpy(), ri), op


def test_search_chunked_composition(snp, monkeypatch):
    """Best-only search for shapes the fused kernel does not take runs in database
    chunks through workspace counts; force small ragged chunks."""
    monkeypatch.setenv("SNP_SEARCH_CHUNK_ROWS", "384")
    nq, nd, nbits = 100, 2000, 300
    db = snpgen.fastid_db(43, np.arange(nd), nbits)
    q, _ = snpgen.fastid_queries(43, nq, nd, nbits)
    _, best = snp.snp_fastid_search(pack_dev(snp, q), pack_dev(snp, db), nbits, ALL_OPS, counts=False,
                                    index_base=5)
    for j, op in enumerate(ALL_OPS):
        rb, ri = oracle.best(oracle.counts(q, db, op), 5)
        assert np.array_equal(u32(best[j][0]), rb) and np.array_equal(best[j][1].cpu().numpy(), ri), op


def test_search_shared_workspace_stays_zero(snp, monkeypatch):
    """snp.h: the search workspace is zero-filled once and every call leaves it zero-filled
    (the fused kernels merge complemented keys with atomicMax, the last CTA clears them; the
    composed paths clear the key region).  ONE workspace through calls that take every path
    (streaming kernel, fused tcgen05 kernel, 64-query slices, the composed chunked path, an
    empty database), each vs the oracle, the workspace checked all-zero after each call."""
    monkeypatch.setenv("SNP_SEARCH_CHUNK_ROWS", "384")
    nbits = 700
    db = snpgen.fastid_db(45, np.arange(3000), nbits)
    D = pack_dev(snp, db)
    shapes = [(1, 3000), (40, 3000), (130, 3000), (100, 2000), (64, 1500), (3, 3000), (40, 0), (40, 2999)]
    need = max(snp.snp_fastid_search_workspace_bytes(nq, nd, nbits, 2) for nq, nd in shapes)
    ws = torch.zeros(need, dtype=torch.uint8, device=DEV)
    for nq, nd in shapes:
        q, _ = snpgen.fastid_queries(46 + nq, nq, max(nd, 1), nbits)
        for counts in (True, False):
            _, best = snp.snp_fastid_search(pack_dev(snp, q), D[:nd], nbits, ("xor", "andnot"), counts=counts,
                                            index_base=7, ws=ws)
            torch.cuda.synchronize()
            for j, op in enumerate(("xor", "andnot")):
                if nd == 0:
                    assert (u32(best[j][0]) == 0xFFFFFFFF).all() and (best[j][1].cpu().numpy() == -1).all()
                    continue
                rb, ri = oracle.best(oracle.counts(q, db[:nd], op), 7)
                assert np.array_equal(u32(best[j][0]), rb), (nq, nd, counts, op, snp.snp_last_kernel())
                assert np.array_equal(best[j][1].cpu().numpy(), ri), (nq, nd, counts, op)
            assert int(ws.count_nonzero()) == 0, (nq, nd, counts, snp.snp_last_kernel())


def test_search_empty_database(snp):
    nbits = 256
    q = snpgen.fastid_db(44, np.arange(5), nbits)
    Q = pack_dev(snp, q)
    D = torch.empty((0, snp.snp_words(nbits)), dtype=torch.uint64, device=DEV)
    _, best = snp.snp_fastid_search(Q, D, nbits, ("xor",), counts=False)
    assert (u32(best[0][0]) == 0xFFFFFFFF).all() and (best[0][1].cpu().numpy() == -1).all()


@pytest.mark.parametrize("variant", ["auto", "popc"])
def test_cfg2_search_1m(snp, variant):
    """configs[1] in the launch configuration bench.py times: ONE search call for XOR +
    ANDNOT with counts and best matches.  Sampled DB columns (every tile-boundary
    neighbourhood included) vs the oracle; best == numpy min/argmin over the full
    count matrices; planted identity copies found."""
    nq, nd, nbits, seed = 64, 1_000_000, 4096, 1002
    D = _gen_dev_fastid(seed, nd, nbits)
    q, plan = snpgen.fastid_queries(seed, nq, nd, nbits)
    Q = snp.snp_pack(to_dev(q))
    cols = _sample_cols(nd, 128, 600, 10)
    dbs = snpgen.fastid_db(seed, cols, nbits)
    _variant(snp, variant)
    popD = snp.snp_row_popc(D, nbits)   # resident with the database, as bench.py prepares it
    try:
        for pd in (None, popD):
            counts, best = snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), popD=pd)
            if variant == "auto":
                assert snp.snp_last_kernel() == "fastid_mxf4"
            for j, op in enumerate(("xor", "andnot")):
                got = u32(counts[j].view(torch.int32)[:, torch.from_numpy(cols).to(DEV)])
                assert np.array_equal(got, oracle.counts(q, dbs, op)), op
                full = counts[j].cpu().numpy().astype(np.uint32)
                assert np.array_equal(u32(best[j][0]), full.min(1)), op
                assert np.array_equal(best[j][1].cpu().numpy(), full.argmin(1)), op
                if op == "xor":
                    for qi, (kind, js, flips) in enumerate(plan):
                        if kind == "copy":
                            assert u32(best[j][0])[qi] <= len(flips)
            _, bonly = snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), counts=False, popD=pd)
            for j in range(2):
                assert torch.equal(bonly[j][0], best[j][0]) and torch.equal(bonly[j][1], best[j][1])
            del counts
    finally:
        _variant(snp, "auto")


def test_ld_cta_pair_kernel_subprocess():
    """The CTA-pair kernels forced (SNP_GEMM_X2=1, read once per process): the general LD
    layout and the whole f3 triangle on ragged shapes spanning several pair tiles and K
    stages (odd tile counts: a phantom lane block), counts + r2 + D' vs the oracle."""
    import subprocess
    import sys
    code = r'''
import numpy as np, torch, sys
sys.path.insert(0, ".")
import oracle, snpgen
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
for (m, n, nbits) in [(512, 256, 1024), (700, 300, 1500), (2048, 2048, 4096)]:
    ga = snpgen.ld_genotypes(51, np.arange(m), nbits, structure=True)
    gb = snpgen.ld_genotypes(52, np.arange(n), nbits, structure=True)
    A = snp.snp_pack(torch.from_numpy(ga).cuda()); B = snp.snp_pack(torch.from_numpy(gb).cuda())
    r2, dp, cnt = snp.snp_ld_r2(A, B, nbits, dprime=True, counts=True)
    r2_ref, dp_ref, n_ref = oracle.ld(ga, gb)
    assert np.array_equal(cnt.cpu().numpy().view(np.uint32), n_ref), (m, n, nbits)
    assert snp.snp_last_kernel() == "tc_mxf4_pair", snp.snp_last_kernel()
    for got, ref in ((r2, r2_ref), (dp, dp_ref)):
        g = got.cpu().numpy().astype(np.float64); z = ref == 0
        assert (g[z] == 0).all() and (np.abs(g[~z] - ref[~z]) <= 1e-6 * np.abs(ref[~z])).all()
# the whole f3 triangle on CTA pairs: odd / even tile counts (T = 1 has a phantom lane
# block), ragged rows, one and several K stages, D' and counts-only
from paper_conf_ipps_binderlp19_b200.multigpu import sym_tile_coords
for (m, nbits) in [(1, 5), (100, 64), (129, 700), (300, 1025), (640, 2000), (1000, 4100)]:
    g = snpgen.ld_genotypes(53, np.arange(m), nbits, structure=True)
    A = snp.snp_pack(torch.from_numpy(g).cuda())
    r2, dp, cnt = snp.snp_ld_sym(A, nbits, r2=True, dprime=True, counts=True)
    assert snp.snp_last_kernel() == "tc_mxf4_sym_pair", snp.snp_last_kernel()
    _, _, c2 = snp.snp_ld_sym(A, nbits, r2=False, counts=True)
    r2_ref, dp_ref, n_ref = oracle.ld(g, g)
    C, C2, R2, DP = (x.cpu().numpy() for x in (cnt, c2, r2, dp))
    for t in range(snp.snp_sym_tiles(m)):
        I, J = sym_tile_coords(m, t)
        rs, cs = slice(128 * I, min(m, 128 * I + 128)), slice(128 * J, min(m, 128 * J + 128))
        h, w = rs.stop - rs.start, cs.stop - cs.start
        for X in (C, C2):
            assert np.array_equal(X[t, :h, :w].view(np.uint32), n_ref[rs, cs]), (m, t)
            assert (X[t, h:, :] == 0).all() and (X[t, :, w:] == 0).all()
        for X, ref in ((R2, r2_ref[rs, cs]), (DP, dp_ref[rs, cs])):
            gx = X[t, :h, :w].astype(np.float64); z = ref == 0
            assert (gx[z] == 0).all() and (np.abs(gx[~z] - ref[~z]) <= 1e-6 * np.abs(ref[~z])).all(), (m, t)
print("ok")
'''
    env = dict(os.environ, SNP_GEMM_X2="1")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-c", code], cwd=root, env=env, capture_output=True, text=True,
                       timeout=600)
    assert r.returncode == 0 and "ok" in r.stdout, r.stdout + r.stderr


@pytest.mark.parametrize("m,nbits", [(2300, 1025), (2200, 64), (300, 1025), (129, 64), (1000, 700)])
def test_selfld_symmetric_mirror(snp, m, nbits):
    """f3: self-LD (B aliases A) computes only the upper-triangle tiles and mirrors the
    off-diagonal ones (from two tile rows up, ragged last tile here); every output
    (counts, r2, D') vs the oracle, and the matrices are exactly symmetric."""
    g = snpgen.ld_genotypes(61, np.arange(m), nbits, structure=True)
    A = pack_dev(snp, g, garbage_seed=9)
    r2, dp, cnt = snp.snp_ld_r2(A, A, nbits, dprime=True, counts=True)
    r2_ref, dp_ref, n_ref = oracle.ld(g, g)
    c = u32(cnt)
    assert np.array_equal(c, n_ref) and np.array_equal(c, c.T)
    check_r2(r2.cpu().numpy(), r2_ref)
    check_r2(dp.cpu().numpy(), dp_ref)
    x = snp.snp_fastid(A, A, nbits, "xor")                 # symmetric op through the same path
    assert np.array_equal(u32(x), oracle.counts(g, g, "xor"))


@pytest.mark.parametrize("with_pop", [False, True])
def test_stream_search_chunks(snp, with_pop):
    """f2: database in pinned host memory streamed in ragged chunks through two device
    buffers; per-query best of XOR and ANDNOT vs the oracle (lowest index on ties)."""
    from paper_conf_ipps_binderlp19_b200.stream import stream_search
    nq, nd, nbits = 40, 5000, 777
    db = snpgen.fastid_db(71, np.arange(nd), nbits)
    q, _ = snpgen.fastid_queries(71, nq, nd, nbits)
    q[3] = db[4500]                                    # exact copy in the last chunk
    D_host = pack_dev(snp, db).cpu().pin_memory()
    pop = snp.snp_row_popc(D_host.to(DEV), nbits).cpu().pin_memory() if with_pop else None
    Q = pack_dev(snp, q)
    res = stream_search(Q, D_host, nbits, ("xor", "andnot"), popD_host=pop, chunk_rows=1500, index_base=11)
    torch.cuda.synchronize()
    for j, op in enumerate(("xor", "andnot")):
        rb, ri = oracle.best(oracle.counts(q, db, op), 11)
        assert np.array_equal(res[j][0].cpu().numpy().astype(np.uint32), rb), op
        assert np.array_equal(res[j][1].cpu().numpy(), ri), op


@pytest.mark.parametrize("nq,nd,chunk", [(40, 1536 + 128, 1536), (64, 4 * 1024 + 100, 1024), (100, 2048 + 40, 2048)])
def test_stream_search_ragged_small_last_chunk(snp, nq, nd, chunk):
    """f2 with a last chunk so short (< 4 nq rows, or < 256 rows past 64 queries) that the
    dispatcher leaves the fused kernel for a path with a larger workspace: the scratch is
    sized for every distinct chunk length, so the stream completes and matches the oracle."""
    from paper_conf_ipps_binderlp19_b200.stream import stream_search
    nbits = 900
    db = snpgen.fastid_db(72, np.arange(nd), nbits)
    q, _ = snpgen.fastid_queries(72, nq, nd, nbits)
    q[1] = db[nd - 3]                                  # exact copy in the short last chunk
    D_host = pack_dev(snp, db).cpu().pin_memory()
    res = stream_search(pack_dev(snp, q), D_host, nbits, ("xor", "andnot"), chunk_rows=chunk)
    torch.cuda.synchronize()
    for j, op in enumerate(("xor", "andnot")):
        rb, ri = oracle.best(oracle.counts(q, db, op))
        assert np.array_equal(res[j][0].cpu().numpy().astype(np.uint32), rb), op
        assert np.array_equal(res[j][1].cpu().numpy(), ri), op


def test_search_general_kernel_forced(snp, monkeypatch):
    """More than 64 queries at few bits with the 64-query slicing disabled: the general
    kernel's paired-op pass (counts of two ops from one AND count) + best pass."""
    monkeypatch.setenv("SNP_SEARCH_SLICES", "0")
    nq, nd, nbits = 70, 513, 1000
    db = snpgen.fastid_db(81, np.arange(nd), nbits)
    q, _ = snpgen.fastid_queries(81, nq, nd, nbits)
    counts, best = snp.snp_fastid_search(pack_dev(snp, q), pack_dev(snp, db), nbits, ALL_OPS, index_base=3)
    assert snp.snp_last_kernel() == "tc_mxf4"
    for j, op in enumerate(ALL_OPS):
        ref = oracle.counts(q, db, op)
        assert np.array_equal(u32(counts[j]), ref), op
        rb, ri = oracle.best(ref, 3)
        assert np.array_equal(u32(best[j][0]), rb) and np.array_equal(best[j][1].cpu().numpy(), ri), op


def test_cfg4_fastid_20m_full_size():
    """configs[3] at full size on one GPU (1,024 queries x 20,000,000 profiles x 8,192
    SNPs, the launch configuration bench.py times for the best matches): planted identity
    copies are found (best count <= flips at the planted row, which at these sizes no other
    row approaches), every best index is in range, and a 1M-row database slice of the XOR /
    ANDNOT counts matches the oracle on sampled rows."""
    import paper_conf_ipps_binderlp19_b200 as snpm
    nq, nd, nbits, seed = 1024, 20_000_000, 8192, 1004
    D = _gen_dev_fastid(seed, nd, nbits, chunk=262144)
    q, plan = snpgen.fastid_queries(seed, nq, nd, nbits)
    Q = snpm.snp_pack(to_dev(q))
    _, best = snpm.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), counts=False)
    bx, ix = u32(best[0][0]), best[0][1].cpu().numpy()
    assert ((ix >= 0) & (ix < nd)).all()
    for qi, (kind, js, flips) in enumerate(plan):
        if kind == "copy":
            assert bx[qi] <= len(flips) and ix[qi] == js[0], (qi, bx[qi], ix[qi], js)
    # counts on a slice of the database: all queries x rows [r0, r0 + 1M), sampled rows
    r0 = 7_000_000
    Dsl = D[r0:r0 + 1_000_000]
    cols = _sample_cols(1_000_000, 128, 200, 11)
    dbs = snpgen.fastid_db(seed, cols + r0, nbits)
    for op in ("xor", "andnot"):
        out = snpm.snp_fastid(Q, Dsl, nbits, op)
        got = u32(out.view(torch.int32)[:, torch.from_numpy(cols).to(DEV)])
        assert np.array_equal(got, oracle.counts(q, dbs, op)), op
        del out


def test_fuzz_shapes(snp):
    """Seeded random shapes through every dispatch path (fused / sliced / general search,
    f3 symmetric and full-tile LD, swapped and unswapped layouts) vs the oracle."""
    rng = np.random.default_rng(2024)
    cases = [(int(rng.integers(1, 200)), int(rng.integers(256, 4000)), int(rng.integers(1, 5000)))
             for _ in range(8)]
    for nq, nd, nbits in cases:
        db = snpgen.fastid_db(91, np.arange(nd), nbits)
        q, _ = snpgen.fastid_queries(91, nq, nd, nbits)
        counts, best = snp.snp_fastid_search(pack_dev(snp, q, garbage_seed=1), pack_dev(snp, db, garbage_seed=2),
                                             nbits, ("xor", "andnot"), index_base=5)
        for j, op in enumerate(("xor", "andnot")):
            ref = oracle.counts(q, db, op)
            assert np.array_equal(u32(counts[j]), ref), (nq, nd, nbits, op)
            rb, ri = oracle.best(ref, 5)
            assert np.array_equal(u32(best[j][0]), rb) and np.array_equal(best[j][1].cpu().numpy(), ri), \
                (nq, nd, nbits, op)
    for m, n, nbits, self_ld in [(2200, 2200, 97, True), (2400, 2400, 33, True), (700, 300, 1300, False),
                                 (300, 700, 64, False), (1, 1, 1, True), (130, 130, 5000, True)]:
        ga = snpgen.ld_genotypes(92, np.arange(m), nbits, structure=True)
        gb = ga if self_ld else snpgen.ld_genotypes(93, np.arange(n), nbits, structure=True)
        A = pack_dev(snp, ga, garbage_seed=3)
        B = A if self_ld else pack_dev(snp, gb, garbage_seed=4)
        r2, dp, cnt = snp.snp_ld_r2(A, B, nbits, dprime=True, counts=True)
        r2_ref, dp_ref, n_ref = oracle.ld(ga, gb)
        assert np.array_equal(u32(cnt), n_ref), (m, n, nbits)
        check_r2(r2.cpu().numpy(), r2_ref)
        check_r2(dp.cpu().numpy(), dp_ref)
        r2b, _, _ = snp.snp_ld_r2(A, B, nbits)                 # r2 only (no counts / D')
        check_r2(r2b.cpu().numpy(), r2_ref)


@pytest.mark.parametrize("self_ld", [True, False])
def test_ld_unaligned_output_rows(snp, self_ld):
    """Output row strides that are not a multiple of 4 words (no 16-byte row copies): the
    scalar full-block and mirror epilogues, counts + r2 + D' and counts + r2, vs the oracle."""
    m, nbits = 300, 1025
    ga = snpgen.ld_genotypes(95, np.arange(m), nbits, structure=True)
    gb = ga if self_ld else snpgen.ld_genotypes(96, np.arange(m), nbits, structure=True)
    A = pack_dev(snp, ga)
    B = A if self_ld else pack_dev(snp, gb)
    r2_ref, dp_ref, n_ref = oracle.ld(ga, gb)
    for ld in (m + 2, m + 3):
        for want_dp in (True, False):
            r2b = torch.full((m, ld), -1.0, dtype=torch.float32, device=DEV)
            cb = torch.zeros((m, ld), dtype=torch.int32, device=DEV).view(torch.uint32)
            dpb = torch.full((m, ld), -2.0, dtype=torch.float32, device=DEV) if want_dp else None
            snp.snp_ld_r2(A, B, nbits, r2=r2b[:, :m], counts=cb[:, :m], dprime=None if dpb is None else dpb[:, :m])
            assert np.array_equal(u32(cb)[:, :m], n_ref), (ld, want_dp)
            check_r2(r2b[:, :m].cpu().numpy(), r2_ref)
            assert (r2b[:, m:].cpu().numpy() == -1.0).all()
            if dpb is not None:
                check_r2(dpb[:, :m].cpu().numpy(), dp_ref)


def _sym_blocks_ref(g, m):
    r2, dp, n = oracle.ld(g, g)
    return r2, dp, n


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("m,nbits", [(300, 1025), (128, 64), (129, 700), (2300, 1025), (1, 5),
                                    (3000, 515), (3100, 700)])   # the last two: CTA pairs in AUTO
def test_ld_sym_packed_tiles(snp, variant, m, nbits):
    """f3 packed triangle: every tile of the row-major upper triangle equals the oracle's
    block (counts bit-exact, r2 / D' within 1e-6 relative, exactly 0 where the oracle is 0);
    entries of ragged tiles past m are 0; snp_sym_unpack rebuilds the full matrices."""
    from paper_conf_ipps_binderlp19_b200.multigpu import sym_tile_coords
    g = snpgen.ld_genotypes(63, np.arange(m), nbits, structure=True)
    A = pack_dev(snp, g, garbage_seed=5)
    _variant(snp, variant)
    try:
        r2, dp, cnt = snp.snp_ld_sym(A, nbits, r2=True, dprime=True, counts=True)
        kern = snp.snp_last_kernel()
    finally:
        _variant(snp, "auto")
    assert kern in (("tc_mxf4_sym", "tc_mxf4_sym_pair") if variant == "tc" else ("popc",))
    r2_ref, dp_ref, n_ref = oracle.ld(g, g)
    R2, DP, C = r2.cpu().numpy(), dp.cpu().numpy(), u32(cnt)
    for t in range(snp.snp_sym_tiles(m)):
        I, J = sym_tile_coords(m, t)
        rs, cs = slice(128 * I, min(m, 128 * I + 128)), slice(128 * J, min(m, 128 * J + 128))
        h, w = rs.stop - rs.start, cs.stop - cs.start
        assert np.array_equal(C[t, :h, :w], n_ref[rs, cs]), (t, I, J)
        check_r2(R2[t, :h, :w], r2_ref[rs, cs])
        check_r2(DP[t, :h, :w], dp_ref[rs, cs])
        for X in (R2, DP):
            assert (X[t, h:, :] == 0).all() and (X[t, :, w:] == 0).all()
        assert (C[t, h:, :] == 0).all() and (C[t, :, w:] == 0).all()
    full = snp.snp_sym_unpack(cnt, m)
    assert np.array_equal(u32(full), n_ref)
    fr2 = snp.snp_sym_unpack(r2, m)
    check_r2(fr2.cpu().numpy(), r2_ref)


@pytest.mark.parametrize("variant", VARIANTS)
def test_ld_sym_tile_ranges_match_whole(snp, variant):
    """One rank's share: tiles [lo, hi) of an uneven plan equal the same tiles of the whole
    call (counts-only and r2-only forms), for every rank of a 3-way plan."""
    m, nbits = 700, 513
    g = snpgen.ld_genotypes(64, np.arange(m), nbits, structure=True)
    A = pack_dev(snp, g)
    _variant(snp, variant)
    try:
        r2w, _, cw = snp.snp_ld_sym(A, nbits, counts=True)
        b = snp.snp_shard_plan_sym(m, 3)
        for r in range(3):
            _, _, c = snp.snp_ld_sym(A, nbits, b[r], b[r + 1], r2=False, counts=True)
            r2, _, _ = snp.snp_ld_sym(A, nbits, b[r], b[r + 1])
            assert torch.equal(c, cw[b[r]:b[r + 1]]), r
            assert torch.equal(r2, r2w[b[r]:b[r + 1]]), r
    finally:
        _variant(snp, "auto")
    assert np.array_equal(u32(snp.snp_sym_unpack(cw, m)), oracle.ld(g, g)[2])


STREAM_SHAPES = [(1, 1, 1), (1, 300, 63), (2, 257, 512), (3, 5000, 513), (4, 4100, 4097), (4, 70000, 2048),
                 (2, 1000, 20000), (1, 256, 130000)]


@pytest.mark.parametrize("nq,nd,nbits", STREAM_SHAPES)
@pytest.mark.parametrize("pre", [False, True], ids=["popD_inkernel", "popD_given"])
def test_fastid_stream_all_ops_counts_and_best(snp, nq, nd, nbits, pre):
    """CUDA-core streaming kernel (nq <= 4): every op's counts and best matches from one
    database pass vs the oracle, ragged 256-row tiles and K tails, garbage in the padding,
    database popcounts given or counted in-kernel; snp_fastid (single op) and accumulate."""
    db = snpgen.fastid_db(81, np.arange(nd), nbits)
    q, _ = snpgen.fastid_queries(81, nq, nd, nbits)
    if nd > 10:
        q[0] = db[nd // 2]                                 # an exact match (count 0)
    D = pack_dev(snp, db, garbage_seed=3)
    Q = pack_dev(snp, q, garbage_seed=4)
    pd = snp.snp_row_popc(D, nbits) if pre else None
    ops = ("and", "xor", "andnot", "notand")
    # AUTO takes the streaming kernel for <= 2 queries (a7); the forced CUDA-core variant for <= 4
    _variant(snp, "auto" if nq <= 2 else "popc")
    try:
        counts, best = snp.snp_fastid_search(Q, D, nbits, ops, index_base=7, popD=pd)
        assert snp.snp_last_kernel() == "popc_stream"
        out = snp.snp_fastid(Q, D, nbits, "xor", popD=pd)
        assert snp.snp_last_kernel() == "popc_stream"
        snp.snp_fastid(Q, D, nbits, "xor", out=out, popD=pd, accumulate=True)
    finally:
        _variant(snp, "auto")
    for j, op in enumerate(ops):
        ref = oracle.counts(q, db, op)
        assert np.array_equal(u32(counts[j]), ref), op
        rb, ri = oracle.best(ref, 7)
        assert np.array_equal(u32(best[j][0]), rb) and np.array_equal(best[j][1].cpu().numpy(), ri), op
    assert np.array_equal(u32(out), 2 * oracle.counts(q, db, "xor"))


def test_fastid_stream_ties_lowest_index(snp):
    """Equal minimum counts in many tiles and CTAs: the lowest database index wins (R4)."""
    nq, nd, nbits = 3, 300_000, 256
    db = snpgen.fastid_db(82, np.arange(nd), nbits)
    q, _ = snpgen.fastid_queries(82, nq, nd, nbits)
    for r in (299_999, 150_000, 40_001, 40_000, 77_777):
        db[r] = q[1]                                       # exact copies of query 1 everywhere
    D, Q = pack_dev(snp, db), pack_dev(snp, q)
    _variant(snp, "popc")
    try:
        _, best = snp.snp_fastid_search(Q, D, nbits, ("xor",), counts=False)
        assert snp.snp_last_kernel() == "popc_stream"
    finally:
        _variant(snp, "auto")
    assert int(best[0][0][1]) == 0 and int(best[0][1][1]) == 40_000
    rb, ri = oracle.best(oracle.counts(q, db, "xor"))
    assert np.array_equal(u32(best[0][0]), rb) and np.array_equal(best[0][1].cpu().numpy(), ri)


@pytest.mark.parametrize("with_host_out", [False, True])
def test_stream_ld_sym_end_to_end(snp, with_host_out):
    """f2 for LD: packed matrix in pinned host memory streamed in reverse row blocks, tile
    rows computed as their blocks land, outputs optionally copied back block by block;
    counts / r2 equal the oracle's (through snp_sym_unpack) and the resident snp_ld_sym."""
    from paper_conf_ipps_binderlp19_b200.stream import stream_ld_sym
    m, nbits = 900, 1100
    g = snpgen.ld_genotypes(66, np.arange(m), nbits, structure=True)
    A_dev = pack_dev(snp, g)
    A_host = A_dev.cpu().pin_memory()
    nt = snp.snp_sym_tiles(m)
    host = ({"r2": torch.empty((nt, 128, 128), dtype=torch.float32).pin_memory(),
             "counts": torch.empty((nt, 128, 128), dtype=torch.int32).pin_memory()} if with_host_out else None)
    outs, _ = stream_ld_sym(A_host, nbits, block_tiles=2, out_host=host)
    torch.cuda.synchronize()
    r2_ref, _, n_ref = oracle.ld(g, g)
    assert np.array_equal(u32(snp.snp_sym_unpack(outs["counts"], m)), n_ref)
    check_r2(snp.snp_sym_unpack(outs["r2"], m).cpu().numpy(), r2_ref)
    r2w, _, cw = snp.snp_ld_sym(A_dev, nbits, counts=True)
    assert torch.equal(cw, outs["counts"]) and torch.equal(r2w, outs["r2"])
    if host is not None:
        assert np.array_equal(host["counts"].numpy().view(np.uint32), u32(cw))
        assert torch.equal(host["r2"], r2w.cpu())


@pytest.mark.parametrize("ldw", [2, 4, 6])
@pytest.mark.parametrize("nq", [1, 3, 32, 100])
def test_narrow_rows_short_profiles(snp, ldw, nq):
    """The paper's FastID profiles are 128-1024 SNPs (Fig. 8): packed rows as
    narrow as 2 words (16 bytes, no padding to the recommended 64) are valid input for every
    op, the fused search and LD; results vs the oracle."""
    nbits = 64 * ldw - 5
    nd = 3000
    db = snpgen.fastid_db(83, np.arange(nd), nbits)
    q, _ = snpgen.fastid_queries(83, nq, nd, nbits)
    D = pack_dev(snp, db, ldw=ldw, garbage_seed=1)
    Q = pack_dev(snp, q, ldw=ldw, garbage_seed=2)
    counts, best = snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), index_base=2)
    for j, op in enumerate(("xor", "andnot")):
        ref = oracle.counts(q, db, op)
        assert np.array_equal(u32(counts[j]), ref), (op, snp.snp_last_kernel())
        rb, ri = oracle.best(ref, 2)
        assert np.array_equal(u32(best[j][0]), rb) and np.array_equal(best[j][1].cpu().numpy(), ri), op
    assert np.array_equal(u32(snp.snp_fastid(Q, D, nbits, "and")), oracle.counts(q, db, "and"))
    g = snpgen.ld_genotypes(84, np.arange(300), nbits, structure=True)
    A = pack_dev(snp, g, ldw=ldw)
    r2, _, cnt = snp.snp_ld_r2(A, A, nbits, counts=True)
    r2_ref, _, n_ref = oracle.ld(g, g)
    assert np.array_equal(u32(cnt), n_ref)
    check_r2(r2.cpu().numpy(), r2_ref)
    _, _, ct = snp.snp_ld_sym(A, nbits, r2=False, counts=True)
    assert np.array_equal(u32(snp.snp_sym_unpack(ct, 300)), n_ref)


@pytest.mark.parametrize("nq,nbits", [(8, 20000), (16, 13000), (12, 30000), (5, 33000)])
@pytest.mark.parametrize("mode", ["counts", "best_only", "mixed"])
def test_search_kchunked_long_profiles(snp, nq, nbits, mode, monkeypatch):
    """<= 64 queries whose expanded batch does not fit the FastID kernel: K-chunked passes that
    add their counts (one DB read in total); every op's counts and best matches vs the oracle,
    with counts stored, best-only (workspace count chunks over row blocks) and mixed."""
    monkeypatch.setenv("SNP_SEARCH_CHUNK_ROWS", "1024")      # several row blocks at this size
    nd = 2600
    db = snpgen.fastid_db(85, np.arange(nd), nbits)
    q, _ = snpgen.fastid_queries(85, nq, nd, nbits)
    q[0] = db[2100]
    D = pack_dev(snp, db, garbage_seed=6)
    Q = pack_dev(snp, q, garbage_seed=7)
    ops = ("and", "xor", "andnot", "notand")
    counts = {"counts": True, "best_only": False,
              "mixed": [torch.empty((nq, nd), dtype=torch.uint32, device=DEV), None, None,
                        torch.empty((nq, nd), dtype=torch.uint32, device=DEV)]}[mode]
    c, best = snp.snp_fastid_search(Q, D, nbits, ops, counts=counts, index_base=4)
    assert snp.snp_last_kernel() == "fastid_mxf4"
    for j, op in enumerate(ops):
        ref = oracle.counts(q, db, op)
        if c[j] is not None:
            assert np.array_equal(u32(c[j]), ref), (op, mode)
        rb, ri = oracle.best(ref, 4)
        assert np.array_equal(u32(best[j][0]), rb) and np.array_equal(best[j][1].cpu().numpy(), ri), (op, mode)


@pytest.mark.parametrize("nq,nd,nbits,tau", [(3, 5000, 700, 0), (40, 3000, 1000, 400), (70, 2000, 4097, 1700),
                                             (1, 1, 64, 64)])
@pytest.mark.parametrize("op", ["xor", "andnot"])
def test_fastid_threshold_matches(snp, nq, nd, nbits, tau, op, monkeypatch):
    """f1 threshold form: the set of (query, row, count) with count <= tau equals the oracle's,
    across database row chunks (small chunks forced), with index_base; truncation keeps the
    total count."""
    monkeypatch.setenv("SNP_SEARCH_CHUNK_ROWS", "768")
    db = snpgen.fastid_db(86, np.arange(nd), nbits)
    q, _ = snpgen.fastid_queries(86, nq, nd, nbits)
    if nd > 10:
        q[0] = db[nd - 5]
    Q, D = pack_dev(snp, q, garbage_seed=8), pack_dev(snp, db, garbage_seed=9)
    qi, cnt, idx, total = snp.snp_fastid_threshold(Q, D, nbits, op, tau=tau, capacity=nq * nd, index_base=10)
    ref = oracle.counts(q, db, op)
    rq, rd = np.nonzero(ref <= tau)
    assert total == len(rq)
    got = sorted(zip(qi.cpu().tolist(), (idx - 10).cpu().tolist(), cnt.cpu().tolist()))
    want = sorted(zip(rq.tolist(), rd.tolist(), ref[rq, rd].tolist()))
    assert got == want
    if total > 3:
        _, _, idx2, total2 = snp.snp_fastid_threshold(Q, D, nbits, op, tau=tau, capacity=3)
        assert total2 == total and idx2.numel() == 3


def test_fuzz_round2_paths(snp):
    """Seeded random shapes through the round-2 paths vs the oracle: the CUDA-core streaming
    kernel (1-4 queries), K-chunked long profiles (<= 16 queries), packed-triangle tile ranges,
    and threshold lists."""
    from paper_conf_ipps_binderlp19_b200.multigpu import sym_tile_coords
    rng = np.random.default_rng(2025)
    for _ in range(4):
        nq, nd, nbits = int(rng.integers(1, 5)), int(rng.integers(1, 3000)), int(rng.integers(1, 6000))
        db = snpgen.fastid_db(97, np.arange(nd), nbits)
        q, _ = snpgen.fastid_queries(97, nq, nd, nbits)
        _variant(snp, "popc")
        try:
            counts, best = snp.snp_fastid_search(pack_dev(snp, q, garbage_seed=1), pack_dev(snp, db, garbage_seed=2),
                                                 nbits, ("xor", "notand"), index_base=3)
        finally:
            _variant(snp, "auto")
        for j, op in enumerate(("xor", "notand")):
            ref = oracle.counts(q, db, op)
            assert np.array_equal(u32(counts[j]), ref), (nq, nd, nbits, op)
            rb, ri = oracle.best(ref, 3)
            assert np.array_equal(u32(best[j][0]), rb) and np.array_equal(best[j][1].cpu().numpy(), ri)
    for _ in range(3):
        nq, nd, nbits = int(rng.integers(2, 17)), int(rng.integers(200, 1500)), int(rng.integers(14000, 40000))
        db = snpgen.fastid_db(98, np.arange(nd), nbits)
        q, _ = snpgen.fastid_queries(98, nq, nd, nbits)
        counts, _ = snp.snp_fastid_search(pack_dev(snp, q, garbage_seed=3), pack_dev(snp, db, garbage_seed=4), nbits,
                                          ("andnot",))
        assert np.array_equal(u32(counts[0]), oracle.counts(q, db, "andnot")), (nq, nd, nbits)
    for _ in range(3):
        m, nbits = int(rng.integers(1, 700)), int(rng.integers(1, 3000))
        g = snpgen.ld_genotypes(99, np.arange(m), nbits, structure=True)
        A = pack_dev(snp, g, garbage_seed=5)
        T = snp.snp_sym_tiles(m)
        lo = int(rng.integers(0, T))
        hi = int(rng.integers(lo + 1, T + 1))
        r2, _, cnt = snp.snp_ld_sym(A, nbits, lo, hi, counts=True)
        r2_ref, _, n_ref = oracle.ld(g, g)
        for u, t in enumerate(range(lo, hi)):
            I, J = sym_tile_coords(m, t)
            rs, cs = slice(128 * I, min(m, 128 * I + 128)), slice(128 * J, min(m, 128 * J + 128))
            assert np.array_equal(u32(cnt[u])[:rs.stop - rs.start, :cs.stop - cs.start], n_ref[rs, cs]), (m, nbits, t)
            check_r2(r2[u].cpu().numpy()[:rs.stop - rs.start, :cs.stop - cs.start], r2_ref[rs, cs])
    nq, nd, nbits = 9, 2500, 333
    db = snpgen.fastid_db(100, np.arange(nd), nbits)
    q, _ = snpgen.fastid_queries(100, nq, nd, nbits)
    qi, cnt, idx, total = snp.snp_fastid_threshold(pack_dev(snp, q), pack_dev(snp, db), nbits, "xor", tau=150,
                                                   capacity=nq * nd)
    ref = oracle.counts(q, db, "xor")
    rq, rd = np.nonzero(ref <= 150)
    assert total == len(rq)
    assert sorted(zip(qi.cpu().tolist(), idx.cpu().tolist())) == sorted(zip(rq.tolist(), rd.tolist()))


def test_cfg2_fastid_1m_full_oracle(snp):
    """configs[1] in full (SURVEY §8d "cfg 1 and 2: full oracle"): every one of the 2 x 64 x 1M
    XOR / ANDNOT counts of the bench's search call (database popcounts given, the fused FastID
    kernel) equals the bit-by-bit CPU oracle, database regenerated on the host in row chunks
    from the same seeded generator; best matches equal the oracle's argmin over all rows."""
    nq, nd, nbits, seed = 64, 1_000_000, 4096, 1002
    D = _gen_dev_fastid(seed, nd, nbits)
    q, _ = snpgen.fastid_queries(seed, nq, nd, nbits)
    Q = snp.snp_pack(to_dev(q))
    counts, best = snp.snp_fastid_search(Q, D, nbits, ("xor", "andnot"), popD=snp.snp_row_popc(D, nbits))
    assert snp.snp_last_kernel() == "fastid_mxf4"
    got = [c.cpu().numpy().view(np.uint32) for c in counts]
    del counts, D
    torch.cuda.empty_cache()
    ref_best = [np.full(nq, 0xFFFFFFFF, dtype=np.int64), np.zeros(nq, dtype=np.int64)], \
               [np.full(nq, 0xFFFFFFFF, dtype=np.int64), np.zeros(nq, dtype=np.int64)]
    step = 125_000
    for r0 in range(0, nd, step):
        db = snpgen.fastid_db(seed, np.arange(r0, min(nd, r0 + step)), nbits)
        for j, op in enumerate(("xor", "andnot")):
            ref = oracle.counts(q, db, op)
            assert np.array_equal(got[j][:, r0:r0 + ref.shape[1]], ref), (op, r0)
            m, a = ref.min(1).astype(np.int64), ref.argmin(1) + r0
            better = m < ref_best[j][0]
            ref_best[j][1][better] = a[better]
            ref_best[j][0][better] = m[better]
    for j in range(2):
        assert np.array_equal(best[j][0].cpu().numpy().astype(np.int64), ref_best[j][0])
        assert np.array_equal(best[j][1].cpu().numpy(), ref_best[j][1])
