"""Pins for the CPU oracle (run with -m "not gpu").

The oracle (oracle/snp_oracle.c) is checked against things other than itself:
hand-worked fixtures (tests/golden/, cited), closed forms on exhaustive k-bit
inputs (Python int popcount), library routines (numpy integer matmul, scipy
Hamming distance, numpy corrcoef, numpy argmin) and invariants the mathematics
fixes (symmetry, diagonal, K-additivity, permutation invariance, identities
popc(a^b) = popc(a)+popc(b)-2popc(a&b), popc(a&~b) = popc(a)-popc(a&b),
complete-LD and sign properties of D').
"""
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle
import snpgen

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _bits(s):
    return np.array([int(ch) for ch in s], dtype=np.uint8)


def _load_ld_fixture():
    rows, pairs = {}, []
    with open(os.path.join(GOLD, "appc_ld.txt")) as f:
        for line in f:
            if line.startswith("#") or not line.strip():
                continue
            t = line.split()
            if t[0] == "row":
                rows[t[1]] = (_bits(t[2]), int(t[3], 16), int(t[4]))
            else:
                pairs.append((t[1], t[2], int(t[3]), int(t[4]), int(t[5]),
                              Fraction(t[6]), Fraction(t[7])))
    return rows, pairs


def _load_fastid_fixture():
    q, db = None, []
    with open(os.path.join(GOLD, "appc_fastid.txt")) as f:
        for line in f:
            if line.startswith("#") or not line.strip():
                continue
            t = line.split()
            if t[0] == "query":
                q = _bits(t[1])
            else:
                db.append((t[1], _bits(t[2]), tuple(int(v) for v in t[3:7])))
    return q, db


# ------------------------------------------------------------ pack / unpack

def test_pack_hand_examples():
    rows, _ = _load_ld_fixture()
    for name, (bits, word, pc) in rows.items():
        p = oracle.pack(bits[None, :])
        assert p.shape == (1, 1)
        assert int(p[0, 0]) == word, name
        assert int(oracle.row_popc(bits[None, :])[0]) == pc
        assert (oracle.unpack(p, 8)[0] == bits).all()


@pytest.mark.parametrize("nbits", [1, 7, 63, 64, 65, 127, 128, 129, 300])
def test_pack_roundtrip_and_zero_padding(nbits):
    rng = np.random.default_rng(nbits)
    g = (rng.random((5, nbits)) < 0.4).astype(np.uint8)
    ldw = (nbits + 63) // 64 + 2
    p = oracle.pack(g, ldw)
    assert (oracle.unpack(p, nbits) == g).all()
    # padding bits past nbits and the extra words are zero (Fig. 2)
    full = oracle.unpack(p, 64 * ldw)
    assert (full[:, nbits:] == 0).all()
    # bit k is in word k//64 at position k%64 (little-endian LSB-first, reading R1),
    # checked against an independent Python-int construction
    for r in range(5):
        v = sum(1 << k for k in range(nbits) if g[r, k])
        words = [(v >> (64 * w)) & ((1 << 64) - 1) for w in range(ldw)]
        assert [int(x) for x in p[r]] == words


def test_nonzero_byte_is_minor_allele():
    rng = np.random.default_rng(3)
    g = (rng.random((6, 100)) < 0.5).astype(np.uint8)
    g2 = g * snpgen.random_bytes_nonzero(g.shape, 4)
    assert (oracle.pack(g2) == oracle.pack(g)).all()
    assert (oracle.counts(g2, g2, "xor") == oracle.counts(g, g, "xor")).all()


# ------------------------------------------------------------ counts

def _all_vectors(k):
    v = np.arange(1 << k)
    return ((v[:, None] >> np.arange(k)[None, :]) & 1).astype(np.uint8)


@pytest.mark.parametrize("k", [1, 3, 6, 8])
def test_counts_exhaustive_closed_forms(k):
    g = _all_vectors(k)
    n = 1 << k
    mask = (1 << k) - 1
    pc = np.array([bin(i).count("1") for i in range(n)])
    I = np.arange(n)[:, None]
    J = np.arange(n)[None, :]
    popc = np.vectorize(lambda x: bin(int(x)).count("1"))
    exp = {
        "and": popc(I & J),
        "xor": popc(I ^ J),
        "andnot": popc(I & (~J & mask)),
        "notand": popc(J & (~I & mask)),
    }
    for op, e in exp.items():
        c = oracle.counts(g, g, op)
        assert (c == e).all(), op
    # row sums of the AND table: popcount(i) * 2^(k-1)
    c = oracle.counts(g, g, "and")
    assert (c.sum(1) == pc * (1 << (k - 1))).all()


def test_counts_vs_library_routines():
    from scipy.spatial.distance import cdist
    rng = np.random.default_rng(7)
    ga = (rng.random((37, 203)) < 0.3).astype(np.uint8)
    gb = (rng.random((29, 203)) < 0.45).astype(np.uint8)
    a64, b64 = ga.astype(np.int64), gb.astype(np.int64)
    assert (oracle.counts(ga, gb, "and") == a64 @ b64.T).all()
    ham = np.rint(cdist(ga, gb, "hamming") * 203).astype(np.int64)
    assert (oracle.counts(ga, gb, "xor") == ham).all()
    assert (oracle.counts(ga, gb, "andnot") == a64 @ (1 - b64).T).all()
    assert (oracle.counts(ga, gb, "notand") == (1 - a64) @ b64.T).all()


def test_counts_identities_and_invariants():
    rng = np.random.default_rng(11)
    ga = (rng.random((20, 150)) < 0.25).astype(np.uint8)
    gb = (rng.random((17, 150)) < 0.4).astype(np.uint8)
    pa = oracle.row_popc(ga).astype(np.int64)
    pb = oracle.row_popc(gb).astype(np.int64)
    c_and = oracle.counts(ga, gb, "and").astype(np.int64)
    c_xor = oracle.counts(ga, gb, "xor").astype(np.int64)
    # popc(a^b) = popc(a) + popc(b) - 2 popc(a&b)
    assert (c_xor == pa[:, None] + pb[None, :] - 2 * c_and).all()
    # popc(a&~b) = popc(a) - popc(a&b);  popc(b&~a) = popc(b) - popc(a&b)
    assert (oracle.counts(ga, gb, "andnot") == pa[:, None] - c_and).all()
    assert (oracle.counts(ga, gb, "notand") == pb[None, :] - c_and).all()
    # Eq. 3 literal form == rewrite r & ~m is what andnot computes; swapping
    # operand roles swaps andnot and notand
    assert (oracle.counts(gb, ga, "andnot") == oracle.counts(ga, gb, "notand").T).all()
    # self-LD symmetry and diagonal = row popcount
    s = oracle.counts(ga, ga, "and")
    assert (s == s.T).all() and (np.diag(s) == pa).all()
    assert (np.diag(oracle.counts(ga, ga, "xor")) == 0).all()
    # K-additivity and invariance under a common K permutation
    k1 = 61
    c1 = oracle.counts(ga[:, :k1], gb[:, :k1], "and").astype(np.int64)
    c2 = oracle.counts(ga[:, k1:], gb[:, k1:], "and").astype(np.int64)
    assert (c1 + c2 == c_and).all()
    perm = rng.permutation(150)
    for op in ("and", "xor", "andnot", "notand"):
        assert (oracle.counts(ga[:, perm], gb[:, perm], op) == oracle.counts(ga, gb, op)).all()


def test_fastid_hand_examples():
    q, db = _load_fastid_fixture()
    d = np.stack([b for _, b, _ in db])
    for j, op in enumerate(("and", "xor", "andnot", "notand")):
        c = oracle.counts(q[None, :], d, op)[0]
        assert [int(v) for v in c] == [e[j] for _, _, e in db], op
    # a zero XOR count is a positive match
    assert oracle.counts(q[None, :], d, "xor")[0, 0] == 0


def test_counts_empty_and_bad_op():
    g = np.zeros((0, 10), np.uint8)
    assert oracle.counts(g, np.ones((3, 10), np.uint8)).shape == (0, 3)
    with pytest.raises(KeyError):
        oracle.counts(np.ones((1, 4), np.uint8), np.ones((1, 4), np.uint8), "or")


# ------------------------------------------------------------ LD r2 / D'

def test_ld_hand_examples():
    rows, pairs = _load_ld_fixture()
    for a, b, nab, num, den, r2f, dpf in pairs:
        ga, gb = rows[a][0][None, :], rows[b][0][None, :]
        r2, dp, cnt = oracle.ld(ga, gb)
        assert int(cnt[0, 0]) == nab
        assert r2[0, 0] == pytest.approx(float(r2f), rel=1e-15, abs=0)
        assert dp[0, 0] == pytest.approx(float(dpf), rel=1e-15, abs=0)
        if r2f == 0:
            assert r2[0, 0] == 0.0
        if dpf == 0:
            assert dp[0, 0] == 0.0


def test_r2_is_squared_pearson():
    rng = np.random.default_rng(5)
    ga = (rng.random((25, 97)) < rng.uniform(0.05, 0.5, (25, 1))).astype(np.uint8)
    gb = (rng.random((19, 97)) < rng.uniform(0.05, 0.5, (19, 1))).astype(np.uint8)
    r2, dp, _ = oracle.ld(ga, gb)
    for i in range(25):
        for j in range(19):
            x, y = ga[i].astype(float), gb[j].astype(float)
            if x.std() == 0 or y.std() == 0:
                assert r2[i, j] == 0.0
                continue
            ref = np.corrcoef(x, y)[0, 1] ** 2
            assert r2[i, j] == pytest.approx(ref, rel=1e-12, abs=1e-15)
            # sign(D') = sign(correlation), D'^2 >= r2, bounds
            corr = np.corrcoef(x, y)[0, 1]
            if abs(corr) > 1e-12:
                assert np.sign(dp[i, j]) == np.sign(corr)
            assert dp[i, j] ** 2 >= r2[i, j] - 1e-12
            assert -1.0 <= dp[i, j] <= 1.0 and 0.0 <= r2[i, j] <= 1.0 + 1e-15


def test_dprime_complete_ld_iff_empty_haplotype_cell():
    g = _all_vectors(6)  # all 64 vectors of 6 samples
    r2, dp, nab = oracle.ld(g, g)
    pc = oracle.row_popc(g).astype(np.int64)
    n = 6
    for i in range(64):
        for j in range(64):
            na, nb, c = pc[i], pc[j], int(nab[i, j])
            poly = 0 < na < n and 0 < nb < n
            cells = [c, na - c, nb - c, n - na - nb + c]  # haplotype counts AB, Ab, aB, ab
            num = n * c - na * nb
            if not poly:
                assert r2[i, j] == 0.0 and dp[i, j] == 0.0
            elif num != 0:
                assert (abs(dp[i, j]) == pytest.approx(1.0, abs=1e-15)) == (min(cells) == 0)
            else:
                assert dp[i, j] == 0.0 and r2[i, j] == 0.0
    # D'(a,a) = 1 and D'(a,~a) = -1 ; r2 = 1 for both (polymorphic a)
    comp = 1 - g
    r2c, dpc, _ = oracle.ld(g, comp)
    for i in range(1, 63):
        assert dp[i, i] == pytest.approx(1.0) and r2[i, i] == pytest.approx(1.0)
        assert dpc[i, i] == pytest.approx(-1.0) and r2c[i, i] == pytest.approx(1.0)
    # complementing one SNP flips the sign of D' and keeps r2; D' symmetric
    assert np.allclose(r2, r2.T) and np.allclose(dp, dp.T)
    r2x, dpx, _ = oracle.ld(comp, g)
    assert np.allclose(r2x, r2) and np.allclose(dpx, -dp)


def test_ld_from_counts_matches_ld():
    # the per-pair statistic depends only on (n, nA, nB, nAB)
    rng = np.random.default_rng(9)
    ga = (rng.random((6, 40)) < 0.3).astype(np.uint8)
    gb = (rng.random((5, 40)) < 0.5).astype(np.uint8)
    r2, dp, nab = oracle.ld(ga, gb)
    pa, pb = oracle.row_popc(ga), oracle.row_popc(gb)
    for i in range(6):
        for j in range(5):
            rr, dd = oracle.ld_from_counts(40, int(pa[i]), int(pb[j]), int(nab[i, j]))
            assert rr == r2[i, j] and dd == dp[i, j]


# ------------------------------------------------------------ best match

def test_best_vs_argmin_and_ties():
    rng = np.random.default_rng(2)
    c = rng.integers(0, 5, size=(13, 40)).astype(np.uint32)
    b, idx = oracle.best(c, index_base=1000)
    assert (b == c.min(1)).all()
    assert (idx == np.argmin(c, axis=1) + 1000).all()   # argmin returns the first (lowest) index
    b0, i0 = oracle.best(np.zeros((2, 0), np.uint32))
    assert (i0 == -1).all() and (b0 == 0xFFFFFFFF).all()


def test_planted_queries_are_found():
    nd, nbits, nq = 300, 256, 10
    db = snpgen.fastid_db(1002, np.arange(nd), nbits)
    q, plan = snpgen.fastid_queries(1002, nq, nd, nbits)
    xor = oracle.counts(q, db, "xor")
    notand = oracle.counts(q, db, "notand")
    for i, (kind, js, flips) in enumerate(plan):
        if kind == "copy":
            assert xor[i, js[0]] == len(flips) <= 8
            b, _ = oracle.best(xor[i:i + 1])
            assert b[0] <= len(flips)
        else:
            # every contributor of a mixture has no minor allele absent from it
            for j in js:
                assert notand[i, j] == 0
