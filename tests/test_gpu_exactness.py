"""GPU parity on every path the dispatcher can select at long K and large n.

The tensor variants multiply bits as e2m1 nibbles and accumulate in fp32 TMEM
(DESIGN.md §6).  Counts are exact integers only if the MMA's accumulation is exact
for integers of the size reached, so these tests drive large, odd, random counts
(rows of density ~0.97 give AND counts ~0.94·nbits) through every kernel at nbits
from 2^14 to 2^24 and compare them with the oracle element by element (exact integer
update γ += Σ POPC, §III).  They also cover the LD epilogue's wide
(n > 46340) integer path (r², D′ from exact n·nAB − nA·nB, §II.A) and the
``kind::i8`` kernel, which is otherwise only reached at nbits ≥ 2^24.
"""
import os
import subprocess
import sys

import numpy as np
import pytest
import torch

import oracle

pytestmark = pytest.mark.gpu

DEV = "cuda"
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def snp(snplib):
    torch.cuda.set_device(0)
    yield snplib
    snplib.snp_set_variant("auto")


def dense_rows(seed, rows, nbits, p):
    """0/1 bytes, row r has density p[r % len(p)] (seeded)."""
    rng = np.random.default_rng(seed)
    dens = np.asarray(p, dtype=np.float64)[np.arange(rows) % len(p)][:, None]
    out = np.empty((rows, nbits), dtype=np.uint8)
    step = max(1, (1 << 24) // nbits)
    for r0 in range(0, rows, step):
        r1 = min(rows, r0 + step)
        out[r0:r1] = rng.random((r1 - r0, nbits), dtype=np.float32) < dens[r0:r1]
    return out


def u32(t):
    return t.cpu().numpy().astype(np.uint32)


def check_rel(got, ref, tol=1e-6):
    g = np.asarray(got, dtype=np.float64)
    z = ref == 0
    assert (g[z] == 0).all(), "nonzero where the oracle is 0"
    err = np.abs(g[~z] - ref[~z]) / np.abs(ref[~z])
    assert err.size == 0 or err.max() <= tol, f"max rel err {err.max():.3e}"


# Long-K tensor paths: odd nbits just above the powers where an fp32 sum would need more
# mantissa bits, densities giving counts near nbits (and a few sparse rows for spread).
LONG_K = [16385, 65537, (1 << 20) + 1, (1 << 23) - 1]


@pytest.mark.parametrize("nbits", LONG_K)
def test_long_k_fastid_counts_all_ops(snp, nbits):
    """FastID shape (few queries, more DB rows) at long K: every op vs the oracle.  Counts
    here are random, odd and up to ~0.97·nbits (above 2^14 from nbits = 2^14 + 1)."""
    nq, nd = (8, 300) if nbits < (1 << 22) else (4, 40)
    q = dense_rows(nbits, nq, nbits, [0.97, 0.99, 0.6])
    db = dense_rows(nbits + 1, nd, nbits, [0.97, 0.995, 0.9, 0.3])
    Q = snp.snp_pack(torch.from_numpy(q).to(DEV))
    D = snp.snp_pack(torch.from_numpy(db).to(DEV))
    ref_and = oracle.counts(q, db, "and")
    assert ref_and.max() > 0.9 * nbits and (ref_and & 1).any()
    for op in ("and", "xor", "andnot", "notand"):
        out = snp.snp_fastid(Q, D, nbits, op)
        assert snp.snp_last_variant() == "tc", "long-K FastID is routed to the tensor variant"
        ref = ref_and if op == "and" else oracle.counts(q, db, op)
        got = u32(out)
        bad = np.argwhere(got != ref)
        assert bad.size == 0, (op, snp.snp_last_kernel(), len(bad), got[tuple(bad[0])], ref[tuple(bad[0])])


@pytest.mark.parametrize("nbits", LONG_K)
def test_long_k_ld_r2_counts(snp, nbits):
    """LD shape (general tensor kernel, f3 symmetric when self) at long K: AND counts,
    r², D′ vs the oracle; n = nbits exceeds 46340 from 65537 up (wide integer path)."""
    m = 160 if nbits < (1 << 22) else 48
    g = dense_rows(nbits + 2, m, nbits, [0.97, 0.5, 0.99, 0.03, 0.8])
    A = snp.snp_pack(torch.from_numpy(g).to(DEV))
    r2, dp, cnt = snp.snp_ld_r2(A, A, nbits, dprime=True, counts=True)
    kern = snp.snp_last_kernel()
    r2_ref, dp_ref, n_ref = oracle.ld(g, g)
    got = u32(cnt)
    bad = np.argwhere(got != n_ref)
    assert bad.size == 0, (kern, len(bad), got[tuple(bad[0])], n_ref[tuple(bad[0])])
    check_rel(r2.cpu().numpy(), r2_ref)
    check_rel(dp.cpu().numpy(), dp_ref)


@pytest.mark.parametrize("nbits", [16385, (1 << 20) + 1])
def test_long_k_many_query_search(snp, nbits):
    """> 64 queries: the general kernel's swapped two-op epilogue + best pass at long K."""
    nq, nd = 80, 400
    q = dense_rows(nbits + 3, nq, nbits, [0.97, 0.99])
    db = dense_rows(nbits + 4, nd, nbits, [0.97, 0.98, 0.5])
    counts, best = snp.snp_fastid_search(snp.snp_pack(torch.from_numpy(q).to(DEV)),
                                         snp.snp_pack(torch.from_numpy(db).to(DEV)), nbits, ("xor", "andnot"))
    for j, op in enumerate(("xor", "andnot")):
        ref = oracle.counts(q, db, op)
        assert np.array_equal(u32(counts[j]), ref), op
        rb, ri = oracle.best(ref)
        assert np.array_equal(u32(best[j][0]), rb) and np.array_equal(best[j][1].cpu().numpy(), ri), op


@pytest.mark.parametrize("n", [46341, 70000])
def test_ld_wide_n_epilogue(snp, n):
    """n > 46340 samples: n² overflows int32, so the epilogue takes its int64 path.
    Mixed densities, duplicated / complemented rows (r² = 1, D′ = ±1) and monomorphic rows."""
    m = 136
    g = dense_rows(n, m, n, [0.5, 0.05, 0.97, 0.3])
    g[1] = 0
    g[2] = 1
    g[5] = g[4]
    g[7] = 1 - g[6]
    A = snp.snp_pack(torch.from_numpy(g).to(DEV))
    r2_ref, dp_ref, n_ref = oracle.ld(g, g)
    for self_ld in (True, False):
        B = A if self_ld else A.clone()
        r2, dp, cnt = snp.snp_ld_r2(A, B, n, dprime=True, counts=True)
        assert np.array_equal(u32(cnt), n_ref), self_ld
        check_rel(r2.cpu().numpy(), r2_ref)
        check_rel(dp.cpu().numpy(), dp_ref)
        r2only, _, _ = snp.snp_ld_r2(A, B, n)
        check_rel(r2only.cpu().numpy(), r2_ref)


def _subprocess(code, env_extra, timeout=900):
    env = dict(os.environ, **env_extra)
    r = subprocess.run([sys.executable, "-c", code], cwd=ROOT, env=env, capture_output=True, text=True,
                       timeout=timeout)
    assert r.returncode == 0 and "ok" in r.stdout, r.stdout[-3000:] + r.stderr[-3000:]
    return r.stdout


_I8_CODE = r'''
import numpy as np, torch, sys
sys.path.insert(0, ".")
import oracle, snpgen
import paper_conf_ipps_binderlp19_b200 as snp
torch.cuda.set_device(0)
snp.snp_set_variant("tc")          # the tensor variant (AUTO streams <= 3 queries on CUDA cores)
rng = np.random.default_rng(7)
def rows(r, k, p):
    return (rng.random((r, k), dtype=np.float32) < p).astype(np.uint8)
for (m, n, nbits) in [(1, 1, 1), (70, 513, 1000), (257, 300, 2049), (130, 130, 4096), (8, 300, 16385)]:
    ga = rows(m, nbits, 0.9); gb = rows(n, nbits, 0.7)
    A = snp.snp_pack(torch.from_numpy(ga).cuda()); B = snp.snp_pack(torch.from_numpy(gb).cuda())
    for op in ("and", "xor", "andnot", "notand"):
        out = snp.snp_fastid(A, B, nbits, op)
        assert snp.snp_last_kernel() == "tc_i8", snp.snp_last_kernel()
        assert np.array_equal(out.cpu().numpy().view(np.uint32), oracle.counts(ga, gb, op)), (m, n, nbits, op)
    r2, dp, cnt = snp.snp_ld_r2(A, B, nbits, dprime=True, counts=True)
    r2_ref, dp_ref, n_ref = oracle.ld(ga, gb)
    assert np.array_equal(cnt.cpu().numpy().view(np.uint32), n_ref)
    for got, ref in ((r2, r2_ref), (dp, dp_ref)):
        g = got.cpu().numpy().astype(np.float64); z = ref == 0
        assert (g[z] == 0).all() and (np.abs(g[~z] - ref[~z]) <= 1e-6 * np.abs(ref[~z])).all()
print("ok")
'''


def test_i8_kernel_subprocess():
    """The tcgen05 kind::i8 kernel (SNP_TC_KIND=i8 is read once per process): every op
    and the LD epilogue on ragged shapes vs the oracle."""
    _subprocess(_I8_CODE, {"SNP_TC_KIND": "i8"})


def test_i8_route_at_2p24_bits(snp):
    """nbits ≥ 2^24 is routed past the mxf4 kernels by default; whatever serves it must be
    exact: two 2^24 + 64-bit operands of density ~0.97 (counts ~1.6e7, odd) vs the oracle."""
    nbits = (1 << 24) + 64
    ga = dense_rows(21, 6, nbits, [0.97, 0.99, 0.5])
    gb = dense_rows(22, 20, nbits, [0.97, 0.6])
    A = snp.snp_pack(torch.from_numpy(ga).to(DEV))
    B = snp.snp_pack(torch.from_numpy(gb).to(DEV))
    for op in ("and", "xor"):
        out = snp.snp_fastid(A, B, nbits, op)
        assert np.array_equal(u32(out), oracle.counts(ga, gb, op)), (op, snp.snp_last_kernel())
