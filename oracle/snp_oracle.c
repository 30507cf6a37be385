/*
 * snp_oracle.c — plain, slow, obviously-correct CPU oracle for SNP comparison.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference leg may load or call this file.  The product
 * (paper_conf_ipps_binderlp19_b200/, include/, csrc/) never includes, links or
 * calls it, and this file includes nothing from the product: the two share no
 * code, headers, tables or constants.
 *
 * Everything works on UNPACKED genotype bytes g[r][k] (non-zero = minor allele,
 * P:L107 "Major alleles are encoded as 0s while minor alleles ... as 1s"),
 * bit by bit, in the order the paper states the definitions.  There is no
 * blocking, no word-level popcount and no reordering.  OpenMP only splits the
 * outermost loop over output rows (independent results).
 *
 * Citation convention: P:Lnn = /root/reference/PAPER.md line nn (section named).
 *
 * Readings of the paper (also listed in DESIGN.md §3):
 *  R1  bit k of packed row r = (w[r][k>>6] >> (k&63)) & 1, little-endian uint64
 *      words, LSB first, zero padding past nbits (Fig. 2 P:L80-93;
 *      the paper does not fix bit order — SURVEY §8c.7).
 *  R2  op AND    : c += x & y                (Eq. 1, §II.A; x^2 = x for bits)
 *      op XOR    : c += x ^ y                (Eq. 2, §II.B)
 *      op ANDNOT : c += (x ^ y) & x          (Eq. 3 literally, §II.C) with
 *                  r = query row x, m = database row y  ("m ... stored in the
 *                  database") == popc(q & ~d)
 *      op NOTAND : c += (y ^ x) & y          (Eq. 3 with r = database row y,
 *                  m = query row x) == popc(d & ~q)
 *  R3  LD: n = nbits (real samples, not padding); nA, nB, nAB exact integers;
 *      D_AB = pAB - pA pB (§II.A) scaled by n^2: num = n*nAB - nA*nB;
 *      r2 = num^2 / (nA (n-nA) nB (n-nB))  (Hill-Robertson r^2; the paper names
 *      only D, citing [10]/[11]);
 *      D' = num / Dmax,  Dmax = min(nA(n-nB), (n-nA)nB) if num > 0,
 *                               min(nA nB, (n-nA)(n-nB)) if num < 0  (Lewontin);
 *      monomorphic SNP (den == 0) => r2 = 0; num == 0 => D' = 0.
 *  R4  best match: per query the minimum count and the LOWEST database index
 *      attaining it ("No set bits ... signifies a positive match";
 *      tie-break not in the paper).
 */
#include <stdint.h>
#include <stddef.h>
#include <math.h>

#define ORACLE_AND 0
#define ORACLE_XOR 1
#define ORACLE_ANDNOT 2
#define ORACLE_NOTAND 3

/* R1: the oracle's own reader of a packed row. */
void oracle_unpack(const uint64_t *packed, int64_t rows, int64_t nbits, int64_t ldw,
                   uint8_t *g, int64_t ldg)
{
    for (int64_t r = 0; r < rows; ++r)
        for (int64_t k = 0; k < nbits; ++k) {
            uint64_t word = packed[r * ldw + (k / 64)];
            g[r * ldg + k] = (uint8_t)((word >> (k % 64)) & 1u);
        }
}

/* R1: the oracle's own writer (encoding + zero padding, Fig. 2). */
void oracle_pack(const uint8_t *g, int64_t rows, int64_t nbits, int64_t ldg,
                 uint64_t *packed, int64_t ldw)
{
    for (int64_t r = 0; r < rows; ++r) {
        for (int64_t w = 0; w < ldw; ++w) packed[r * ldw + w] = 0;   /* padding = 0 */
        for (int64_t k = 0; k < nbits; ++k)
            if (g[r * ldg + k] != 0)
                packed[r * ldw + (k / 64)] |= ((uint64_t)1) << (k % 64);
    }
}

/* p_A, p_B of P:L44 as integer counts: number of minor alleles in each row. */
void oracle_row_popc(const uint8_t *g, int64_t rows, int64_t nbits, int64_t ldg,
                     uint32_t *popc)
{
    for (int64_t r = 0; r < rows; ++r) {
        uint32_t c = 0;
        for (int64_t k = 0; k < nbits; ++k) c += (g[r * ldg + k] != 0) ? 1u : 0u;
        popc[r] = c;
    }
}

/* R2: C[i][j] = sum_k op(x_ik, y_jk), Eqs. (1)-(3) and the
 * GEMM-update form gamma_ij += sum_k POPC(alpha_ik & beta_kj). */
int oracle_counts(const uint8_t *ga, int64_t m, int64_t lda,
                  const uint8_t *gb, int64_t n, int64_t ldb,
                  int64_t nbits, int op, uint32_t *c, int64_t ldc)
{
    if (op < 0 || op > 3) return -1;
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t i = 0; i < m; ++i) {
        for (int64_t j = 0; j < n; ++j) {
            uint32_t acc = 0;
            for (int64_t k = 0; k < nbits; ++k) {
                unsigned x = ga[i * lda + k] != 0;
                unsigned y = gb[j * ldb + k] != 0;
                unsigned t;
                switch (op) {
                case ORACLE_AND:    t = x & y; break;            /* Eq. (1) */
                case ORACLE_XOR:    t = x ^ y; break;            /* Eq. (2) */
                case ORACLE_ANDNOT: t = (x ^ y) & x; break;      /* Eq. (3), r = x */
                default:            t = (y ^ x) & y; break;      /* Eq. (3), r = y */
                }
                acc += t;
            }
            c[i * ldc + j] = acc;
        }
    }
    return 0;
}

/* R3: LD statistics from exact integer counts (§II.A). */
static void ld_pair(int64_t n, int64_t na, int64_t nb, int64_t nab,
                    double *r2, double *dp)
{
    int64_t num = n * nab - na * nb;                         /* n^2 * D_AB, exact */
    __int128 den = (__int128)(na * (n - na)) * (__int128)(nb * (n - nb));
    if (den == 0) *r2 = 0.0;
    else *r2 = ((double)num * (double)num) / (double)den;
    int64_t dmax;
    if (num > 0) {
        int64_t a = na * (n - nb), b = (n - na) * nb;
        dmax = a < b ? a : b;
    } else if (num < 0) {
        int64_t a = na * nb, b = (n - na) * (n - nb);
        dmax = a < b ? a : b;
    } else {
        dmax = 0;
    }
    *dp = dmax ? (double)num / (double)dmax : 0.0;
}

int oracle_ld(const uint8_t *ga, int64_t m, int64_t lda,
              const uint8_t *gb, int64_t n, int64_t ldb, int64_t nbits,
              double *r2, double *dprime, uint32_t *nab_out, int64_t ldc)
{
    if (nbits < 1) return -1;
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t i = 0; i < m; ++i) {
        int64_t na = 0;
        for (int64_t k = 0; k < nbits; ++k) na += ga[i * lda + k] != 0;
        for (int64_t j = 0; j < n; ++j) {
            int64_t nb = 0, nab = 0;
            for (int64_t k = 0; k < nbits; ++k) {
                unsigned x = ga[i * lda + k] != 0;
                unsigned y = gb[j * ldb + k] != 0;
                nb += y;
                nab += x & y;                                    /* Eq. (1) */
            }
            double rr, dd;
            ld_pair(nbits, na, nb, nab, &rr, &dd);
            if (r2) r2[i * ldc + j] = rr;
            if (dprime) dprime[i * ldc + j] = dd;
            if (nab_out) nab_out[i * ldc + j] = (uint32_t)nab;
        }
    }
    return 0;
}

/* Same statistic from given integer counts (used to pin ld_pair itself). */
void oracle_ld_from_counts(int64_t n, int64_t na, int64_t nb, int64_t nab,
                           double *r2, double *dprime)
{
    ld_pair(n, na, nb, nab, r2, dprime);
}

/* R4: per-query minimum and lowest index attaining it, plus index_base. */
void oracle_best(const uint32_t *c, int64_t nq, int64_t nd, int64_t ldc,
                 int64_t index_base, uint32_t *best, int64_t *idx)
{
    for (int64_t i = 0; i < nq; ++i) {
        uint32_t b = 0xFFFFFFFFu;
        int64_t bi = -1;
        for (int64_t j = 0; j < nd; ++j)
            if (bi < 0 || c[i * ldc + j] < b) { b = c[i * ldc + j]; bi = j; }
        best[i] = b;
        idx[i] = bi < 0 ? -1 : bi + index_base;
    }
}
