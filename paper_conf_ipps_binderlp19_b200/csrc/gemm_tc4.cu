// gemm_tc4.cu — general tensor-core bit-GEMM (LD all pairs, FastID with many queries):
//
//   C[i][j] = sum_k A_ik & B_jk        (Eq. 1; GEMM form P:L116)
//   + fused epilogue: counts / FastID op identities / LD r2, D' (a5)
//
// Bits become e2m1 nibbles (1 -> 1.0) and are multiplied with tcgen05.mma kind::mxf4
// (scale factors 2^0, exact fp32 sums below 2^24).
// 128 x 128 output tiles, persistent CTAs (one per SM), K in 512-bit stages.
//
// Per stage, for the 128 lane rows (A) and 128 column rows (B) of the tile:
//   TMA warp      one 2-D TMA load per operand (128 rows x 64 B, 64B-swizzled) into
//                 the packed ring slot of the stage;
//   expander group g (stages it = g mod 3; 4 warps, one per TMEM lane quarter):
//                 LDS the packed rows, accumulate row popcounts, expand each 32-bit word
//                 to four words of nibbles (shifts on the FMA pipe via IMAD.HI), write A
//                 into TMEM (tcgen05.st; MMA operand A from TMEM) and B into the stage's
//                 K-major no-swizzle shared-memory operand;
//   MMA warp      8 x tcgen05.mma (M = N = 128, K = 64) from one elected lane, commit;
//   8 epilogue warps  drain the other TMEM accumulator (double-buffered), apply the
//                 identity / LD statistic, store.
// Resource plan: TMEM 2 x 128 accumulator + 3 x 64 A-stage + 32 scale-factor columns;
// shared memory 3 x 16 KB packed + 3 x 32 KB expanded B + barriers/popcounts.
#include "snp_internal.h"
#include "tc_ptx.cuh"
#include "e2m1.cuh"

#include <cuda.h>
#include <cstdio>
#include <cstdlib>

// LD output stores: evict-first streaming stores (st.global.cs) by default — an LD output is
// written once and must not push the packed operands out of L2 (with write-back stores LD-32K
// re-read 2.2 instead of 1.6 GB from DRAM and ran ~2 % slower under the power cap);
// -DGEMM_STORE_WB makes them write-back.  The swapped FastID count stores are write-back
// (SWAP_STG_FN: FastID-20M 125.1 -> 121.1 ms).
#ifdef GEMM_STORE_WB
#define STG_OUT "st.global"
#define STG_OUT_FN(p, v) (void)(*(p) = (v))
#else
#define STG_OUT "st.global.cs"
#define STG_OUT_FN(p, v) __stcs((p), (v))
#endif
#define SWAP_STG_FN(p, v) (void)(*(p) = (v))

namespace snp {

// Pipeline trace of CTA 0 (profiling aid, SNP_TRACE=1): per iteration it < 2048,
// [0] expander before waits, [1] after waits, [2] after packed LDS, [3] half 0 published,
// [4] half 1 published, [5] MMA got half 0, [6] MMA got half 1, [7] MMA commit issued.
__device__ long long g_gemm_trace[8 * 2048];
// Per-CTA timeline (build with -DSNP_PROFILING -DGEMM_TRACE3, read with snp_debug_gemm_cta):
// globaltimer ns at [0] entry, [1] setup done, [2] griddepcontrol.wait returned, [3] first
// packed stage arrived (expander 0), [4] first accumulator ready (epilogue warp 0), [5] last
// tile stored (epilogue warp 0), [6] exit barrier passed.
__device__ long long g_gemm_cta[8 * 1024];
__device__ long long g_gemm_cta2[8 * 1024];   // epilogue warp 0, first tile: [2 hh] after TMEM load, [2 hh + 1] after block
#ifdef GEMM_TRACE3
#define GEMM_T3(k, cond) do { if ((cond) && blockIdx.x < 1024) g_gemm_cta[8 * blockIdx.x + (k)] = (long long)ptx::globaltimer_ns(); } while (0)
#define GEMM_T3B(k, cond) do { if ((cond) && blockIdx.x < 1024) g_gemm_cta2[8 * blockIdx.x + (k)] = (long long)ptx::globaltimer_ns(); } while (0)
#else
#define GEMM_T3(k, cond) do { } while (0)
#define GEMM_T3B(k, cond) do { } while (0)
#endif

namespace {

constexpr int BM = 128, BN = 128;
constexpr int KBITS = 512;
constexpr int KW = KBITS / 32;                 // 16 packed words per row per stage
#ifndef GEMM_NS
#define GEMM_NS 3
#endif
constexpr int NS = GEMM_NS;                    // expanded slots (TMEM A stage + smem B stage)
#ifndef GEMM_NP
#define GEMM_NP 6
#endif
constexpr int NP = GEMM_NP;                    // packed TMA ring: NP x 16 KB in flight per SM
#ifndef GEMM_HALF
#define GEMM_HALF 0
#endif
constexpr int GH = GEMM_HALF ? 2 : 1;          // full barriers per stage (half-stage publishing)
                                               // (3 slots left the expanders waiting on L2)
#ifndef GEMM_G
#define GEMM_G 2
#endif
constexpr int G = GEMM_G;                      // expander groups (group g takes stages it = g mod G)
constexpr int NEXP = 8 * G;                    // per group: 4 A-warps (TMEM) + 4 B-warps (smem)
constexpr int NEPI = 8;
constexpr int EPI_WARP0 = NEXP;                // 16..23
constexpr int TMA_WARP = NEXP + NEPI;          // 24
constexpr int MMA_WARP = NEXP + NEPI + 1;      // 25 (highest id: scheduler priority)
constexpr int NTHREADS = (NEXP + NEPI + 2) * 32;
constexpr int PROW = KBITS / 8;                // 64 packed bytes per row per stage
constexpr int PSLOT = (BM + BN) * PROW;        // 16 KB packed per slot (A then B)
constexpr int BSLOT = BN * KBITS / 2;          // 32 KB expanded B per slot
constexpr int ACC_COLS = BN;
constexpr int A_COL0 = 2 * ACC_COLS;           // 256
constexpr int SF_COL = A_COL0 + NS * 64;       // 448
static_assert(SF_COL + 32 <= 512, "TMEM budget");
constexpr int TRW = 32 * 32 * 4;                // per epilogue warp: 32 x 32 count transpose
constexpr size_t SMEM = (size_t)NP * PSLOT + (size_t)NS * BSLOT + (size_t)NEPI * TRW + 1024;
static_assert(SMEM <= 232448, "227 KB opt-in shared memory");

struct GArgs {
    int64_t nl, nc, nbits;
    int swap, op, accumulate;
    int64_t ldo;
    uint32_t *C;
    float *r2, *dprime;
    int64_t nlb, ncb;
    int nst;
    int trace;
    int debug_skip;   // profiling experiment (build with -DGEMM_DEBUG_SKIP): expanders only pass
                      // tokens, results invalid
    int order;        // tile raster: 2 grouped (default), 1 lane-block-major, 0 column-block-major
    int off32;        // every output element offset (row * ldo + col) fits in 32 bits
    int sym;          // f3 symmetric self-LD: only tiles lb <= cb, off-diagonal ones mirrored
    int v4;           // outputs 16-byte aligned with ldo % 4 == 0: vector copy-out
    int op2;          // EPI_COUNTS, swapped layout: second op written to C2 (or C2 = NULL)
    uint32_t *C2;
    const uint32_t *popL, *popC;   // row popcounts (row_popc pre-pass), NULL if unused
    // f3 packed triangle (snp_ld_sym): tiles tlo .. tlo + ntri - 1 of the row-major upper
    // triangle of the T x T tile grid (T = nlb), tile u of the launch stored as a dense
    // 128 x 128 row-major block at element offset u * 128 * 128 of C / r2 / dprime (ldo = 128)
    int tri;
    int64_t tlo, ntri, mreal;
};


// LD statistics in fp32 from exact integers (reading R3).  num, nA(n-nA), nB(n-nB) are
// exact integers; each is rounded once to fp32, so r2 and D' carry a relative error of
// a few 2^-24 (< 1e-6), and are exactly 0 where the exact value is 0.
__device__ __forceinline__ void ld_stats_f32(int64_t n, int64_t na, int64_t nb, int64_t nab, float &r2,
                                             float &dp) {
    const int64_t num = n * nab - na * nb;
    const int64_t da = na * (n - na), db = nb * (n - nb);
    if (num == 0 || da == 0 || db == 0) {
        r2 = 0.f;
        dp = 0.f;
        return;
    }
    const float fn = (float)num;
    r2 = __fdiv_rn(fn, (float)da) * __fdiv_rn(fn, (float)db);
    int64_t dmax;
    if (num > 0) {
        const int64_t x = na * (n - nb), y = (n - na) * nb;
        dmax = x < y ? x : y;
    } else {
        const int64_t x = na * nb, y = (n - na) * (n - nb);
        dmax = x < y ? x : y;
    }
    dp = __fdiv_rn(fn, (float)dmax);
}


// 1/d in fp32: d rounded to fp32, then a correctly rounded reciprocal (2 roundings; FP64
// division is avoided: the DFMA pipe throttled the epilogue); 0 for d = 0 (monomorphic
// SNP: r2 = 0).
__device__ __forceinline__ float inv_exact(int64_t d) { return d ? __frcp_rn((float)d) : 0.f; }

// Exact count from the fp32 accumulator (an integer < 2^24): the 2^23 magic add below
// 2^23 (FMA pipe, no F2I), F2I above.
__device__ __forceinline__ uint32_t acc_count(uint32_t v, bool small) {
    return small ? __float_as_uint(__fadd_rn(__uint_as_float(v), 8388608.0f)) - 0x4B000000u
                 : __float2uint_rn(__uint_as_float(v));
}

// Epilogue of a 32-row x 32-column block when the output's row index is the TMEM lane
// (no operand swap): c[j] holds (row = this lane, column j) as fp32 accumulator bits.  The block is transposed
// through the warp's 4 KB of shared memory (16-byte chunks XOR-swizzled by row: 4
// wavefronts per STS.128, conflict-free LDS.32) so that afterwards lane = output column
// and every store of a row is one coalesced 128-byte line.  Row quantities (nA, 1/da)
// are broadcast from their lane by shuffles.
//   counts: x = op identity of SURVEY §8a a4 with (pQ, pD) = (row, column) popcounts
//   LD:     reading R3 from exact integers: num = n nAB - nA nB (int32 for n <= 46340),
//           r2 = min(1, (num / da) (num / db)) with 1/da, 1/db from 2 roundings each: 9
//           fp32 roundings in total, relative error <= 9 * 2^-24 = 5.4e-7;
//           exactly 0 where num = 0.  D' = num / Dmax (correctly rounded division).

// predicated evict-first stores (no branch around them: shuffles stay converged)
__device__ __forceinline__ void st_cs_pred_f32(float *p, float v, uint32_t ok) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p " STG_OUT ".f32 [%0], %1;\n\t}" ::"l"(p), "f"(v),
                 "r"(ok)
                 : "memory");
}
__device__ __forceinline__ void st_cs_pred_u32(uint32_t *p, uint32_t v, uint32_t ok) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p " STG_OUT ".u32 [%0], %1;\n\t}" ::"l"(p), "r"(v),
                 "r"(ok)
                 : "memory");
}
// f3 symmetric self-LD: the mirror image of an off-diagonal block.  Block (rows row0 + lane,
// columns col0 + u) is also block (rows col0 + u, columns row0 + lane) of the output, and
// every output is symmetric (AND / XOR counts, r2, D'), so before the transpose (lane = row
// i, c[u] = column col0 + u) each u is one coalesced 128-byte store of row col0 + u.
template <int EPI>
__device__ __forceinline__ void epi_mirror(const GArgs &args, const uint32_t (&c)[32], int lane, int64_t row0,
                                           int64_t col0, uint32_t pl, uint32_t pcol, float ia, bool small_n,
                                           bool want_dp) {
    const int64_t gi = row0 + lane;                 // becomes the output column
    const bool ok_i = gi < args.nl;
    const int64_t ldo = args.ldo;
    const int64_t n = args.nbits;
    const int32_t n32 = (int32_t)n;
    const int ncol = (int)(args.nc - col0 < 32 ? args.nc - col0 : 32);   // output rows here
    const float ibl = EPI == EPI_LD ? inv_exact((int64_t)pcol * (n - (int64_t)pcol)) : 0.f;
    const int64_t o0 = col0 * ldo + gi;
    if (EPI == EPI_COUNTS && !args.accumulate && args.off32) {
        uint32_t off = (uint32_t)o0;
        const uint32_t ld32 = (uint32_t)ldo;
        const bool xo = args.op == 1;   // XOR (else AND): the symmetric ops
#pragma unroll
        for (int u = 0; u < 32; ++u) {
            const uint32_t pb = __shfl_sync(0xffffffffu, pcol, u);
            const uint32_t x = xo ? pl + pb - 2u * c[u] : c[u];
            st_cs_pred_u32(args.C + off, x, (ok_i && u < ncol) ? 1u : 0u);
            off += ld32;
        }
        return;
    }
    if (EPI == EPI_LD && small_n && !want_dp && args.off32) {
        // the benchmarked path: 32-bit element offsets, predicated evict-first stores
        float *const r2b = args.r2;
        uint32_t *const cb = args.C;
        const bool has_c = cb != nullptr;
        uint32_t off = (uint32_t)o0;
        const uint32_t ld32 = (uint32_t)ldo;
        const int32_t npl = -(int32_t)pl;
#pragma unroll
        for (int u = 0; u < 32; ++u) {
            const int32_t pb = (int32_t)__shfl_sync(0xffffffffu, pcol, u);
            const float ib = __shfl_sync(0xffffffffu, ibl, u);
            const int32_t num = n32 * (int32_t)c[u] + npl * pb;
            const float fn = (float)num;
            const float r2v = fminf(__fmul_rn(__fmul_rn(fn, ia), __fmul_rn(fn, ib)), 1.0f);
            const uint32_t okr = (ok_i && u < ncol) ? 1u : 0u, okc = (okr && has_c) ? 1u : 0u;
            asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p " STG_OUT ".f32 [%0], %1;\n\t}" ::"l"(
                             r2b + off),
                         "f"(r2v), "r"(okr)
                         : "memory");
            asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p " STG_OUT ".u32 [%0], %1;\n\t}" ::"l"(
                             cb + off),
                         "r"(c[u]), "r"(okc)
                         : "memory");
            off += ld32;
        }
        return;
    }
#pragma unroll
    for (int u = 0; u < 32; ++u) {   // fully unrolled: c[u] stays in registers
        const uint32_t pb = __shfl_sync(0xffffffffu, pcol, u);   // popcount of SNP col0 + u
        const float ib = EPI == EPI_LD ? __shfl_sync(0xffffffffu, ibl, u) : 0.f;
        if (!ok_i || u >= ncol) continue;
        const int64_t o = o0 + (int64_t)u * ldo;
        const uint32_t cu = c[u];
        if (EPI == EPI_COUNTS) {
            const uint32_t x = args.op == 0 ? cu : pl + pb - 2u * cu;   // AND or XOR (symmetric)
            if (args.accumulate) args.C[o] += x;
            else STG_OUT_FN(args.C + o, x);
        } else {
            float r2v, dpv = 0.f;
            if (small_n) {
                const int32_t num = n32 * (int32_t)cu - (int32_t)pl * (int32_t)pb;
                const float fn = (float)num;
                r2v = fminf(__fmul_rn(__fmul_rn(fn, ia), __fmul_rn(fn, ib)), 1.0f);
                if (want_dp && num != 0) {
                    const int32_t pa_ = (int32_t)pl, pb_ = (int32_t)pb;
                    const int32_t dmax = num > 0 ? min(pa_ * (n32 - pb_), (n32 - pa_) * pb_)
                                                 : min(pa_ * pb_, (n32 - pa_) * (n32 - pb_));
                    dpv = __fdiv_rn(fn, (float)dmax);
                }
            } else {
                ld_stats_f32(n, (int64_t)pl, (int64_t)pb, (int64_t)cu, r2v, dpv);
            }
            STG_OUT_FN(args.r2 + o, r2v);
            if (want_dp) STG_OUT_FN(args.dprime + o, dpv);
            if (args.C) STG_OUT_FN(args.C + o, cu);
        }
    }
}


// f3 fast path for an off-diagonal full 32 x 32 block of the benchmarked LD output (r2 +
// counts, n <= 46340, no D'): r2 is computed ONCE in the pre-transpose layout (lane = row
// i), stored mirrored straight away, and staged through the warp's transpose buffer for
// the normal-orientation stores; the counts follow through the same buffer.
__device__ __forceinline__ void epi_ld_sym_fast(const GArgs &args, const uint32_t (&c)[32], uint32_t *tw, int lane,
                                                int64_t row0, int64_t col0, uint32_t pl, uint32_t pcol, float ia) {
    const int64_t ldo = args.ldo;
    const int32_t n32 = (int32_t)args.nbits;
    const uint32_t ld32 = (uint32_t)ldo;
    float *const r2b = args.r2;
    uint32_t *const cb = args.C;
    const uint32_t has_c = cb != nullptr ? 1u : 0u;
    const bool ok_i = row0 + lane < args.nl;                         // mirror column / normal row
    const int ncol = (int)(args.nc - col0 < 32 ? args.nc - col0 : 32);
    const uint32_t okn = (col0 + lane < args.nc) ? 1u : 0u;           // normal column
    const uint32_t *twl = tw + (lane & 3);
    const uint32_t xl = (uint32_t)(lane >> 2);
    // 1. stage the counts (row i = lane, 16-byte chunks XOR-swizzled by row)
    __syncwarp();   // the previous block's reads of tw are done
#pragma unroll
    for (int k = 0; k < 8; ++k) {
        const uint32_t a = ptx::smem_u32(tw + lane * 32 + ((k ^ (lane & 7)) << 2));
        asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(c[4 * k]), "r"(c[4 * k + 1]),
                     "r"(c[4 * k + 2]), "r"(c[4 * k + 3])
                     : "memory");
    }
    __syncwarp();
    // 2. counts in the normal orientation (lane = column)
    if (has_c) {
        uint32_t off = (uint32_t)(row0 * ldo + col0 + lane);
#pragma unroll
        for (int r = 0; r < 32; ++r) {
            st_cs_pred_u32(cb + off, twl[r * 32 + ((xl ^ (uint32_t)(r & 7)) << 2)], okn);
            off += ld32;
        }
    }
    __syncwarp();
    // 3. r2 once per element from this lane's own row chunks: mirrored stores (row col0 + u,
    //    column row0 + lane; counts too), and r2 written back over the chunk just read
    const float ibl = inv_exact((int64_t)pcol * ((int64_t)n32 - (int64_t)pcol));
    const int32_t npl = -(int32_t)pl;
    uint32_t offm = (uint32_t)(col0 * ldo + row0 + lane);
#pragma unroll
    for (int k = 0; k < 8; ++k) {
        const uint32_t a = ptx::smem_u32(tw + lane * 32 + ((k ^ (lane & 7)) << 2));
        uint32_t cc[4];
        asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(cc[0]), "=r"(cc[1]), "=r"(cc[2]), "=r"(cc[3])
                     : "r"(a) : "memory");
        float r[4];
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            const int u = 4 * k + t;
            const int32_t pb = (int32_t)__shfl_sync(0xffffffffu, pcol, u);
            const float ib = __shfl_sync(0xffffffffu, ibl, u);
            const int32_t num = n32 * (int32_t)cc[t] + npl * pb;
            const float fn = (float)num;
            r[t] = fminf(__fmul_rn(__fmul_rn(fn, ia), __fmul_rn(fn, ib)), 1.0f);
            const uint32_t ok = (ok_i && u < ncol) ? 1u : 0u;
            st_cs_pred_f32(r2b + offm, r[t], ok);
            st_cs_pred_u32(cb + offm, cc[t], ok & has_c);
            offm += ld32;
        }
        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a), "f"(r[0]), "f"(r[1]), "f"(r[2]), "f"(r[3])
                     : "memory");
    }
    __syncwarp();
    // 4. r2 in the normal orientation
    uint32_t off = (uint32_t)(row0 * ldo + col0 + lane);
#pragma unroll
    for (int r = 0; r < 32; ++r) {
        st_cs_pred_f32(r2b + off, __uint_as_float(twl[r * 32 + ((xl ^ (uint32_t)(r & 7)) << 2)]), okn);
        off += ld32;
    }
}


// Full 32 x 32 LD block with a 16-byte-aligned output (32 valid columns, ldo % 4 == 0):
// r2 is computed in the pre-transpose layout (lane = row i, u = column: the column terms are
// shuffled), optionally stored mirrored (f3), and both r2 and the counts leave through the
// transpose buffer with 16-byte copies: per warp instruction 4 rows x 128 bytes (one
// LDS.128 + one STG.128 per 4 elements instead of one LDS + one STG per element).
__device__ __forceinline__ void copy_out_v4(const uint32_t *tw, int lane, uint32_t *dst, uint32_t off0, uint32_t ld32) {
    const int cchunk = lane & 7, rsub = lane >> 3;
#pragma unroll
    for (int it = 0; it < 8; ++it) {
        const int r = 4 * it + rsub;
        uint4 x = *reinterpret_cast<const uint4 *>(tw + r * 32 + ((cchunk ^ (r & 7)) << 2));
        uint4 *d = reinterpret_cast<uint4 *>(dst + off0 + (uint32_t)r * ld32 + 4u * (uint32_t)cchunk);
        STG_OUT_FN(d, x);
    }
}
__device__ __forceinline__ void epi_ld_fast_v4(const GArgs &args, const uint32_t (&c)[32], uint32_t *tw, int lane,
                                               int64_t row0, int64_t col0, uint32_t pl, uint32_t pcol, float ia,
                                               bool mirror) {
    const int64_t ldo = args.ldo;
    const int32_t n32 = (int32_t)args.nbits;
    const uint32_t ld32 = (uint32_t)ldo;
    float *const r2b = args.r2;
    uint32_t *const cb = args.C;
    const uint32_t has_c = cb != nullptr ? 1u : 0u;
    const uint32_t off_n = (uint32_t)(row0 * ldo + col0);           // normal block origin
    __syncwarp();   // the previous block's reads of tw are done
    if (has_c) {    // counts: stage (row i = lane, chunks XOR-swizzled by row), copy out
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            const uint32_t a = ptx::smem_u32(tw + lane * 32 + ((k ^ (lane & 7)) << 2));
            asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(c[4 * k]), "r"(c[4 * k + 1]),
                         "r"(c[4 * k + 2]), "r"(c[4 * k + 3])
                         : "memory");
        }
        __syncwarp();
        copy_out_v4(tw, lane, cb, off_n, ld32);
        __syncwarp();
    }
    const bool ok_i = row0 + lane < args.nl;
    const float ibl = inv_exact((int64_t)pcol * ((int64_t)n32 - (int64_t)pcol));
    const int32_t npl = -(int32_t)pl;
    uint32_t offm = (uint32_t)(col0 * ldo + row0 + lane);           // mirror: row col0 + u
#pragma unroll
    for (int k = 0; k < 8; ++k) {
        float r[4];
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            const int u = 4 * k + t;
            const int32_t pb = (int32_t)__shfl_sync(0xffffffffu, pcol, u);
            const float ib = __shfl_sync(0xffffffffu, ibl, u);
            const int32_t num = n32 * (int32_t)c[u] + npl * pb;
            const float fn = (float)num;
            r[t] = fminf(__fmul_rn(__fmul_rn(fn, ia), __fmul_rn(fn, ib)), 1.0f);
            if (mirror) {
                const uint32_t ok = ok_i ? 1u : 0u;
                st_cs_pred_f32(r2b + offm, r[t], ok);
                st_cs_pred_u32(cb + offm, c[u], ok & has_c);
                offm += ld32;
            }
        }
        const uint32_t a = ptx::smem_u32(tw + lane * 32 + ((k ^ (lane & 7)) << 2));
        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a), "f"(r[0]), "f"(r[1]), "f"(r[2]), "f"(r[3])
                     : "memory");
    }
    __syncwarp();
    copy_out_v4(tw, lane, reinterpret_cast<uint32_t *>(r2b), off_n, ld32);
}

template <int EPI>
__device__ __forceinline__ void epi_transposed(const GArgs &args, uint32_t (&c)[32], uint32_t *tw, int lane,
                                               int64_t row0, int64_t col0, uint32_t pl, uint32_t pcol, float ia,
                                               bool small_n, bool want_dp, bool mirror) {
    const bool small = args.nbits < (1LL << 23);
#pragma unroll
    for (int i = 0; i < 32; ++i) c[i] = acc_count(c[i], small);   // in place: c is the TMEM load
    if (EPI == EPI_LD && small_n && !want_dp && args.off32 && args.v4 && args.nl - row0 >= 32 &&
        args.nc - col0 >= 32) {
        epi_ld_fast_v4(args, c, tw, lane, row0, col0, pl, pcol, ia, mirror);
        return;
    }
    if (EPI == EPI_LD && mirror && small_n && !want_dp && args.off32 && args.nl - row0 >= 32) {
        epi_ld_sym_fast(args, c, tw, lane, row0, col0, pl, pcol, ia);
        return;
    }
    if (mirror) epi_mirror<EPI>(args, c, lane, row0, col0, pl, pcol, ia, small_n, want_dp);
    __syncwarp();   // the previous block's reads of tw are done
#pragma unroll
    for (int k = 0; k < 8; ++k) {
        const uint32_t a = ptx::smem_u32(tw + lane * 32 + ((k ^ (lane & 7)) << 2));
        asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(c[4 * k]), "r"(c[4 * k + 1]),
                     "r"(c[4 * k + 2]), "r"(c[4 * k + 3])
                     : "memory");
    }
    __syncwarp();
    const int64_t gc = col0 + lane;
    const bool colok = gc < args.nc;
    const int64_t ldo = args.ldo;
    const int64_t n = args.nbits;
    const int32_t n32 = (int32_t)n;
    const int32_t pb = (int32_t)pcol;
    const int rows = (int)(args.nl - row0 < 32 ? args.nl - row0 : 32);   // warp-uniform
    const int64_t o0 = row0 * ldo + gc;
    if (EPI == EPI_COUNTS && rows == 32 && !args.accumulate && args.off32) {
        // full block, fully unrolled: x = cq pQ + cd pD + cc c, predicated
        // evict-first stores at 32-bit element offsets
        const int op = args.op;
        const uint32_t cq = (op == 1 || op == 2) ? 1u : 0u, cdp = (op == 1 || op == 3) ? pcol : 0u;
        const uint32_t cc = op == 0 ? 1u : op == 1 ? (uint32_t)-2 : (uint32_t)-1;
        const uint32_t *twl = tw + (lane & 3);
        const uint32_t xl = (uint32_t)(lane >> 2);
        const uint32_t okn = colok ? 1u : 0u;
        uint32_t off = (uint32_t)o0;
        const uint32_t ld32 = (uint32_t)ldo;
#pragma unroll
        for (int r = 0; r < 32; ++r) {
            const uint32_t plr = __shfl_sync(0xffffffffu, pl, r);
            const uint32_t c = twl[r * 32 + ((xl ^ (uint32_t)(r & 7)) << 2)];
            st_cs_pred_u32(args.C + off, cc * c + (cq * plr + cdp), okn);
            off += ld32;
        }
        return;
    }
    if (EPI == EPI_COUNTS) {
        uint32_t *cp = args.C + o0;
        const int op = args.op;
        const bool acc = args.accumulate != 0;
#pragma unroll 4
        for (int r = 0; r < 32; ++r) {
            const uint32_t plr = __shfl_sync(0xffffffffu, pl, r);
            if (r >= rows) break;
            const uint32_t c = tw[r * 32 + ((((lane >> 2) ^ (r & 7))) << 2) + (lane & 3)];
            const uint32_t x = op == 0 ? c : op == 1 ? plr + pcol - 2u * c : op == 2 ? plr - c : pcol - c;
            if (colok) {
                if (acc) *cp += x;
                else STG_OUT_FN(cp, x);
            }
            cp += ldo;
        }
        return;
    }
    float *rp = args.r2 + o0;
    if (small_n && !want_dp && rows == 32 && args.off32) {
        // the benchmarked LD path, full 32-row block: fully unrolled, 32-bit element
        // offsets (off32: every output offset < 2^32), the 8 swizzled LDS column offsets
        // precomputed; per element 2 SHFL (row terms), LDS, 2 IMAD, I2F, 3 FMUL, FMNMX,
        // 1 address IMAD per output array and 1-2 STG
        const float ib = inv_exact((int64_t)pb * (n - (int64_t)pb));
        const int32_t npb = -pb;
        const bool has_c = args.C != nullptr;
        uint32_t cofs[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) cofs[k] = (uint32_t)(((((lane >> 2) ^ k)) << 2) + (lane & 3));
        uint32_t off = (uint32_t)o0;
        const uint32_t ld32 = (uint32_t)ldo;
        float *const r2b = args.r2;
        uint32_t *const cb = args.C;
        const uint32_t okr = colok ? 1u : 0u, okc = (colok && has_c) ? 1u : 0u;
#pragma unroll
        for (int r = 0; r < 32; ++r) {
            const int32_t plr = (int32_t)__shfl_sync(0xffffffffu, pl, r);
            const float iar = __shfl_sync(0xffffffffu, ia, r);
            const int32_t c = (int32_t)tw[r * 32 + cofs[r & 7]];
            const int32_t num = n32 * c + plr * npb;
            const float fn = (float)num;
            const float r2v = fminf(__fmul_rn(__fmul_rn(fn, iar), __fmul_rn(fn, ib)), 1.0f);
            // predicated evict-first stores (outputs are written once; the packed operands
            // stay in L2): no branch, so the shuffles stay in a converged straight line
            asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p " STG_OUT ".f32 [%0], %1;\n\t}" ::"l"(
                             r2b + off),
                         "f"(r2v), "r"(okr)
                         : "memory");
            asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p " STG_OUT ".u32 [%0], %1;\n\t}" ::"l"(
                             cb + off),
                         "r"(c), "r"(okc)
                         : "memory");
            off += ld32;
        }
        return;
    }
    if (small_n && !want_dp) {
        // the benchmarked LD path: per element 2 IMAD, I2F, 3 FMUL, FMNMX, 1-2 STG
        const float ib = inv_exact((int64_t)pb * (n - (int64_t)pb));
        const int32_t npb = -pb;
        uint32_t *cp = args.C ? args.C + o0 : nullptr;
#pragma unroll 4
        for (int r = 0; r < 32; ++r) {
            const int32_t plr = (int32_t)__shfl_sync(0xffffffffu, pl, r);
            const float iar = __shfl_sync(0xffffffffu, ia, r);
            if (r >= rows) break;
            const int32_t c = (int32_t)tw[r * 32 + ((((lane >> 2) ^ (r & 7))) << 2) + (lane & 3)];
            const int32_t num = n32 * c + plr * npb;
            const float fn = (float)num;
            const float r2v = fminf(__fmul_rn(__fmul_rn(fn, iar), __fmul_rn(fn, ib)), 1.0f);
            if (colok) {
                STG_OUT_FN(rp, r2v);   // outputs are written once: evict-first keeps the packed
                if (cp) STG_OUT_FN(cp, (uint32_t)c);   // operands resident in L2
            }
            rp += ldo;
            if (cp) cp += ldo;
        }
        return;
    }
    const float ib = inv_exact((int64_t)pb * (n - (int64_t)pb));
#pragma unroll 1
    for (int r = 0; r < rows; ++r) {
        const uint32_t plr = __shfl_sync(0xffffffffu, pl, r);
        const float iar = __shfl_sync(0xffffffffu, ia, r);
        const uint32_t cr = tw[r * 32 + ((((lane >> 2) ^ (r & 7))) << 2) + (lane & 3)];
        if (!colok) continue;
        const int64_t o = o0 + (int64_t)r * ldo;
        float r2v, dpv = 0.f;
        if (small_n) {
            const int32_t num = n32 * (int32_t)cr - (int32_t)plr * pb;
            const float fn = (float)num;
            r2v = fminf(__fmul_rn(__fmul_rn(fn, iar), __fmul_rn(fn, ib)), 1.0f);
            if (num != 0) {
                const int32_t pa_ = (int32_t)plr;
                const int32_t dmax = num > 0 ? min(pa_ * (n32 - pb), (n32 - pa_) * pb)
                                             : min(pa_ * pb, (n32 - pa_) * (n32 - pb));
                dpv = __fdiv_rn(fn, (float)dmax);
            }
        } else {
            ld_stats_f32(n, (int64_t)plr, (int64_t)pb, (int64_t)cr, r2v, dpv);
        }
        STG_OUT_FN(args.r2 + o, r2v);
        if (want_dp) STG_OUT_FN(args.dprime + o, dpv);
        if (args.C) STG_OUT_FN(args.C + o, cr);
    }
}


// Counts epilogue of the swapped layout (lane = output column j = database row, the 32
// accumulator columns u = output rows i = queries): for each u the 32 lanes store 32
// consecutive words.  Each op is x = cq pQ + cd pD + cc c, two IMADs;
// running output pointers; up to two ops (C, C2) from the same count.
__device__ __forceinline__ void op_coef(int op, uint32_t &cq, uint32_t &cd, uint32_t &cc) {
    cq = (op == 1 || op == 2) ? 1u : 0u;
    cd = (op == 1 || op == 3) ? 1u : 0u;
    cc = op == 0 ? 1u : op == 1 ? (uint32_t)-2 : (uint32_t)-1;
}
__device__ __forceinline__ void epi_swapped_counts(const GArgs &args, uint32_t (&v)[32], int lane, int64_t gl,
                                                   int64_t col0, int ncols, uint32_t pl, uint32_t pcol) {
    const bool small = args.nbits < (1LL << 23);
    const bool rowok = gl < args.nl;
    const int64_t ldo = args.ldo;
    const bool two = args.C2 != nullptr;
    const bool acc = args.accumulate != 0;
    uint32_t cq1, cd1, cc1, cq2, cd2, cc2;
    op_coef(args.op, cq1, cd1, cc1);
    op_coef(two ? args.op2 : 0, cq2, cd2, cc2);
    const uint32_t b1 = cd1 * pl, b2 = cd2 * pl;   // database-row terms (this lane)
    uint32_t *o1 = args.C + col0 * ldo + gl;
    uint32_t *o2 = two ? args.C2 + col0 * ldo + gl : nullptr;
#ifdef GEMM_DEBUG_NOSTORE
    uint32_t sink = 0;
#endif
#pragma unroll
    for (int u = 0; u < 32; ++u) {
        const uint32_t pq = __shfl_sync(0xffffffffu, pcol, u);   // query popcount of column u
        const uint32_t c = acc_count(v[u], small);
        const bool ok = rowok && u < ncols;
        const uint32_t x1 = cc1 * c + (cq1 * pq + b1);
#ifdef GEMM_DEBUG_NOSTORE   // profiling experiment: the epilogue without its stores (results invalid)
        sink ^= x1;
        if (two) sink ^= cc2 * c + (cq2 * pq + b2);
        continue;
#endif
        if (ok) {
            if (acc) *o1 += x1;
            else SWAP_STG_FN(o1, x1);
        }
        o1 += ldo;
        if (two) {
            const uint32_t x2 = cc2 * c + (cq2 * pq + b2);
            if (ok) SWAP_STG_FN(o2, x2);
            o2 += ldo;
        }
    }
#ifdef GEMM_DEBUG_NOSTORE
    if (sink == 0x9e3779b9u) *o1 = sink;
#endif
}

template <int EPI, bool TRI = false, bool BPRE = false>
__global__ void __launch_bounds__(NTHREADS, 1)
gemm_tc4_kernel(const __grid_constant__ CUtensorMap tmL, const __grid_constant__ CUtensorMap tmC,
                const GArgs args) {
    extern __shared__ __align__(1024) uint8_t smem[];
    uint8_t *ring = smem;                                        // [NP][PSLOT]
    uint8_t *bexp = smem + (size_t)NP * PSLOT;                   // [NS][BSLOT]
    uint32_t *trs = reinterpret_cast<uint32_t *>(bexp + (size_t)NS * BSLOT);   // [NEPI][32][32]
    uint64_t *bars = reinterpret_cast<uint64_t *>(trs + NEPI * 32 * 32);
    uint64_t *pfull = bars;            // [NP] TMA -> expanders
    uint64_t *pempty = pfull + NP;     // [NP] expanders -> TMA
    uint64_t *full = pempty + NP;      // [NS][GH] expanders -> MMA
    uint64_t *empty = full + NS * GH;  // [NS] MMA -> expanders
    uint64_t *accf = empty + NS;       // [2]
    uint64_t *acce = accf + 2;         // [2]
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(acce + 2);

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    GEMM_T3(0, tid == 0);
    const int64_t nbits = args.nbits;
    const int nst = args.nst;
    const int64_t ntiles = TRI ? args.ntri : args.sym ? args.nlb * (args.nlb + 1) / 2 : args.nlb * args.ncb;
    // 32-bit tile arithmetic (ntiles < 2^31): a 64-bit division is a subroutine CALL, and
    // any call in the kernel made ptxas drop the MMA issue loop out of uniform registers
    const uint32_t nlb32 = (uint32_t)args.nlb, ncb32 = (uint32_t)args.ncb;
    // tile t -> (lane block, column block).  order 2 (default): groups of RG lane blocks;
    // inside a group the lane block varies fastest, so the ~148 tiles in flight cover RG
    // lane blocks x ~148/RG column blocks: each packed column block is read from DRAM once
    // per group and reused RG times from L2, the group's lane blocks stay L2-resident for
    // its whole column sweep (DRAM reads ~ nlb/RG x the column operand instead of ~nlb x).
    // order 1: lane-block-major; order 0: column-block-major.
    constexpr uint32_t RG = 16;
    // f3: the upper triangle (lb <= cb) of the T x T tile grid in groups of RG lane blocks;
    // inside a group column block major, lane block fastest (a triangle, then a rectangle)
    auto decode_sym = [&](uint32_t t, uint32_t &lb, uint32_t &cb) {
        const uint32_t T = nlb32;
        uint32_t g0 = 0;
        for (;;) {
            const uint32_t R = T - g0 < RG ? T - g0 : RG;
            const uint32_t nt = R * (R + 1) / 2 + R * (T - g0 - R);
            if (t < nt || R < RG) break;
            t -= nt;
            g0 += R;
        }
        const uint32_t R = T - g0 < RG ? T - g0 : RG;
        const uint32_t tri = R * (R + 1) / 2;
        if (t < tri) {
            uint32_t k = 0;
            while ((k + 1) * (k + 2) / 2 <= t) ++k;
            cb = g0 + k;
            lb = g0 + (t - k * (k + 1) / 2);
        } else {
            t -= tri;
            cb = g0 + R + t / R;
            lb = g0 + t % R;
        }
    };
    auto tile_lb = [&](uint32_t t) -> uint32_t {
        if (args.sym) { uint32_t lb, cb; decode_sym(t, lb, cb); return lb; }
        if (args.order == 2) {
            const uint32_t g = t / (RG * ncb32), w = t - g * RG * ncb32;
            const uint32_t rows = nlb32 - g * RG < RG ? nlb32 - g * RG : RG;
            return g * RG + w % rows;
        }
        return args.order ? t / ncb32 : t % nlb32;
    };
    auto tile_cb = [&](uint32_t t) -> uint32_t {
        if (args.sym) { uint32_t lb, cb; decode_sym(t, lb, cb); return cb; }
        if (args.order == 2) {
            const uint32_t g = t / (RG * ncb32), w = t - g * RG * ncb32;
            const uint32_t rows = nlb32 - g * RG < RG ? nlb32 - g * RG : RG;
            return w / rows;
        }
        return args.order ? t % ncb32 : t / nlb32;
    };
    const int64_t my_tiles =
        ntiles > blockIdx.x ? (int64_t)(((uint32_t)ntiles - 1u - blockIdx.x) / gridDim.x + 1u) : 0;
    const int64_t total_it = my_tiles * nst;
    const int64_t full32 = nbits / 32;

    if (tid == 0) {
        for (int i = 0; i < NP; ++i) {
            ptx::mbar_init(&pfull[i], 1);
            ptx::mbar_init(&pempty[i], BPRE ? 4 : 8);   // BPRE: only the A warps read the ring
        }
        for (int i = 0; i < NS; ++i) {
            // BPRE: the 4 A warps + the TMA producer's expect_tx for the pre-expanded B tile
            for (int h = 0; h < GH; ++h) ptx::mbar_init(&full[i * GH + h], BPRE ? 5 : 8);
            ptx::mbar_init(&empty[i], 1);
        }
        for (int i = 0; i < 2; ++i) {
            ptx::mbar_init(&accf[i], 1);
            ptx::mbar_init(&acce[i], NEPI);
        }
        ptx::fence_mbar_init();
    }
    if (warp == TMA_WARP && lane == 0) {
        ptx::prefetch_tensormap(&tmL);
        ptx::prefetch_tensormap(&tmC);
    }
    if (warp == MMA_WARP) ptx::tmem_alloc<512>(tmem_slot);
    ptx::tc_fence_before();
    __syncthreads();
    ptx::tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    if (warp >= EPI_WARP0 && warp < EPI_WARP0 + 4) {
        const int q = warp & 3;
        uint32_t v[32];
#pragma unroll
        for (int i = 0; i < 32; ++i) v[i] = 0x7F7F7F7Fu;   // ue8m0 2^0 in every scale byte
        ptx::tmem_st32(tmem + ((uint32_t)(q * 32) << 16) + SF_COL, v);
        ptx::tmem_st_wait();
    }
    ptx::tc_fence_before();
    __syncthreads();
    ptx::tc_fence_after();
    GEMM_T3(1, tid == 0);
    // programmatic dependent launch: the setup above overlapped the previous kernel (the
    // row-popcount pre-pass); its results are visible after this wait, and nothing global
    // was read or written before it
    asm volatile("griddepcontrol.wait;" ::: "memory");
    GEMM_T3(2, tid == 0);

    if (warp == TMA_WARP) {
        // ------------------------------------------------------------ TMA producer
        if (lane == 0) {
            int p = 0;
            uint32_t round = 0;
            int bs = 0;           // BPRE: B slot of the stage and how often it was used
            uint32_t buse = 0;
            for (int64_t tl = 0; tl < my_tiles; ++tl) {
                const int64_t t = blockIdx.x + tl * gridDim.x;
                const uint32_t t32 = (uint32_t)t;
                uint32_t lbt, cbt;
                if (BPRE) decode_sym(t32, lbt, cbt);   // grouped triangle raster (B blocks reused from L2)
                else if (TRI) tri_decode(args.nlb, args.tlo + t, lbt, cbt);
                else if (args.sym) decode_sym(t32, lbt, cbt);
                else { lbt = tile_lb(t32); cbt = tile_cb(t32); }
                const int32_t rl = (int32_t)(lbt * BM), rc = (int32_t)(cbt * BN);
                for (int s = 0; s < nst; ++s) {
                    if (round > 0) ptx::mbar_wait(&pempty[p], (round - 1) & 1);   // lane 0 only
#ifdef GEMM_DEBUG_SKIP
                    const bool no_b = BPRE || SNP_PROF(args.debug_skip == 3);
#else
                    constexpr bool no_b = BPRE;
#endif
                    ptx::mbar_arrive_expect_tx(&pfull[p], no_b ? BM * PROW : PSLOT);
                    ptx::tma_load_2d(ring + p * PSLOT, &tmL, &pfull[p], s * KW, rl);
                    if (!no_b) ptx::tma_load_2d(ring + p * PSLOT + BM * PROW, &tmC, &pfull[p], s * KW, rc);
                    if (++p == NP) { p = 0; ++round; }
                    if (BPRE) {
                        // the stage's B operand arrives pre-expanded (128-byte rows, 128B swizzle)
                        // straight into its MMA slot once the MMA has released that slot
                        if (buse > 0) ptx::mbar_wait(&empty[bs], (buse - 1) & 1);
                        ptx::mbar_arrive_expect_tx(&full[bs * GH], BSLOT);
                        uint8_t *dst = bexp + (size_t)bs * BSLOT;
                        ptx::tma_load_2d(dst, &tmC, &full[bs * GH], s * (KW * 4), rc);
                        ptx::tma_load_2d(dst + BSLOT / 2, &tmC, &full[bs * GH], s * (KW * 4) + KW * 2, rc);
                        if (++bs == NS) { bs = 0; ++buse; }
                    }
                }
            }
        }
    } else if (warp < NEXP) {
        // ------------------------------------------------------------ expanders
        // group g = warp / 8 takes stages it = g, g + G, ...; within a group warps 0-3 expand
        // the A rows of lane quarter q into TMEM, warps 4-7 the B rows into shared memory,
        // so the TMEM and shared-memory chains of a stage run in parallel.
        const int g = warp >> 3, r8 = warp & 7;
        const bool is_a = r8 < 4;
        const int q = r8 & 3;
        const int row = q * 32 + lane;
        const int sw = (row >> 1) & 3;                  // TMA 64B swizzle of a 64-byte row
        const uint32_t tAq = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)A_COL0;
        const int64_t my_total_it = (BPRE && !is_a) ? 0 : total_it;   // BPRE: B arrives expanded
        int64_t tl = g / nst;
        int s = g % nst;
        int slot = g % NS;
        uint32_t use = (uint32_t)(g / NS);              // how often `slot` was used before
        static_assert(NP % G == 0, "each packed slot belongs to one expander group");
        int pk = g;                                     // packed slot (group g: g, g + G, ...)
        uint32_t pround = 0;
        for (int64_t it = g; it < my_total_it; it += G) {
#ifdef GEMM_TRACE
            const bool tr = SNP_PROF(args.trace) && blockIdx.x == 0 && r8 == 0 && lane == 0 && it < 2048;
#endif
#ifdef GEMM_TRACE
            if (tr) g_gemm_trace[8 * it + 0] = clock64();
#endif
            // empty BEFORE pfull: both groups share the slots, so a warp may reach use u+2 of
            // a slot while its pfull barrier is only at phase u+1; waiting for the MMA to
            // release use u+1 first rules out parity aliasing on pfull (same parity as u)
            if (use > 0) ptx::mbar_wait_warp(&empty[slot], (use - 1) & 1);
            ptx::mbar_wait_warp(&pfull[pk], pround & 1);
            GEMM_T3(3, it == 0 && warp == 0 && lane == 0);
#ifdef GEMM_TRACE
            if (tr) g_gemm_trace[8 * it + 1] = clock64();
#endif
#ifdef GEMM_DEBUG_SKIP
            // debug_skip 1: every expander skips; 2: only the A warps on the MMA warp's sub-partition
            if (SNP_PROF(args.debug_skip == 1 || (args.debug_skip == 2 && is_a && q == (MMA_WARP & 3)))) {
                __syncwarp();
                if (lane == 0) {
                    ptx::mbar_arrive(&pempty[pk]);
                    for (int h = 0; h < GH; ++h) ptx::mbar_arrive(&full[slot * GH + h]);
                }
                s += G;
                while (s >= nst) { s -= nst; ++tl; }
                slot += G;
                if (slot >= NS) { slot -= NS; ++use; }
                pk += G;
                if (pk >= NP) { pk -= NP; ++pround; }
                continue;
            }
#endif
            const uint8_t *src = ring + pk * PSLOT + (is_a ? 0 : BM * PROW) + row * PROW;
            uint32_t w[KW];
#ifdef GEMM_DEBUG_SKIP
            // debug_skip 3: the B operand's packed words are not loaded (nor read): the cost of
            // the B half of the packed ring in shared memory (results invalid)
            if (SNP_PROF(args.debug_skip == 3 && !is_a)) {
#pragma unroll
                for (int i = 0; i < KW; ++i) w[i] = (uint32_t)(lane * 0x9E3779B9u + i + s);
            } else
#endif
#pragma unroll
            for (int c = 0; c < 4; ++c) {
                const uint4 x = *reinterpret_cast<const uint4 *>(src + ((c ^ sw) << 4));
                w[4 * c] = x.x; w[4 * c + 1] = x.y; w[4 * c + 2] = x.z; w[4 * c + 3] = x.w;
            }
#ifdef GEMM_TRACE
            if (tr) g_gemm_trace[8 * it + 2] = clock64();
#endif
            const int64_t w0 = (int64_t)s * KW;
            if (w0 + KW > full32) {
#pragma unroll
                for (int i = 0; i < KW; ++i) w[i] &= word_mask(w0 + i, nbits);
            }
            if (is_a) {
                const uint32_t tA = tAq + 64 * slot;
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    uint32_t v[32];
#pragma unroll
                    for (int i = 0; i < 8; ++i)
                        expandA(w[8 * h + i], v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
                    ptx::tmem_st32(tA + 32 * h, v);
                    if (GH == 2 && h == 0) {   // publish the first 256 bits
                        ptx::tmem_st_wait();
                        ptx::tc_fence_before();
                        __syncwarp();
                        if (lane == 0) ptx::mbar_arrive(&full[slot * GH]);
                    }
                }
                ptx::tmem_st_wait();
                ptx::tc_fence_before();
            } else {
                uint8_t *dstB = bexp + (size_t)slot * BSLOT + row * 16;
#pragma unroll
                for (int i = 0; i < KW; ++i) {          // chunk i of the K-major operand = word i
                    uint4 o;
                    expandB(w[i], o.x, o.y, o.z, o.w);
                    *reinterpret_cast<uint4 *>(dstB + (size_t)i * BN * 16) = o;
                    if (GH == 2 && i == KW / 2 - 1) {   // publish the first 256 bits
                        ptx::fence_proxy_async_smem();
                        __syncwarp();
                        if (lane == 0) ptx::mbar_arrive(&full[slot * GH]);
                    }
                }
                ptx::fence_proxy_async_smem();
            }
            __syncwarp();
            if (lane == 0) {
                // release the packed slot only now: every lane has consumed its LDS results
                // (an arrive right after the loads could let the next TMA overwrite data
                // that is still in flight to registers)
                ptx::mbar_arrive(&pempty[pk]);
                ptx::mbar_arrive(&full[slot * GH + GH - 1]);
            }
#ifdef GEMM_TRACE
            if (tr) g_gemm_trace[8 * it + 3] = clock64();
#endif
            s += G;
            while (s >= nst) { s -= nst; ++tl; }
            slot += G;
            if (slot >= NS) { slot -= NS; ++use; }
            pk += G;
            if (pk >= NP) { pk -= NP; ++pround; }
        }
    } else if (warp == MMA_WARP) {
        // ------------------------------------------------------------ MMA issuer
        // Warp-uniform loop (votes for the waits, tmem via a warp reduction): the TMEM
        // addresses and descriptors stay in uniform registers and each MMA is one UTCOMMA.
        constexpr uint32_t IDESC = idesc_mxf4(BM, BN);
        const uint32_t tmu = __reduce_or_sync(0xffffffffu, tmem);
        const uint32_t sfa = tmu + SF_COL, sfb = tmu + SF_COL + 16;
        const uint64_t bdesc0 = BPRE ? ptx::smem_desc_kmajor_sw128(ptx::smem_u32(bexp))
                                     : ptx::smem_desc_kmajor_noswizzle(ptx::smem_u32(bexp), BN * 16, 128);
        constexpr uint32_t BSTEP = (2 * BN * 16) >> 4;
        int b = 0;
        uint32_t round = 0;
        for (int64_t tl = 0; tl < my_tiles; ++tl) {
            const int acc = (int)(tl & 1);
#ifdef GEMM_TRACE4
            const bool tr4 = SNP_PROF(args.trace) && blockIdx.x == 0 && lane == 0 && tl < 2048;
            long long fw = 0;
            if (tr4) g_gemm_trace[8 * tl + 0] = clock64();
#endif
            if (tl >= 2) ptx::mbar_wait_uniform(&acce[acc], (uint32_t)(((tl >> 1) - 1) & 1));
#ifdef GEMM_TRACE4
            if (tr4) g_gemm_trace[8 * tl + 1] = clock64();
#endif
            ptx::tc_fence_after();
            const uint32_t d = tmu + (uint32_t)(acc * ACC_COLS);
            for (int s = 0; s < nst; ++s) {
#ifdef GEMM_TRACE4
                const long long w0 = clock64();
#endif
                ptx::mbar_wait_uniform(&full[b * GH], round & 1);
#ifdef GEMM_TRACE4
                fw += clock64() - w0;
#endif
                ptx::tc_fence_after();
                const uint32_t a0 = tmu + (uint32_t)(A_COL0 + 64 * b);
                const uint64_t b0 = bdesc0 + (uint64_t)(((uint32_t)b * BSLOT) >> 4);
                if (GH == 1) {
                    // one elected lane issues the stage's MMAs back to back and commits them
                    // (one elect.sync per stage, not per MMA; the FastID kernel measured this
                    // on its critical path)
                    if (ptx::elect_one()) {
#pragma unroll
                        for (int k = 0; k < KBITS / 64; ++k) {
                            // BPRE: K-step k is bytes [32 (k % 4), +32) of the 128-byte rows of half
                            // k / 4 (16 KB each; the descriptor's start address moves inside the
                            // swizzle atom)
                            const uint64_t bk = BPRE ? b0 + (uint64_t)((((k >> 2) * (BSLOT / 2)) + (k & 3) * 32) >> 4)
                                                     : b0 + (uint64_t)(k * BSTEP);
                            ptx::mma_mxf4_ts_one(d, a0 + 8 * k, bk, IDESC, (s | k) != 0 ? 1u : 0u, sfa, sfb);
                        }
                        ptx::mma_commit_one(&empty[b]);
                        if (s == nst - 1) ptx::mma_commit_one(&accf[acc]);
                    }
                    __syncwarp();
                } else {
#pragma unroll
                    for (int k = 0; k < KBITS / 64; ++k) {
                        if (GH == 2 && k == KBITS / 128) {
                            ptx::mbar_wait_uniform(&full[b * GH + 1], round & 1);
                            ptx::tc_fence_after();
                        }
                        const uint64_t bk = BPRE ? b0 + (uint64_t)((((k >> 2) * (BSLOT / 2)) + (k & 3) * 32) >> 4)
                                                 : b0 + (uint64_t)(k * BSTEP);
                        ptx::mma_mxf4_ts(d, a0 + 8 * k, bk, IDESC, (s | k) != 0 ? 1u : 0u, sfa, sfb);
                    }
                    ptx::mma_commit_uniform(&empty[b]);
                }
                if (++b == NS) { b = 0; ++round; }
            }
            if (GH != 1) ptx::mma_commit_uniform(&accf[acc]);
#ifdef GEMM_TRACE4
            if (tr4) { g_gemm_trace[8 * tl + 2] = clock64(); g_gemm_trace[8 * tl + 5] = fw; }
#endif
        }
        __syncwarp();
    } else {
        // ------------------------------------------------------------ epilogue (8 warps)
        // warp e: TMEM lane quarter e % 4 (lane rows), accumulator columns [64 h, 64 h + 64)
        const int e = warp - EPI_WARP0;
        const int q = e & 3, h = e >> 2;
        const int li = q * 32 + lane;
        const int c0 = 64 * h;
        const int64_t ldo = args.ldo;
        const int64_t n = nbits;
        const bool small_n = n <= 46340;                 // n^2 < 2^31: exact int32 LD arithmetic
        const bool need_pop = EPI == EPI_LD || args.op != 0 || (args.C2 && args.op2 != 0);
        const bool want_dp = EPI == EPI_LD && args.dprime != nullptr;
        for (int64_t tl = 0; tl < my_tiles; ++tl) {
            const int acc = (int)(tl & 1);
            const uint32_t ph = (uint32_t)((tl >> 1) & 1);
            const int64_t t = blockIdx.x + tl * gridDim.x;
            const uint32_t t32 = (uint32_t)t;
            uint32_t lbt, cbt;
            if (BPRE) decode_sym(t32, lbt, cbt);
            else if (TRI) tri_decode(args.nlb, args.tlo + t, lbt, cbt);
            else if (args.sym) decode_sym(t32, lbt, cbt);
            else { lbt = tile_lb(t32); cbt = tile_cb(t32); }
            // BPRE processes the whole triangle in the grouped raster; the tile's packed-triangle
            // storage slot is its row-major triangle index
            const int64_t tst = BPRE ? tri_start(args.nlb, lbt) + (int64_t)(cbt - lbt) : t;
            const bool mirror = !TRI && args.sym && lbt != cbt;   // f3: also write the mirror block
            // packed triangle: the epilogue addresses the tile as rows t * 128 .. t * 128 + 127
            // of a [ntri * 128][128] matrix (args.nl / nc / ldo are those virtual sizes), so
            // its (row * ldo + col) addressing lands in the dense block t; the real size m
            // (args.mreal) bounds only the popcount loads here — entries past m are written
            // as the zeros they compute (no popcount, TMA zero fill)
            const int64_t nlr = TRI ? args.mreal : args.nl, ncr = TRI ? args.mreal : args.nc;
            const int64_t gl = (int64_t)lbt * BM + li;
            const int64_t gc0 = (int64_t)cbt * BN + c0;
            const int64_t erow0 = TRI ? tst * BM + q * 32 : gl - lane;   // epilogue block origin
            const int64_t ecol0 = TRI ? (int64_t)c0 : gc0;
            const bool rows_ok = gl < args.nl && gc0 < args.nc;
            const int ncols = gc0 < ncr ? (int)(ncr - gc0 < 64 ? ncr - gc0 : 64) : 0;
            // popcounts: lane j holds the column popcounts of columns c0 + j and c0 + 32 + j
            uint32_t pl = 0, pcol0 = 0, pcol1 = 0;
            if (need_pop) {
                if (gl < nlr) pl = __ldg(args.popL + gl);
                if (lane < ncols) pcol0 = __ldg(args.popC + gc0 + lane);
                if (32 + lane < ncols) pcol1 = __ldg(args.popC + gc0 + 32 + lane);
            }
            ptx::mbar_wait_warp(&accf[acc], ph);
            GEMM_T3(4, tl == 0 && e == 0 && lane == 0);
#ifdef GEMM_TRACE4
            if (SNP_PROF(args.trace) && blockIdx.x == 0 && e == 0 && lane == 0 && tl < 2048) g_gemm_trace[8 * tl + 3] = clock64();
            if (SNP_PROF(args.trace) && blockIdx.x == 0 && e == 7 && lane == 0 && tl < 2048) g_gemm_trace[8 * tl + 6] = clock64();
#endif
            ptx::tc_fence_after();
            const bool full_vec = ncols == 64 && !args.swap;
            const uint32_t ta = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(acc * ACC_COLS + c0);
            const int32_t n32 = (int32_t)n, pl32 = (int32_t)pl;
            const int32_t da32 = pl32 * (n32 - pl32);
            // 1 / (nA (n - nA)) of this lane's row, one rounding (0 for a monomorphic SNP)
            const float ia = (EPI == EPI_LD && !args.swap) ? inv_exact((int64_t)pl * (n - (int64_t)pl)) : 0.f;
            // two halves of 32 accumulator columns; the accumulator is released right after
            // the second TMEM load, before that half is processed
#pragma unroll 1
            for (int hh = 0; hh < 2; ++hh) {
                uint32_t v[32];
                __syncwarp();            // tcgen05.ld is warp-collective: re-converge first
                ptx::tmem_ld32(ta + 32 * hh, v);
                ptx::tmem_ld_wait();
                GEMM_T3B(2 * hh, tl == 0 && e == 0 && lane == 0);
                if (hh == 1) {
                    ptx::tc_fence_before();
                    __syncwarp();
                    if (lane == 0) ptx::mbar_arrive(&acce[acc]);   // accumulator drained
#ifdef GEMM_TRACE4
                    if (SNP_PROF(args.trace) && blockIdx.x == 0 && (e == 0 || e == 7) && lane == 0 && tl < 2048)
                        g_gemm_trace[8 * tl + (e == 0 ? 4 : 7)] = clock64();
#endif
                }
                const uint32_t pcol = hh ? pcol1 : pcol0;
                if (!args.swap) {
                    epi_transposed<EPI>(args, v, trs + e * 32 * 32, lane, erow0, ecol0 + 32 * hh, pl, pcol,
                                        ia, small_n, want_dp, mirror);
                    GEMM_T3B(2 * hh + 1, tl == 0 && e == 0 && lane == 0);
                    continue;
                }
                if (EPI == EPI_COUNTS) {
                    epi_swapped_counts(args, v, lane, gl, gc0 + 32 * hh, ncols - 32 * hh, pl, pcol);
                    continue;
                }
                if (!__any_sync(0xffffffffu, rows_ok)) continue;   // warp-uniform skip only:
                // the column popcounts are shuffled across the warp, so every lane runs the
                // loop and only rows_ok lanes store
#pragma unroll
                for (int uu = 0; uu < 32; uu += 4) {
                    const int u0 = 32 * hh + uu;
                    uint32_t c[4], pc[4];
#pragma unroll
                    for (int k = 0; k < 4; ++k) {
                        c[k] = __float2uint_rn(__uint_as_float(v[uu + k]));    // exact count
                        pc[k] = __shfl_sync(0xffffffffu, pcol, uu + k);
                    }
                    if (EPI == EPI_COUNTS) {
                        // swapped layout (lane = output column): per output column k the 32
                        // lanes store 32 consecutive words.  Up to two ops from the one AND
                        // count (f1: XOR + ANDNOT in one pass over the database).
                        if (!rows_ok) continue;
#pragma unroll
                        for (int jj = 0; jj < 2; ++jj) {
                            uint32_t *const Cb = jj ? args.C2 : args.C;
                            if (jj && !Cb) break;
                            const int op = jj ? args.op2 : args.op;
#pragma unroll
                            for (int k = 0; k < 4; ++k) {
                                if (u0 + k >= ncols) break;
                                const uint32_t pq = pc[k], pd = pl;
                                const uint32_t r = op == 0 ? c[k] : op == 1 ? pq + pd - 2u * c[k]
                                                 : op == 2 ? pq - c[k] : pd - c[k];
                                uint32_t *o = Cb + (gc0 + u0 + k) * ldo + gl;
                                if (args.accumulate) *o += r;
                                else STG_OUT_FN(o, r);
                            }
                        }
                    } else {
                        float r2v[4], dpv[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
                        for (int k = 0; k < 4; ++k) {
                            // reading R3 from exact integers; (A, B) = (lane, column) or swapped
                            if (small_n) {
                                const int32_t pb = (int32_t)pc[k];
                                const int32_t num = n32 * (int32_t)c[k] - pl32 * pb;
                                const int32_t db = pb * (n32 - pb);
                                if (num == 0 || da32 == 0 || db == 0) {
                                    r2v[k] = 0.f;
                                } else {
                                    const float fn = (float)num;
                                    r2v[k] = __fdiv_rn(fn * fn, (float)da32 * (float)db);
                                    if (want_dp) {
                                        const int32_t pa_ = args.swap ? pb : pl32, pb_ = args.swap ? pl32 : pb;
                                        int32_t dmax;
                                        if (num > 0) dmax = min(pa_ * (n32 - pb_), (n32 - pa_) * pb_);
                                        else dmax = min(pa_ * pb_, (n32 - pa_) * (n32 - pb_));
                                        dpv[k] = __fdiv_rn(fn, (float)dmax);
                                    }
                                }
                            } else {
                                const int64_t pa_ = args.swap ? pc[k] : pl, pb_ = args.swap ? pl : pc[k];
                                ld_stats_f32(n, pa_, pb_, (int64_t)c[k], r2v[k], dpv[k]);
                            }
                        }
                        if (!rows_ok) continue;
                        if (full_vec) {
                            const int64_t o = gl * ldo + gc0 + u0;
                            if ((o & 3) == 0) {
                                *reinterpret_cast<float4 *>(args.r2 + o) = make_float4(r2v[0], r2v[1], r2v[2], r2v[3]);
                                if (want_dp)
                                    *reinterpret_cast<float4 *>(args.dprime + o) = make_float4(dpv[0], dpv[1], dpv[2], dpv[3]);
                                if (args.C) *reinterpret_cast<uint4 *>(args.C + o) = make_uint4(c[0], c[1], c[2], c[3]);
                                continue;
                            }
                        }
#pragma unroll
                        for (int k = 0; k < 4; ++k) {
                            if (u0 + k >= ncols) break;
                            const int64_t o = args.swap ? (gc0 + u0 + k) * ldo + gl : gl * ldo + gc0 + u0 + k;
                            args.r2[o] = r2v[k];
                            if (want_dp) args.dprime[o] = dpv[k];
                            if (args.C) args.C[o] = c[k];
                        }
                    }
                }
            }
        }
    }

    GEMM_T3(5, warp == EPI_WARP0 && lane == 0);
    ptx::tc_fence_before();
    __syncthreads();
    GEMM_T3(6, tid == 0);
    if (warp == MMA_WARP) {
        ptx::tc_fence_after();
        ptx::tmem_dealloc<512>(tmem);
    }
}


// ============================================================================ CTA-pair kernel
// gemm_tc4x2_kernel: the same bit-GEMM with tcgen05.mma.cta_group::2 on a cluster of two
// CTAs (one TPC).  A pair tile is 256 lane rows x 128 columns: each CTA expands its own
// 128 lane rows into its TMEM (MMA operand A from TMEM) and only 64 of the 128 column
// rows into its shared memory (the pair's B operand is split N/2 per CTA); the leader
// CTA's single thread issues M = 256, N = 128, K = 64 MMAs that read both CTAs' halves.
// Per CTA and stage this halves the B-side nibble writes to shared memory (16 KB instead
// of 32 KB) and cuts packed loads and expansion ALU work by a quarter — the shared-memory
// pipe and the ALU were the binding resources of the 1-CTA kernel.
// Cross-CTA protocol:
//   full[s]   (leader)  12 arrivals: the 6 expander warps of the stage's group in BOTH CTAs,
//                       remote mbarrier.arrive after their TMEM / shared writes;
//   empty[s]  (both)    tcgen05.commit multicast from the leader's MMA thread;
//   accf[a]   (both)    tcgen05.commit multicast at the end of a pair tile;
//   acce[a]   (leader)  16 arrivals: 8 epilogue warps of each CTA after draining TMEM.
namespace x2 {
constexpr int BNP = 128;                       // pair tile columns
constexpr int BNH = BNP / 2;                   // column rows per CTA
constexpr int NS = 3;                          // TMEM A / smem B stages
#ifndef X2_NP
#define X2_NP 8
#endif
#ifndef X2_G
#define X2_G 2
#endif
constexpr int NP = X2_NP;                      // packed TMA ring
constexpr int G = X2_G;                        // expander groups
constexpr int GW = 6;                          // warps per group: 4 A (lane quarters) + 2 B
constexpr int NEXP = G * GW;                   // 12
constexpr int NEPI = 8;
constexpr int EPI_WARP0 = NEXP;                // 12..19
constexpr int TMA_WARP = NEXP + NEPI;          // 20
constexpr int MMA_WARP = NEXP + NEPI + 1;      // 21
constexpr int NTHREADS = (NEXP + NEPI + 2) * 32;
constexpr int PSLOT = (BM + BNH) * PROW;       // 12 KB packed per slot (128 A rows, 64 C rows)
constexpr int BSLOT = BNH * KBITS / 2;         // 16 KB expanded B per slot
constexpr int ACC_COLS = BNP;                  // 128
constexpr int A_COL0 = 2 * ACC_COLS;           // 256
constexpr int SF_COL = A_COL0 + NS * 64;       // 448
static_assert(SF_COL + 32 <= 512, "TMEM budget");
constexpr size_t SMEM = (size_t)NP * PSLOT + (size_t)NS * BSLOT + (size_t)NEPI * TRW + 1024;
static_assert(SMEM <= 232448, "227 KB opt-in shared memory");

__device__ __forceinline__ uint32_t cta_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t cluster_id() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%clusterid.x;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t num_clusters() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%nclusterid.x;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// arrive on the barrier at the same shared-memory offset in CTA `rank` of the cluster
__device__ __forceinline__ void arrive_remote(uint64_t *bar, uint32_t rank) {
    uint32_t ra;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(ptx::smem_u32(bar)), "r"(rank));
    // default semantics (release, CTA scope), as for any producer signalling the pair's MMA: the
    // data it publishes is this CTA's own shared memory / TMEM, already ordered for the tensor
    // core by fence.proxy.async / tcgen05.fence::before_thread_sync.  A cluster-scope release
    // here cost ~1,500 cycles per arrival (measured: scripts/trace_x2.py)
    asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" ::"r"(ra) : "memory");
}
__device__ __forceinline__ bool try_wait_cluster(uint64_t *bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(ptx::smem_u32(bar)), "r"(parity), "r"(100000u)
        : "memory");
    return ok != 0;
}
// warp-uniform wait with cluster-scope acquire (the arrivals come from both CTAs)
__device__ __forceinline__ bool try_wait_cluster_now(uint64_t *bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(ptx::smem_u32(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}
__device__ __forceinline__ void wait_cluster_uniform(uint64_t *bar, uint32_t parity) {
    if (__all_sync(0xffffffffu, try_wait_cluster_now(bar, parity))) return;
    const uint64_t t0 = ptx::globaltimer_ns();
    while (!__all_sync(0xffffffffu, try_wait_cluster(bar, parity))) {
        if (__any_sync(0xffffffffu, ptx::globaltimer_ns() - t0 > 4000000000ull)) __trap();
    }
}
__device__ __forceinline__ void mma_mxf4_ts2(uint32_t d, uint32_t a, uint64_t b, uint32_t idesc, uint32_t accumulate,
                                             uint32_t sfa, uint32_t sfb) {
    asm volatile(
        "{\n\t.reg .pred e, p;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "@e tcgen05.mma.cta_group::2.kind::mxf4.block_scale.block32 [%0], [%1], %2, %3, [%5], [%6], p;\n\t}" ::"r"(d),
        "r"(a), "l"(b), "r"(idesc), "r"(accumulate), "r"(sfa), "r"(sfb)
        : "memory");
}
__device__ __forceinline__ void mma_mxf4_ts2_one(uint32_t d, uint32_t a, uint64_t b, uint32_t idesc, uint32_t accumulate,
                                                 uint32_t sfa, uint32_t sfb) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::2.kind::mxf4.block_scale.block32 [%0], [%1], %2, %3, [%5], [%6], p;\n\t}" ::"r"(d),
        "r"(a), "l"(b), "r"(idesc), "r"(accumulate), "r"(sfa), "r"(sfb)
        : "memory");
}
__device__ __forceinline__ void commit_both_one(uint64_t *bar) {   // by the issuing thread alone
    asm volatile(
        "{\n\t.reg .b16 m;\n\tmov.b16 m, 3;\n\t"
        "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], m;\n\t}" ::"r"(
            ptx::smem_u32(bar))
        : "memory");
}
// commit the leader's outstanding MMAs to the barrier at this offset in BOTH CTAs
__device__ __forceinline__ void commit_both(uint64_t *bar) {
    asm volatile(
        "{\n\t.reg .pred e;\n\t.reg .b16 m;\n\tmov.b16 m, 3;\n\telect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], m;\n\t}" ::"r"(
            ptx::smem_u32(bar))
        : "memory");
}
}  // namespace x2

// f3 on CTA pairs: pair tile u <-> (P, J), lane blocks 2P and 2P + 1 (one per CTA) x column
// block J, J = 2P .. T - 1 in row-major order, start(P) = P (T + 1 - P).  The pair's lower
// tile (2P + 1, 2P) and lane block T (odd T) are computed on zeros / below the diagonal and
// not stored.
__host__ __device__ __forceinline__ int64_t pair_start(int64_t T, int64_t P) { return P * (T + 1 - P); }
__host__ __device__ __forceinline__ void pair_decode(int64_t T, int64_t u, uint32_t &P, uint32_t &J) {
    const double b = (double)T + 1.0;
    int64_t p = (int64_t)((b - sqrt(b * b - 4.0 * (double)u)) * 0.5);
    const int64_t np = (T + 1) / 2;
    if (p < 0) p = 0;
    if (p > np - 1) p = np - 1;
    while (p > 0 && pair_start(T, p) > u) --p;
    while (p + 1 < np && pair_start(T, p + 1) <= u) ++p;
    P = (uint32_t)p;
    J = (uint32_t)(2 * p + (u - pair_start(T, p)));
}

template <int EPI, bool TRI = false>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(x2::NTHREADS, 1)
gemm_tc4x2_kernel(const __grid_constant__ CUtensorMap tmL, const __grid_constant__ CUtensorMap tmC,
                  const GArgs args) {
    constexpr int NS = x2::NS, NP = x2::NP, G = x2::G, GW = x2::GW, NEXP = x2::NEXP, NEPI = x2::NEPI;
    constexpr int EPI_WARP0 = x2::EPI_WARP0, TMA_WARP = x2::TMA_WARP, MMA_WARP = x2::MMA_WARP;
    constexpr int PSLOT = x2::PSLOT, BSLOT = x2::BSLOT, ACC_COLS = x2::ACC_COLS, A_COL0 = x2::A_COL0;
    constexpr int SF_COL = x2::SF_COL, BNP = x2::BNP, BNH = x2::BNH;
    using x2::cta_rank; using x2::cluster_id; using x2::num_clusters; using x2::cluster_sync;
    using x2::arrive_remote; using x2::wait_cluster_uniform; using x2::mma_mxf4_ts2; using x2::commit_both;
    using x2::mma_mxf4_ts2_one; using x2::commit_both_one;
    extern __shared__ __align__(1024) uint8_t smem[];
    uint8_t *ring = smem;                                        // [NP][PSLOT]
    uint8_t *bexp = smem + (size_t)NP * PSLOT;                   // [NS][BSLOT]
    uint32_t *trs = reinterpret_cast<uint32_t *>(bexp + (size_t)NS * BSLOT);   // [NEPI][32][32]
    uint64_t *bars = reinterpret_cast<uint64_t *>(trs + NEPI * 32 * 32);
    uint64_t *pfull = bars;            // [NP] TMA -> expanders (local)
    uint64_t *pempty = pfull + NP;     // [NP] expanders -> TMA (local)
    uint64_t *full = pempty + NP;      // [NS] expanders of both CTAs -> leader MMA
    uint64_t *empty = full + NS;       // [NS] MMA -> expanders (multicast commit)
    uint64_t *accf = empty + NS;       // [2]  MMA -> epilogues (multicast commit)
    uint64_t *acce = accf + 2;         // [2]  epilogues of both CTAs -> leader MMA
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(acce + 2);

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const uint32_t rank = cta_rank();
    const bool leader = rank == 0;
    const int64_t nbits = args.nbits;
    const int nst = args.nst;
    // pair tiles: nlb = lane blocks of 256 rows, ncb = column blocks of 128
    const uint32_t nlb32 = (uint32_t)args.nlb, ncb32 = (uint32_t)args.ncb;
    // TRI: nlb = T (128-row blocks of the m x m triangle), ntri = pair tiles
    const uint32_t ntiles = TRI ? (uint32_t)args.ntri : nlb32 * ncb32;
    const uint32_t cid = cluster_id(), ncl = num_clusters();
    const int64_t my_tiles = ntiles > cid ? (int64_t)((ntiles - 1u - cid) / ncl + 1u) : 0;
    const int64_t total_it = my_tiles * nst;
    const int64_t full32 = nbits / 32;
    constexpr uint32_t RG = 8;   // grouped raster (see gemm_tc4_kernel), lane block fastest
    auto tile_lb = [&](uint32_t t) -> uint32_t {
        const uint32_t g = t / (RG * ncb32), w = t - g * RG * ncb32;
        const uint32_t rows = nlb32 - g * RG < RG ? nlb32 - g * RG : RG;
        return g * RG + w % rows;
    };
    auto tile_cb = [&](uint32_t t) -> uint32_t {
        const uint32_t g = t / (RG * ncb32), w = t - g * RG * ncb32;
        const uint32_t rows = nlb32 - g * RG < RG ? nlb32 - g * RG : RG;
        return w / rows;
    };

    if (tid == 0) {
        for (int i = 0; i < NP; ++i) {
            ptx::mbar_init(&pfull[i], 1);
            ptx::mbar_init(&pempty[i], GW);
        }
        for (int i = 0; i < NS; ++i) {
            ptx::mbar_init(&full[i], 2 * GW);
            ptx::mbar_init(&empty[i], 1);
        }
        for (int i = 0; i < 2; ++i) {
            ptx::mbar_init(&accf[i], 1);
            ptx::mbar_init(&acce[i], 2 * NEPI);
        }
        ptx::fence_mbar_init();
    }
    if (warp == TMA_WARP && lane == 0) {
        ptx::prefetch_tensormap(&tmL);
        ptx::prefetch_tensormap(&tmC);
    }
    if (warp == MMA_WARP) {   // both CTAs, same warp id: one 2-SM allocation
        asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(ptx::smem_u32(tmem_slot))
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
    }
    ptx::tc_fence_before();
    __syncthreads();
    ptx::tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    if (warp >= EPI_WARP0 && warp < EPI_WARP0 + 4) {
        const int q = warp & 3;
        uint32_t v[32];
#pragma unroll
        for (int i = 0; i < 32; ++i) v[i] = 0x7F7F7F7Fu;   // ue8m0 2^0 in every scale byte
        ptx::tmem_st32(tmem + ((uint32_t)(q * 32) << 16) + SF_COL, v);
        ptx::tmem_st_wait();
    }
    ptx::tc_fence_before();
    cluster_sync();   // barriers initialised and TMEM allocated in both CTAs
    ptx::tc_fence_after();

    if (warp == TMA_WARP) {
        // ------------------------------------------------------------ TMA producer (each CTA)
        if (lane == 0) {
            int p = 0;
            uint32_t round = 0;
            for (int64_t tl = 0; tl < my_tiles; ++tl) {
                const uint32_t t32 = cid + (uint32_t)tl * ncl;
                int32_t rl, rc;
                if (TRI) {
                    uint32_t P, J;
                    pair_decode(nlb32, t32, P, J);
                    rl = (int32_t)((2 * P + rank) * BM);
                    rc = (int32_t)(J * BNP + rank * BNH);
                } else {
                    rl = (int32_t)(tile_lb(t32) * (2 * BM) + rank * BM);
                    rc = (int32_t)(tile_cb(t32) * BNP + rank * BNH);
                }
                for (int s = 0; s < nst; ++s) {
                    if (round > 0) ptx::mbar_wait(&pempty[p], (round - 1) & 1);
                    ptx::mbar_arrive_expect_tx(&pfull[p], PSLOT);
                    ptx::tma_load_2d(ring + p * PSLOT, &tmL, &pfull[p], s * KW, rl);
                    ptx::tma_load_2d(ring + p * PSLOT + BM * PROW, &tmC, &pfull[p], s * KW, rc);
                    if (++p == NP) { p = 0; ++round; }
                }
            }
        }
    } else if (warp < NEXP) {
        // ------------------------------------------------------------ expanders (each CTA)
        // group g = warp / 6: warps 0-3 expand the 128 lane rows (lane quarter q) into TMEM,
        // warps 4-5 the 64 column rows (32 each) into the stage's shared-memory B operand.
        // A warps take the TMEM lane quarter warp % 4 (a warp may only access that quarter:
        // the 4 A warps of a group are 4 consecutive warp ids, so they cover all four)
        const int g = warp / GW, r6 = warp - g * GW;
        const bool is_a = r6 < 4;
        const int row = is_a ? (warp & 3) * 32 + lane : (r6 - 4) * 32 + lane;
        const int sw = (row >> 1) & 3;                  // TMA 64B swizzle of a 64-byte row
        const uint32_t tAq = tmem + ((uint32_t)((warp & 3) * 32) << 16) + (uint32_t)A_COL0;
        int s = g % nst;
        int slot = g % NS;
        uint32_t use = (uint32_t)(g / NS);
        static_assert(NP % G == 0, "each packed slot belongs to one expander group");
        int pk = g;
        uint32_t pround = 0;
        for (int64_t it = g; it < total_it; it += G) {
#ifdef GEMM_TRACE
            // warp 0 (group 0, lane quarter 0) of both CTAs of cluster 0: loop start, empty
            // seen, packed stage seen, arrivals done
            const bool tr = SNP_PROF(args.trace) && blockIdx.x < 2 && warp == 0 && lane == 0 && it < 4096;
            long long *tp = g_gemm_trace + 8 * (it >> 1) + 4 * blockIdx.x;
            if (tr) tp[0] = clock64();
#endif
            if (use > 0) ptx::mbar_wait_warp(&empty[slot], (use - 1) & 1);
#ifdef GEMM_TRACE
            if (tr) tp[1] = clock64();
#endif
            ptx::mbar_wait_warp(&pfull[pk], pround & 1);
#ifdef GEMM_TRACE
            if (tr) tp[2] = clock64();
#endif
#ifdef GEMM_DEBUG_SKIP
            if (SNP_PROF(args.debug_skip)) {   // profiling experiment: tokens only (results invalid)
                __syncwarp();
                if (lane == 0) { ptx::mbar_arrive(&pempty[pk]); arrive_remote(&full[slot], 0); }
#ifdef GEMM_TRACE
                if (tr) tp[3] = clock64();
#endif
                s += G;
                while (s >= nst) s -= nst;
                slot += G;
                if (slot >= NS) { slot -= NS; ++use; }
                pk += G;
                if (pk >= NP) { pk -= NP; ++pround; }
                continue;
            }
#endif
            const uint8_t *src = ring + pk * PSLOT + (is_a ? 0 : BM * PROW) + row * PROW;
            uint32_t w[KW];
#pragma unroll
            for (int c = 0; c < 4; ++c) {
                const uint4 x = *reinterpret_cast<const uint4 *>(src + ((c ^ sw) << 4));
                w[4 * c] = x.x; w[4 * c + 1] = x.y; w[4 * c + 2] = x.z; w[4 * c + 3] = x.w;
            }
            const int64_t w0 = (int64_t)s * KW;
            if (w0 + KW > full32) {
#pragma unroll
                for (int i = 0; i < KW; ++i) w[i] &= word_mask(w0 + i, nbits);
            }
            if (is_a) {
                const uint32_t tA = tAq + 64 * slot;
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    uint32_t v[32];
#pragma unroll
                    for (int i = 0; i < 8; ++i)
                        expandA(w[8 * h + i], v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
                    ptx::tmem_st32(tA + 32 * h, v);
                }
                ptx::tmem_st_wait();
                ptx::tc_fence_before();
            } else {
                uint8_t *dstB = bexp + (size_t)slot * BSLOT + row * 16;
#pragma unroll
                for (int i = 0; i < KW; ++i) {          // chunk i of the K-major operand = word i
                    uint4 o;
                    expandB(w[i], o.x, o.y, o.z, o.w);
                    *reinterpret_cast<uint4 *>(dstB + (size_t)i * BNH * 16) = o;
                }
                ptx::fence_proxy_async_smem();
            }
            __syncwarp();
            if (lane == 0) {
                ptx::mbar_arrive(&pempty[pk]);
                arrive_remote(&full[slot], 0);   // the leader's MMA waits for both CTAs
            }
            s += G;
            while (s >= nst) s -= nst;
            slot += G;
            if (slot >= NS) { slot -= NS; ++use; }
            pk += G;
            if (pk >= NP) { pk -= NP; ++pround; }
        }
    } else if (warp == MMA_WARP) {
        // ------------------------------------------------------------ MMA issuer (leader only)
        if (leader) {
            constexpr uint32_t IDESC = idesc_mxf4(2 * BM, BNP);
            const uint32_t tmu = __reduce_or_sync(0xffffffffu, tmem);
            const uint32_t sfa = tmu + SF_COL, sfb = tmu + SF_COL + 16;
            const uint64_t bdesc0 = ptx::smem_desc_kmajor_noswizzle(ptx::smem_u32(bexp), BNH * 16, 128);
            constexpr uint32_t BSTEP = (2 * BNH * 16) >> 4;
            int b = 0;
            uint32_t round = 0;
            for (int64_t tl = 0; tl < my_tiles; ++tl) {
                const int acc = (int)(tl & 1);
#ifdef GEMM_TRACE4
                const bool tr4 = SNP_PROF(args.trace) && blockIdx.x == 0 && lane == 0 && tl < 2048;
                long long fw = 0;
                if (tr4) g_gemm_trace[8 * tl + 0] = clock64();
#endif
                if (tl >= 2) wait_cluster_uniform(&acce[acc], (uint32_t)(((tl >> 1) - 1) & 1));
#ifdef GEMM_TRACE4
                if (tr4) g_gemm_trace[8 * tl + 1] = clock64();
#endif
                ptx::tc_fence_after();
                const uint32_t d = tmu + (uint32_t)(acc * ACC_COLS);
                for (int s = 0; s < nst; ++s) {
#ifdef GEMM_TRACE4
                    const long long w0 = clock64();
#endif
                    wait_cluster_uniform(&full[b], round & 1);
#ifdef GEMM_TRACE4
                    fw += clock64() - w0;
#endif
                    ptx::tc_fence_after();
                    const uint32_t a0 = tmu + (uint32_t)(A_COL0 + 64 * b);
                    const uint64_t b0 = bdesc0 + (uint64_t)(((uint32_t)b * BSLOT) >> 4);
#ifndef GEMM_X2_ELECT_STAGE
#define GEMM_X2_ELECT_STAGE 0   // one elect per stage: measured LD-32K 2.91 -> 3.00 ms, off
#endif
                    if (GEMM_X2_ELECT_STAGE) {
                        if (ptx::elect_one()) {
#pragma unroll
                            for (int k = 0; k < KBITS / 64; ++k)
                                mma_mxf4_ts2_one(d, a0 + 8 * k, b0 + (uint64_t)(k * BSTEP), IDESC,
                                                 (s | k) != 0 ? 1u : 0u, sfa, sfb);
                            commit_both_one(&empty[b]);
                            if (s == nst - 1) commit_both_one(&accf[acc]);
                        }
                        __syncwarp();
                    } else {
#pragma unroll
                        for (int k = 0; k < KBITS / 64; ++k)
                            mma_mxf4_ts2(d, a0 + 8 * k, b0 + (uint64_t)(k * BSTEP), IDESC, (s | k) != 0 ? 1u : 0u,
                                         sfa, sfb);
                        commit_both(&empty[b]);
                        if (s == nst - 1) commit_both(&accf[acc]);
                    }
                    if (++b == NS) { b = 0; ++round; }
                }
#ifdef GEMM_TRACE4
                if (tr4) { g_gemm_trace[8 * tl + 2] = clock64(); g_gemm_trace[8 * tl + 5] = fw; }
#endif
            }
        }
        __syncwarp();
    } else {
        // ------------------------------------------------------------ epilogue (each CTA)
        // warp e: TMEM lane quarter e % 4 of this CTA's 128 lane rows, columns [64 h, 64 h + 64)
        const int e = warp - EPI_WARP0;
        const int q = e & 3, h = e >> 2;
        const int li = q * 32 + lane;
        const int c0 = 64 * h;
        const int64_t n = nbits;
        const bool small_n = n <= 46340;
        const bool need_pop = EPI == EPI_LD || args.op != 0 || (args.C2 && args.op2 != 0);
        const bool want_dp = EPI == EPI_LD && args.dprime != nullptr;
        for (int64_t tl = 0; tl < my_tiles; ++tl) {
            const int acc = (int)(tl & 1);
            const uint32_t ph = (uint32_t)((tl >> 1) & 1);
            const uint32_t t32 = cid + (uint32_t)tl * ncl;
            int64_t gl, gc0, erow0 = 0;
            bool store = true;
            if (TRI) {   // this CTA's tile (I, J) of the pair; virtual [ntri 128][128] output
                uint32_t P, J;
                pair_decode(nlb32, t32, P, J);
                const uint32_t I = 2 * P + rank;
                store = I <= J && I < nlb32;
                gl = (int64_t)I * BM + li;
                gc0 = (int64_t)J * BNP + c0;
                erow0 = (store ? tri_start(nlb32, I) + (int64_t)(J - I) : 0) * BM + q * 32;
            } else {
                gl = (int64_t)tile_lb(t32) * (2 * BM) + rank * BM + li;
                gc0 = (int64_t)tile_cb(t32) * BNP + c0;
            }
            const int64_t nlr = TRI ? args.mreal : args.nl, ncr = TRI ? args.mreal : args.nc;
            const int ncols = gc0 < ncr ? (int)(ncr - gc0 < 64 ? ncr - gc0 : 64) : 0;
            uint32_t pl = 0, pcol0 = 0, pcol1 = 0;
            if (need_pop) {
                if (gl < nlr) pl = __ldg(args.popL + gl);
                if (lane < ncols) pcol0 = __ldg(args.popC + gc0 + lane);
                if (32 + lane < ncols) pcol1 = __ldg(args.popC + gc0 + 32 + lane);
            }
            ptx::mbar_wait_warp(&accf[acc], ph);
#ifdef GEMM_TRACE4
            if (SNP_PROF(args.trace) && blockIdx.x == 0 && e == 0 && lane == 0 && tl < 2048) g_gemm_trace[8 * tl + 3] = clock64();
#endif
            ptx::tc_fence_after();
            const uint32_t ta = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(acc * ACC_COLS + c0);
            const float ia = EPI == EPI_LD ? inv_exact((int64_t)pl * (n - (int64_t)pl)) : 0.f;
#pragma unroll 1
            for (int hh = 0; hh < 2; ++hh) {
                uint32_t v[32];
                __syncwarp();
                ptx::tmem_ld32(ta + 32 * hh, v);
                ptx::tmem_ld_wait();
                if (hh == 1) {
                    ptx::tc_fence_before();
                    __syncwarp();
                    if (lane == 0) arrive_remote(&acce[acc], 0);   // drained: the leader may reuse it
#ifdef GEMM_TRACE4
                    if (SNP_PROF(args.trace) && blockIdx.x == 0 && e == 0 && lane == 0 && tl < 2048) g_gemm_trace[8 * tl + 4] = clock64();
#endif
                }
                if (TRI) {
                    if (store)
                        epi_transposed<EPI>(args, v, trs + e * 32 * 32, lane, erow0, (int64_t)c0 + 32 * hh, pl,
                                            hh ? pcol1 : pcol0, ia, small_n, want_dp, false);
                    continue;
                }
                epi_transposed<EPI>(args, v, trs + e * 32 * 32, lane, gl - lane, gc0 + 32 * hh, pl,
                                    hh ? pcol1 : pcol0, ia, small_n, want_dp, false);
            }
        }
    }

    ptx::tc_fence_before();
    __syncthreads();
    cluster_sync();   // no CTA leaves (or frees TMEM) while its peer may still signal it
    if (warp == MMA_WARP) {
        ptx::tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 512;" ::"r"(tmem) : "memory");
    }
}

bool make_map(CUtensorMap *tm, const uint32_t *base, int64_t rows, int64_t ld32, uint32_t box_rows = 128) {
    return make_map_u32_2d(tm, base, rows, ld32, KW, box_rows, CU_TENSOR_MAP_SWIZZLE_64B);
}

// Pre-expanded column operand (BPRE): word w of row r -> the 16 bytes expandB(w) at
// out[r * wrow + w], zeros for words past nbits (so the row pitch wrow * 16 bytes holds
// whole 512-bit stages).  Coalesced 4-byte reads, 16-byte writes.
__global__ void expand_b_kernel(const uint32_t *__restrict__ A, int64_t m, int64_t lda32, int64_t nbits,
                                int64_t wrow, uint4 *__restrict__ out) {
    const int64_t total = m * wrow;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = i / wrow, w = i - r * wrow;
        const uint32_t msk = word_mask(w, nbits);
        const uint32_t x = msk ? __ldg(A + r * lda32 + w) & msk : 0u;
        uint4 o;
        expandB(x, o.x, o.y, o.z, o.w);
        out[i] = o;
    }
}

template <int EPI, bool TRI = false, bool BPRE = false>
cudaError_t launch_g(const GArgs &g, const uint32_t *L, int64_t ldl32, const uint32_t *Cn, int64_t ldc32,
                     cudaStream_t s) {
    CUtensorMap tmL, tmC;
    // packed-triangle launches keep virtual output sizes in g.nl / g.nc: the operands have m rows
    const int64_t rows_l = TRI ? g.mreal : g.nl, rows_c = TRI ? g.mreal : g.nc;
    if (!make_map(&tmL, L, rows_l, ldl32)) return cudaErrorInvalidValue;
    if (BPRE) {   // Cn = the expanded operand, ldc32 its row pitch in 32-bit words; 128-byte boxes
        if (!make_map_u32_2d(&tmC, Cn, rows_c, ldc32, 32, BN, CU_TENSOR_MAP_SWIZZLE_128B))
            return cudaErrorInvalidValue;
    } else if (!make_map(&tmC, Cn, rows_c, ldc32)) {
        return cudaErrorInvalidValue;
    }
    auto kern = gemm_tc4_kernel<EPI, TRI, BPRE>;
    if (cudaError_t e = ensure_dyn_smem(reinterpret_cast<const void *>(kern), (int)SMEM); e != cudaSuccess) return e;
    const int64_t ntiles = TRI ? g.ntri : g.sym ? g.nlb * (g.nlb + 1) / 2 : g.nlb * g.ncb;
    if (ntiles <= 0) return cudaSuccess;
    const int grid = (int)(ntiles < device_sms() ? ntiles : device_sms());
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3((unsigned)NTHREADS);
    cfg.dynamicSmemBytes = SMEM;
    cfg.stream = s;
    cudaLaunchAttribute pdl[1];
    pdl[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    pdl[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = pdl;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, kern, tmL, tmC, g);
    count_launches(1);
    if (e != cudaSuccess) return e;
    return cudaGetLastError();
}

template <int EPI, bool TRI = false>
cudaError_t launch_g2(GArgs g, const uint32_t *L, int64_t ldl32, const uint32_t *Cn, int64_t ldc32, cudaStream_t s) {
    CUtensorMap tmL, tmC;
    const int64_t rows_l = TRI ? g.mreal : g.nl, rows_c = TRI ? g.mreal : g.nc;
    if (!make_map(&tmL, L, rows_l, ldl32, 128) || !make_map(&tmC, Cn, rows_c, ldc32, x2::BNH))
        return cudaErrorInvalidValue;
    auto kern = gemm_tc4x2_kernel<EPI, TRI>;
    if (cudaError_t e = ensure_dyn_smem(reinterpret_cast<const void *>(kern), (int)x2::SMEM); e != cudaSuccess)
        return e;
    int64_t npairs;
    if (TRI) {   // g.nlb = T; pair tiles over the whole triangle
        npairs = pair_start(g.nlb, (g.nlb + 1) / 2);
        g.ntri = npairs;
    } else {
        g.nlb = (g.nl + 2 * BM - 1) / (2 * BM);
        g.ncb = (g.nc + x2::BNP - 1) / x2::BNP;
        npairs = g.nlb * g.ncb;
    }
    // co-resident 2-CTA clusters: a GPC with an odd SM count leaves one SM unpaired, so
    // SMs / 2 clusters would run a second wave of a few clusters (doubling the time)
    int pairs = device_sms() / 2;
    {
        cudaLaunchConfig_t qc{};
        qc.gridDim = dim3(2 * (unsigned)pairs);
        qc.blockDim = dim3((unsigned)x2::NTHREADS);
        qc.dynamicSmemBytes = x2::SMEM;
        cudaLaunchAttribute ca[1];
        ca[0].id = cudaLaunchAttributeClusterDimension;
        ca[0].val.clusterDim.x = 2; ca[0].val.clusterDim.y = 1; ca[0].val.clusterDim.z = 1;
        qc.attrs = ca;
        qc.numAttrs = 1;
        int nc = 0;
        if (cudaOccupancyMaxActiveClusters(&nc, reinterpret_cast<const void *>(kern), &qc) == cudaSuccess && nc > 0 &&
            nc < pairs)
            pairs = nc;
        static const bool report = std::getenv("SNP_X2_REPORT") != nullptr;
        if (report) fprintf(stderr, "x2: %d co-resident clusters (SMs %d)\n", nc, device_sms());
    }
    const int grid = 2 * (int)(npairs < pairs ? npairs : pairs);
    kern<<<grid, x2::NTHREADS, x2::SMEM, s>>>(tmL, tmC, g);
    count_launches(1);
    return cudaGetLastError();
}

}  // namespace

namespace {
thread_local bool g_last_sym = false;
thread_local bool g_last_pair = false;
}
bool gemm_tc4_last_sym() { return g_last_sym; }
bool gemm_tc4_last_pair() { return g_last_pair; }

size_t gemm_tc4_bpre_bytes(int64_t m, int64_t nbits) {
    return (size_t)m * (size_t)((nbits + KBITS - 1) / KBITS) * KW * 16;
}

bool gemm_tc4_supported(int64_t m, int64_t n, int64_t nbits) {
    return m >= 1 && n >= 1 && nbits >= 1 && nbits < (1LL << 24) && m < (1LL << 31) && n < (1LL << 31);
}

// SNP_GEMM_X2: "1" forces the CTA-pair kernel where it applies, "0" the 1-CTA kernel,
// unset = the shape default
static int x2_mode() {
    static const int m = [] {
        const char *e = std::getenv("SNP_GEMM_X2");
        return e && e[0] == '1' ? 1 : e && e[0] == '0' ? 0 : -1;
    }();
    return m;
}

cudaError_t launch_gemm_tc4(const GemmArgs &a, int epi, cudaStream_t s) {
    GArgs g{};
    g_last_pair = false;
#ifdef SNP_PROFILING
    static const bool trace = std::getenv("SNP_TRACE") && std::getenv("SNP_TRACE")[0] == '1';
    g.trace = trace ? 1 : 0;
    static const char *skip = std::getenv("SNP_DEBUG_SKIP_EXPAND");
    g.debug_skip = skip ? skip[0] - '0' : 0;
#endif
    if (a.tri_n >= 0) {   // f3 packed triangle: self-LD only (A == B), no swap, no mirror
        if (a.m != a.n || a.A != a.B || a.lda32 != a.ldb32 || a.C2) return cudaErrorInvalidValue;
        g.popL = a.popA;
        g.popC = a.popA;
        g.mreal = a.m;
        g.nl = a.tri_n * BM;   // the epilogue's virtual [ntri * 128][128] output (see the kernel)
        g.nc = BN;
        g.nbits = a.nbits;
        g.op = a.op;
        g.accumulate = a.accumulate;
        g.ldo = BN;
        g.C = a.C;
        g.r2 = a.r2;
        g.dprime = a.dprime;
        g.nlb = g.ncb = (a.m + BM - 1) / BM;
        g.nst = (int)((a.nbits + KBITS - 1) / KBITS);
        g.tri = 1;
        g.tlo = a.tri_lo;
        g.ntri = a.tri_n;
        g.off32 = (uint64_t)a.tri_n * BM * BN < (1ull << 32) ? 1 : 0;   // virtual row * 128 + col
        g.v4 = (((uintptr_t)a.r2 & 15u) == 0 && ((uintptr_t)a.C & 15u) == 0) ? 1 : 0;
        g.order = 2;
        g_last_sym = true;
        const int64_t T = g.nlb;
        const bool whole = a.tri_lo == 0 && a.tri_n == T * (T + 1) / 2 && a.tri_n < (1LL << 31);
        const int x2m = x2_mode();
        if (whole && !a.bpre && (x2m == 1 || (x2m < 0 && pair_start(T, (T + 1) / 2) >= device_sms()))) {
            // whole triangle on CTA pairs (tcgen05 cta_group::2, M = 256 pair tiles): half of
            // the B operand's expansion, shared-memory writes and MMA reads per SM (LD-32K
            // 3.50 -> 2.95 ms).  Default from two waves of pair tiles up (LD-2K, one wave:
            // equal kernel time, +1 us launch), partial ranges keep the 1-CTA kernel
            g_last_pair = true;
            return epi == EPI_LD ? launch_g2<EPI_LD, true>(g, a.A, a.lda32, a.A, a.lda32, s)
                                 : launch_g2<EPI_COUNTS, true>(g, a.A, a.lda32, a.A, a.lda32, s);
        }
        if (a.bpre && whole) {
            // whole triangle with the pre-expanded column operand (a.bpre: bpre_bytes(m, nbits))
            const int64_t wrow = (int64_t)g.nst * KW;
            const int64_t total = a.m * wrow;
            const int blocks = (int)std::min<int64_t>((total + 255) / 256, (int64_t)device_sms() * 16);
            expand_b_kernel<<<blocks, 256, 0, s>>>(a.A, a.m, a.lda32, a.nbits, wrow, reinterpret_cast<uint4 *>(a.bpre));
            count_launches(1);
            if (cudaError_t e = cudaGetLastError(); e != cudaSuccess) return e;
            return epi == EPI_LD ? launch_g<EPI_LD, true, true>(g, a.A, a.lda32, a.bpre, wrow * 4, s)
                                 : launch_g<EPI_COUNTS, true, true>(g, a.A, a.lda32, a.bpre, wrow * 4, s);
        }
        return epi == EPI_LD ? launch_g<EPI_LD, true>(g, a.A, a.lda32, a.A, a.lda32, s)
                             : launch_g<EPI_COUNTS, true>(g, a.A, a.lda32, a.A, a.lda32, s);
    }
    const bool swap = a.m < a.n;     // larger operand on TMEM lanes
    g.popL = swap ? a.popB : a.popA;
    g.popC = swap ? a.popA : a.popB;
    const uint32_t *L = swap ? a.B : a.A, *Cn = swap ? a.A : a.B;
    const int64_t ldl32 = swap ? a.ldb32 : a.lda32, ldc32 = swap ? a.lda32 : a.ldb32;
    g.nl = swap ? a.n : a.m;
    g.nc = swap ? a.m : a.n;
    g.nbits = a.nbits;
    g.swap = swap ? 1 : 0;
    g.op = a.op;
    g.op2 = a.op2;
    g.C2 = a.C2;
    if (g.C2 && !swap) return cudaErrorInvalidValue;   // two-op epilogue: swapped layout only
    g.accumulate = a.accumulate;
    g.ldo = a.ldc;
    g.C = a.C;
    g.r2 = a.r2;
    g.dprime = a.dprime;
    g.nlb = (g.nl + BM - 1) / BM;
    g.ncb = (g.nc + BN - 1) / BN;
    g.nst = (int)((a.nbits + KBITS - 1) / KBITS);
    g.off32 = (uint64_t)(swap ? a.n : a.m) * (uint64_t)a.ldc < (1ull << 32) ? 1 : 0;
    g.v4 = (a.ldc % 4 == 0 && ((uintptr_t)a.r2 & 15u) == 0 && ((uintptr_t)a.C & 15u) == 0) ? 1 : 0;
    // f3 symmetric self-LD (B aliases A, symmetric output: LD statistics, AND or XOR
    // counts): only the upper-triangle tiles are computed, off-diagonal ones mirrored.
    // With the vectorised mirror epilogue this wins from two tile rows up (LD-2K 41.6 ->
    // 35.5 us, LD-32K 7.1 -> 4.0 ms).  SNP_GEMM_SYM=0 computes every tile.
    static const char *syme = std::getenv("SNP_GEMM_SYM");
    const int64_t full_tiles = ((a.m + BM - 1) / BM) * ((a.n + BN - 1) / BN);
    g.sym = (!swap && a.A == a.B && a.m == a.n && a.lda32 == a.ldb32 && (epi == EPI_LD || a.op <= 1) &&
             full_tiles > 1 && !(syme && syme[0] == '0')) ? 1 : 0;
    static const char *ord = std::getenv("SNP_GEMM_ORDER");
    // raster: grouped (2) for LD; lane-block-major (1) for the swapped many-query FastID shape,
    // where all query blocks of a database block run together (configs[3] on 1 GPU: 102.7 ->
    // 95.8 ms for the counts pass; scripts/gpu_f20m_order.sh)
    g.order = ord ? (ord[0] - '0') : (swap ? 1 : 2);
    // CTA-pair kernel for the unswapped shapes with more than one lane block: opt-in
    // (SNP_GEMM_X2=1) here, see DESIGN.md §9 for the measured default.
    const bool use_x2 = !swap && g.nl > BM && x2_mode() == 1;
    if (use_x2) g.sym = 0;
    g_last_sym = g.sym != 0;
    g_last_pair = use_x2;
    if (use_x2)
        return epi == EPI_LD ? launch_g2<EPI_LD>(g, L, ldl32, Cn, ldc32, s) : launch_g2<EPI_COUNTS>(g, L, ldl32, Cn, ldc32, s);
    return epi == EPI_LD ? launch_g<EPI_LD>(g, L, ldl32, Cn, ldc32, s) : launch_g<EPI_COUNTS>(g, L, ldl32, Cn, ldc32, s);
}

}  // namespace snp

#ifdef SNP_PROFILING
extern "C" int snp_debug_gemm_cta2(long long *host, int n) {
    if (n > 8 * 1024) n = 8 * 1024;
    return (int)cudaMemcpyFromSymbol(host, snp::g_gemm_cta2, sizeof(long long) * n);
}

extern "C" int snp_debug_gemm_cta(long long *host, int n) {
    if (n > 8 * 1024) n = 8 * 1024;
    return (int)cudaMemcpyFromSymbol(host, snp::g_gemm_cta, sizeof(long long) * n);
}

extern "C" int snp_debug_gemm_trace(long long *host, int n) {
    if (n > 8 * 2048) n = 8 * 2048;
    return (int)cudaMemcpyFromSymbol(host, snp::g_gemm_trace, sizeof(long long) * n);
}

// Debug aid (not in include/snp.h): mode 1 makes a stuck gemm_tc4 pipeline record where
// it waited and release all waits instead of trapping; returns and clears the record.
extern "C" int snp_debug_gemm_watchdog(int mode, int *record8) {
    cudaMemcpyToSymbol(snp::ptx::g_snp_watchdog_mode, &mode, sizeof(int));
    if (record8) cudaMemcpyFromSymbol(record8, snp::ptx::g_snp_watchdog, 8 * sizeof(int));
    int zero[8] = {0};
    cudaMemcpyToSymbol(snp::ptx::g_snp_watchdog, zero, sizeof(zero));
    return (int)cudaGetLastError();
}
#endif  // SNP_PROFILING
