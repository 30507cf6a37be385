// bitgemm_popc.cu — CUDA-core variant of the bit-GEMM:
//
//   C[i][j] = sum_w POPC(A[i][w] op B[j][w])     (§III: "logical and (&),
//   population count (POPC), and integer addition (+)" replacing multiply-add)
//
// op = AND (Eq. 1), XOR (Eq. 2), ANDNOT = A & ~B and NOTAND = ~A & B
// (Eq. 3 rewritten).  Each op is ONE LOP3 on sm_100a, so AND, XOR and
// AND-NOT run at the same rate (the paper's Fig. 9 observation for NVIDIA).
//
// B200 design (not the paper's OpenCL BLIS mapping, which is prior art):
//  * Block tile BM x BN outputs, 256 threads, each thread an 8x8 register tile
//    (64 uint32 accumulators).  Per 32-bit k-word a thread does 4 LDS.128 and
//    64 x (LOP3 + POPC + IADD): the POPC pipe (16/clk/SM) binds, LOP3/IADD3
//    use < 40 % of the ALU pipe.
//  * K is streamed in BK = 16-word (512-bit) stages through a double-buffered
//    shared-memory tile stored k-major ([BK][BM]) so that a thread's 4 rows are one
//    LDS.128; the next stage is prefetched into registers with 128-bit global
//    loads while the current one is consumed.
//  * Tail bits >= nbits are masked to zero in BOTH operands at load time, so every
//    op contributes 0 there; rows past m/n are zero-filled and never stored.
//  * Epilogues fused: counts (=, +=) or the LD statistics r2 / D'
//    from exact integers.
#include "snp_internal.h"
#include "e2m1.cuh"

namespace snp {
namespace {

constexpr int BK = 16;        // uint32 k-words per stage (512 bits)
constexpr int TM = 8, TN = 8; // per-thread register tile
constexpr int NT = 256;

template <int OP>
__device__ __forceinline__ uint32_t bitop(uint32_t a, uint32_t b) {
    if (OP == 0) return a & b;        // AND    (Eq. 1)
    if (OP == 1) return a ^ b;        // XOR    (Eq. 2)
    if (OP == 2) return a & ~b;       // ANDNOT (Eq. 3, r = A row)
    return ~a & b;                    // NOTAND (Eq. 3, r = B row)
}


// LD statistics from exact integers (reading R3).
__device__ __forceinline__ void ld_stats(int64_t n, int64_t na, int64_t nb, int64_t nab,
                                         float &r2, float &dp) {
    const int64_t num = n * nab - na * nb;
    const int64_t da = na * (n - na), db = nb * (n - nb);
    r2 = (da == 0 || db == 0) ? 0.f
                               : (float)(((double)num * (double)num) / ((double)da * (double)db));
    int64_t dmax = 0;
    if (num > 0) {
        const int64_t x = na * (n - nb), y = (n - na) * nb;
        dmax = x < y ? x : y;
    } else if (num < 0) {
        const int64_t x = na * nb, y = (n - na) * (n - nb);
        dmax = x < y ? x : y;
    }
    dp = dmax ? (float)((double)num / (double)dmax) : 0.f;
}

template <int BM, int BN, int OP, int EPI>
__global__ void __launch_bounds__(NT, 1)
bitgemm_popc_kernel(const GemmArgs args) {
    constexpr int TX = BN / TN;              // threads along N
    constexpr int TY = BM / TM;              // threads along M
    static_assert(TX * TY == NT, "tile/threads mismatch");
    constexpr int A_VEC = BM * BK / 4 / NT;  // uint4 loads per thread per stage
    constexpr int B_VEC = BN * BK / 4 / NT;

    __shared__ __align__(16) uint32_t As[2][BK][BM];
    __shared__ __align__(16) uint32_t Bs[2][BK][BN];

    const int tid = threadIdx.x;
    const int tx = tid % TX, ty = tid / TX;
    int64_t m0 = (int64_t)blockIdx.y * BM;
    int64_t n0 = (int64_t)blockIdx.x * BN;
    // outputs: row-major [m][ldc], or (f3 packed triangle) tile blockIdx.x of the call as a
    // dense BM x BN block — shifting the bases keeps the (row * ldc + col) addressing below
    uint32_t *Cp = args.C;
    float *r2p = args.r2, *dpp = args.dprime;
    int64_t ldc = args.ldc;
    const bool tri = args.tri_n >= 0;
    if (tri) {
        uint32_t I, J;
        tri_decode((args.m + BM - 1) / BM, args.tri_lo + blockIdx.x, I, J);
        m0 = (int64_t)I * BM;
        n0 = (int64_t)J * BN;
        ldc = BN;
        const int64_t delta = (int64_t)blockIdx.x * (BM * BN) - m0 * BN - n0;
        if (Cp) Cp += delta;
        if (r2p) r2p += delta;
        if (dpp) dpp += delta;
    }
    const int64_t nbits = args.nbits;
    const int64_t nchunk32 = ((nbits + 127) / 128) * 4;   // uint32 words actually read
    const int nstages = (int)((nchunk32 + BK - 1) / BK);

    // global -> register staging.  Element e of this thread: row = e_lin % ROWS,
    // vec = e_lin / ROWS, so consecutive threads take consecutive rows (conflict-free STS).
    uint4 ra[A_VEC], rb[B_VEC];

    auto load_stage = [&](int st) {
        const int64_t kw0 = (int64_t)st * BK;
#pragma unroll
        for (int e = 0; e < A_VEC; ++e) {
            const int lin = tid + e * NT;
            const int r = lin % BM, v = lin / BM;
            const int64_t gr = m0 + r, kw = kw0 + 4 * v;
            uint4 x = make_uint4(0, 0, 0, 0);
            if (gr < args.m && kw < nchunk32) {
                x = __ldg(reinterpret_cast<const uint4 *>(args.A + gr * args.lda32 + kw));
                if (kw + 4 > nbits / 32) {
                    x.x &= word_mask(kw, nbits); x.y &= word_mask(kw + 1, nbits);
                    x.z &= word_mask(kw + 2, nbits); x.w &= word_mask(kw + 3, nbits);
                }
            }
            ra[e] = x;
        }
#pragma unroll
        for (int e = 0; e < B_VEC; ++e) {
            const int lin = tid + e * NT;
            const int r = lin % BN, v = lin / BN;
            const int64_t gr = n0 + r, kw = kw0 + 4 * v;
            uint4 x = make_uint4(0, 0, 0, 0);
            if (gr < args.n && kw < nchunk32) {
                x = __ldg(reinterpret_cast<const uint4 *>(args.B + gr * args.ldb32 + kw));
                if (kw + 4 > nbits / 32) {
                    x.x &= word_mask(kw, nbits); x.y &= word_mask(kw + 1, nbits);
                    x.z &= word_mask(kw + 2, nbits); x.w &= word_mask(kw + 3, nbits);
                }
            }
            rb[e] = x;
        }
    };
    auto store_stage = [&](int buf) {
#pragma unroll
        for (int e = 0; e < A_VEC; ++e) {
            const int lin = tid + e * NT;
            const int r = lin % BM, v = lin / BM;
            As[buf][4 * v + 0][r] = ra[e].x; As[buf][4 * v + 1][r] = ra[e].y;
            As[buf][4 * v + 2][r] = ra[e].z; As[buf][4 * v + 3][r] = ra[e].w;
        }
#pragma unroll
        for (int e = 0; e < B_VEC; ++e) {
            const int lin = tid + e * NT;
            const int r = lin % BN, v = lin / BN;
            Bs[buf][4 * v + 0][r] = rb[e].x; Bs[buf][4 * v + 1][r] = rb[e].y;
            Bs[buf][4 * v + 2][r] = rb[e].z; Bs[buf][4 * v + 3][r] = rb[e].w;
        }
    };

    uint32_t acc[TM][TN];
#pragma unroll
    for (int i = 0; i < TM; ++i)
#pragma unroll
        for (int j = 0; j < TN; ++j) acc[i][j] = 0;

    if (nstages > 0) {
        load_stage(0);
        store_stage(0);
    }
    __syncthreads();

    for (int st = 0; st < nstages; ++st) {
        const int buf = st & 1;
        if (st + 1 < nstages) load_stage(st + 1);
#pragma unroll 4
        for (int kk = 0; kk < BK; ++kk) {
            uint32_t a0[TM], b0[TN];
            // rows ty*4..+3 and BM/2+ty*4..+3 ; cols tx*4..+3 and BN/2+tx*4..+3
            *reinterpret_cast<uint4 *>(&a0[0]) = *reinterpret_cast<const uint4 *>(&As[buf][kk][ty * 4]);
            *reinterpret_cast<uint4 *>(&a0[4]) = *reinterpret_cast<const uint4 *>(&As[buf][kk][BM / 2 + ty * 4]);
            *reinterpret_cast<uint4 *>(&b0[0]) = *reinterpret_cast<const uint4 *>(&Bs[buf][kk][tx * 4]);
            *reinterpret_cast<uint4 *>(&b0[4]) = *reinterpret_cast<const uint4 *>(&Bs[buf][kk][BN / 2 + tx * 4]);
#pragma unroll
            for (int i = 0; i < TM; ++i)
#pragma unroll
                for (int j = 0; j < TN; ++j)
                    acc[i][j] += __popc(bitop<OP>(a0[i], b0[j]));
        }
        if (st + 1 < nstages) {
            store_stage(buf ^ 1);
        }
        __syncthreads();
    }

    // ---------------- epilogue
#pragma unroll
    for (int i = 0; i < TM; ++i) {
        const int64_t gi = m0 + (i < 4 ? ty * 4 + i : BM / 2 + ty * 4 + (i - 4));
        // packed triangle: a tile's entries past m are written too, as the zeros they compute
        if (gi >= args.m && !tri) continue;
        int64_t na = 0;
        if (EPI == EPI_LD && gi < args.m) na = args.popA[gi];
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int64_t gj0 = n0 + (h == 0 ? tx * 4 : BN / 2 + tx * 4);
            const int64_t base = gi * ldc + gj0;
            if (EPI == EPI_COUNTS) {
                uint32_t v[4] = {acc[i][4 * h], acc[i][4 * h + 1], acc[i][4 * h + 2], acc[i][4 * h + 3]};
                const bool vec = (tri || gj0 + 4 <= args.n) && ((base & 3) == 0);
                if (vec) {
                    uint4 *p = reinterpret_cast<uint4 *>(Cp + base);
                    if (args.accumulate) {
                        uint4 o = *p;
                        v[0] += o.x; v[1] += o.y; v[2] += o.z; v[3] += o.w;
                    }
                    *p = make_uint4(v[0], v[1], v[2], v[3]);
                } else {
#pragma unroll
                    for (int q = 0; q < 4; ++q)
                        if (tri || gj0 + q < args.n)
                            Cp[base + q] = args.accumulate ? Cp[base + q] + v[q] : v[q];
                }
            } else {
                float r2v[4], dpv[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int64_t gj = gj0 + q;
                    const int64_t nb = gj < args.n ? (int64_t)args.popB[gj] : 0;
                    ld_stats(args.nbits, na, nb, (int64_t)acc[i][4 * h + q], r2v[q], dpv[q]);
                }
                const bool vec = (tri || gj0 + 4 <= args.n) && ((base & 3) == 0);
                if (vec) {
                    *reinterpret_cast<float4 *>(r2p + base) = make_float4(r2v[0], r2v[1], r2v[2], r2v[3]);
                    if (dpp)
                        *reinterpret_cast<float4 *>(dpp + base) = make_float4(dpv[0], dpv[1], dpv[2], dpv[3]);
                    if (Cp)
                        *reinterpret_cast<uint4 *>(Cp + base) =
                            make_uint4(acc[i][4 * h], acc[i][4 * h + 1], acc[i][4 * h + 2], acc[i][4 * h + 3]);
                } else {
#pragma unroll
                    for (int q = 0; q < 4; ++q)
                        if (tri || gj0 + q < args.n) {
                            r2p[base + q] = r2v[q];
                            if (dpp) dpp[base + q] = dpv[q];
                            if (Cp) Cp[base + q] = acc[i][4 * h + q];
                        }
                }
            }
        }
    }
}

template <int BM, int BN, int EPI>
cudaError_t launch_tile(const GemmArgs &a, cudaStream_t s) {
    dim3 grid((unsigned)((a.n + BN - 1) / BN), (unsigned)((a.m + BM - 1) / BM));
    if (a.tri_n >= 0) {   // packed triangle: one block per tile of the call
        if (a.tri_n == 0) return cudaSuccess;
        grid = dim3((unsigned)a.tri_n, 1);
    }
    switch (a.op) {
    case 0: bitgemm_popc_kernel<BM, BN, 0, EPI><<<grid, NT, 0, s>>>(a); break;
    case 1: bitgemm_popc_kernel<BM, BN, 1, EPI><<<grid, NT, 0, s>>>(a); break;
    case 2: bitgemm_popc_kernel<BM, BN, 2, EPI><<<grid, NT, 0, s>>>(a); break;
    default: bitgemm_popc_kernel<BM, BN, 3, EPI><<<grid, NT, 0, s>>>(a); break;
    }
    count_launches(1);
    return cudaGetLastError();
}

}  // namespace

cudaError_t launch_bitgemm_popc(const GemmArgs &a, int epi, cudaStream_t s) {
    if (a.tri_n >= 0) {   // f3 packed triangle: 128 x 128 tiles, grid.x = tiles (< 2^31)
        if (a.tri_n > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
        return epi == EPI_LD ? launch_tile<128, 128, EPI_LD>(a, s) : launch_tile<128, 128, EPI_COUNTS>(a, s);
    }
    // gridDim.y <= 65535: walk M in chunks (offsetting every row-indexed pointer).
    const int64_t BMmax = a.m <= 64 ? 64 : 128;
    const int64_t chunk = 65535 * BMmax;
    for (int64_t r0 = 0; r0 < a.m; r0 += chunk) {
        GemmArgs c = a;
        c.m = a.m - r0 < chunk ? a.m - r0 : chunk;
        c.A = a.A + r0 * a.lda32;
        if (a.C) c.C = a.C + r0 * a.ldc;
        if (a.r2) c.r2 = a.r2 + r0 * a.ldc;
        if (a.dprime) c.dprime = a.dprime + r0 * a.ldc;
        if (a.popA) c.popA = a.popA + r0;
        cudaError_t e;
        if (a.m <= 64)
            e = epi == EPI_LD ? launch_tile<64, 256, EPI_LD>(c, s) : launch_tile<64, 256, EPI_COUNTS>(c, s);
        else
            e = epi == EPI_LD ? launch_tile<128, 128, EPI_LD>(c, s) : launch_tile<128, 128, EPI_COUNTS>(c, s);
        if (e != cudaSuccess) return e;
    }
    return cudaSuccess;
}

}  // namespace snp
