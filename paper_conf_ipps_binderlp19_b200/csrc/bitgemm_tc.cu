// bitgemm_tc.cu — tensor-core variant of the bit-GEMM (SURVEY §8a row a3, §8a "tensor variant").
//
//   C[i][j] = sum_k A_ik & B_jk  (Eq. 1)   computed as an integer GEMM
//
// sm_100a has no native 1-bit MMA (mma.sync ... b1.and.popc is emulated),
// so bits are expanded ON-CHIP to u8 {0,1} and multiplied with tcgen05.mma kind::i8
// (u8 x u8 -> s32, exact for any K < 2^31) with the accumulator in TMEM.  The packed
// operands are what crosses HBM/L2 (8x less traffic than pre-expanded bytes).
//
//   * CTA tile: 128 "lane" rows (the larger operand, TMEM lanes) x BN "column" rows
//     (BN = 64/128/256), the full K loop inside the CTA.
//   * K streamed in stages of 256 bits.  All 8 warps load the packed 256-bit slice of
//     every row of the tile (128-bit LDG, prefetched two stages ahead in registers),
//     expand each 32-bit word w into 32 bytes with (w >> t) & 0x01010101, t = 0..7
//     (2 ALU ops per 4 bytes; a fixed permutation of the 32 bits inside each word,
//     applied identically to both operands, so every count is unchanged), and store
//     them into the K-major no-swizzle UMMA layout of the stage buffer.
//   * One thread issues 8 x tcgen05.mma (M=128, N=BN, K=32) per stage and commits to
//     the stage's mbarrier; the buffer is refilled once that barrier flips, so the
//     expansion of stage s+1 overlaps the MMAs of stage s.
//   * Row popcounts (p_A, p_B of P:L44) are accumulated from the same packed words, so
//     XOR = pQ + pD - 2 AND, ANDNOT = pQ - AND, NOTAND = pD - AND and the LD r2/D'
//     epilogue need no extra pass over HBM.
//   * Epilogue: tcgen05.ld 32x32b.x8 from TMEM, op identity / LD statistics, stores.
//     When the lane side is the second operand (FastID: database rows on lanes,
//     queries on columns) the output is written transposed, coalesced along lanes.
#include "snp_internal.h"
#include "e2m1.cuh"
#include "tc_ptx.cuh"

namespace snp {
namespace {

constexpr int BM = 128;              // MMA M = TMEM lanes
constexpr int KBITS = 256;           // K bits per pipeline stage
constexpr int KW = KBITS / 32;       // packed u32 words per row per stage (= MMA K-steps)
constexpr int NT = 256;              // 8 warps

template <int BN>
struct Cfg {
    static constexpr int ROWS = BM + BN;
    static constexpr int A_BYTES = BM * KBITS;         // expanded: one byte per bit
    static constexpr int B_BYTES = BN * KBITS;
    static constexpr int STAGE = A_BYTES + B_BYTES;
    static constexpr int NS = BN >= 256 ? 2 : (BN >= 128 ? 3 : 4);
    static constexpr int UNITS = (ROWS * 2 + NT - 1) / NT;  // 128-bit packed loads per thread per stage
    static constexpr int TMEM_COLS = BN < 32 ? 32 : BN;
    static constexpr size_t SMEM = (size_t)NS * STAGE + 2048;   // + barriers / popcounts / tmem slot
};

struct TcArgs {
    const uint32_t *L;   // lane-side operand (packed rows, u32 view)
    const uint32_t *Cn;  // column-side operand
    int64_t nl, nc;      // rows
    int64_t ldl32, ldc32;
    int64_t nbits;
    int swap;            // 1: user (i, j) = (column row, lane row)
    int op;
    int accumulate;
    int64_t ldo;
    uint32_t *C;
    float *r2;
    float *dprime;
};


__device__ __forceinline__ void ld_stats(int64_t n, int64_t na, int64_t nb, int64_t nab, float &r2, float &dp) {
    const int64_t num = n * nab - na * nb;
    const int64_t da = na * (n - na), db = nb * (n - nb);
    r2 = (da == 0 || db == 0) ? 0.f : (float)(((double)num * (double)num) / ((double)da * (double)db));
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

template <int BN, int EPI>
__global__ void __launch_bounds__(NT, 1) bitgemm_tc_kernel(const TcArgs args) {
    using C = Cfg<BN>;
    extern __shared__ __align__(1024) uint8_t smem[];
    uint8_t *stage_base = smem;
    uint64_t *empty_bar = reinterpret_cast<uint64_t *>(smem + (size_t)C::NS * C::STAGE);
    uint64_t *done_bar = empty_bar + C::NS;
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(done_bar + 1);
    uint32_t *popL = tmem_slot + 4;            // [BM]
    uint32_t *popC = popL + BM;                // [BN]

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int64_t l0 = (int64_t)blockIdx.x * BM;
    const int64_t c0 = (int64_t)blockIdx.y * BN;
    const int64_t nbits = args.nbits;
    const int64_t nw32 = ((nbits + 127) / 128) * 4;        // u32 words that may be read per row
    const int nstages = (int)((nbits + KBITS - 1) / KBITS);

    for (int r = tid; r < C::ROWS; r += NT) (r < BM ? popL[r] : popC[r - BM]) = 0;
    if (tid == 0) {
        for (int i = 0; i < C::NS; ++i) ptx::mbar_init(&empty_bar[i], 1);
        ptx::mbar_init(done_bar, 1);
        ptx::fence_mbar_init();
    }
    if (warp == 0) ptx::tmem_alloc<C::TMEM_COLS>(tmem_slot);
    ptx::tc_fence_before();
    __syncthreads();
    ptx::tc_fence_after();
    const uint32_t tmem_d = *tmem_slot;

    // ---- per-thread unit assignment: unit u -> (row = u % ROWS, half = u / ROWS)
    int urow[C::UNITS], uhalf[C::UNITS];
    bool uvalid[C::UNITS];
    const uint32_t *uptr[C::UNITS];
#pragma unroll
    for (int e = 0; e < C::UNITS; ++e) {
        const int u = tid + e * NT;
        uvalid[e] = u < C::ROWS * 2;
        const int row = u % C::ROWS;
        urow[e] = row;
        uhalf[e] = u / C::ROWS;
        const bool lane_side = row < BM;
        const int64_t g = lane_side ? l0 + row : c0 + (row - BM);
        const bool in = uvalid[e] && (lane_side ? g < args.nl : g < args.nc);
        uvalid[e] = in;
        uptr[e] = in ? (lane_side ? args.L + g * args.ldl32 : args.Cn + g * args.ldc32) : nullptr;
    }
    uint32_t upop[C::UNITS];
#pragma unroll
    for (int e = 0; e < C::UNITS; ++e) upop[e] = 0;

    auto load = [&](int s, uint4 (&r)[C::UNITS]) {
#pragma unroll
        for (int e = 0; e < C::UNITS; ++e) {
            const int64_t w = (int64_t)s * KW + 4 * uhalf[e];
            uint4 x = make_uint4(0, 0, 0, 0);
            if (uvalid[e] && s < nstages && w < nw32) {
                x = __ldg(reinterpret_cast<const uint4 *>(uptr[e] + w));
                if (w + 4 > nbits / 32) {
                    x.x &= word_mask(w, nbits); x.y &= word_mask(w + 1, nbits);
                    x.z &= word_mask(w + 2, nbits); x.w &= word_mask(w + 3, nbits);
                }
            }
            r[e] = x;
        }
    };

    auto expand_store = [&](int b, const uint4 (&r)[C::UNITS]) {
        uint8_t *sb = stage_base + (size_t)b * C::STAGE;
#pragma unroll
        for (int e = 0; e < C::UNITS; ++e) {
            if (tid + e * NT >= C::ROWS * 2) continue;
            const int row = urow[e];
            const bool lane_side = row < BM;
            const int R = lane_side ? BM : BN;
            const int rr = lane_side ? row : row - BM;
            uint8_t *base = sb + (lane_side ? 0 : C::A_BYTES) + rr * 16;
            const uint32_t wv[4] = {r[e].x, r[e].y, r[e].z, r[e].w};
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                const uint32_t x = wv[i];
                upop[e] += __popc(x);
                const int kstep = 4 * uhalf[e] + i;          // MMA K-step within the stage
                const uint32_t M = 0x01010101u;
                uint4 lo = make_uint4(x & M, (x >> 1) & M, (x >> 2) & M, (x >> 3) & M);
                uint4 hi = make_uint4((x >> 4) & M, (x >> 5) & M, (x >> 6) & M, (x >> 7) & M);
                *reinterpret_cast<uint4 *>(base + (size_t)(2 * kstep) * R * 16) = lo;
                *reinterpret_cast<uint4 *>(base + (size_t)(2 * kstep + 1) * R * 16) = hi;
            }
        }
    };

    constexpr uint32_t IDESC = ptx::idesc_u8_s32(BM, BN);
    auto issue = [&](int s, int b) {
        const uint32_t sa = ptx::smem_u32(stage_base + (size_t)b * C::STAGE);
        const uint32_t sbm = sa + C::A_BYTES;
#pragma unroll
        for (int k = 0; k < KW; ++k) {
            const uint64_t ad = ptx::smem_desc_kmajor_noswizzle(sa + 2 * k * BM * 16, BM * 16, 128);
            const uint64_t bd = ptx::smem_desc_kmajor_noswizzle(sbm + 2 * k * BN * 16, BN * 16, 128);
            ptx::mma_i8_ss(tmem_d, ad, bd, IDESC, (s | k) != 0 ? 1u : 0u);
        }
        ptx::mma_commit(&empty_bar[b]);
    };

    auto stage = [&](int s, const uint4 (&r)[C::UNITS]) {
        const int b = s % C::NS;
        if (s >= C::NS) ptx::mbar_wait(&empty_bar[b], (uint32_t)(((s / C::NS) - 1) & 1));
        expand_store(b, r);
        ptx::fence_proxy_async_smem();
        __syncthreads();
        if (tid == 0) {
            ptx::tc_fence_after();
            issue(s, b);
        }
    };

    uint4 r0[C::UNITS], r1[C::UNITS];
    load(0, r0);
    load(1, r1);
    for (int s = 0; s < nstages; s += 2) {
        stage(s, r0);
        load(s + 2, r0);
        if (s + 1 < nstages) {
            stage(s + 1, r1);
            load(s + 3, r1);
        }
    }
    if (tid == 0) ptx::mma_commit(done_bar);

    // popcounts of this tile's rows (masked words only)
#pragma unroll
    for (int e = 0; e < C::UNITS; ++e)
        if (tid + e * NT < C::ROWS * 2) {
            const int row = urow[e];
            atomicAdd(row < BM ? &popL[row] : &popC[row - BM], upop[e]);
        }
    ptx::mbar_wait(done_bar, 0);
    __syncthreads();
    ptx::tc_fence_after();

    // ---- epilogue: warp w reads TMEM lane quarter (w & 3), column half (w >> 2)
    const int q = warp & 3, half = warp >> 2;
    const int li = q * 32 + lane;                  // lane row within the tile
    const int64_t gl = l0 + li;
    const bool lvalid = gl < args.nl;
    const int64_t pl = popL[li];
    const int64_t n = nbits;
    for (int cb = half * (BN / 2); cb < (half + 1) * (BN / 2); cb += 8) {
        uint32_t v[8];
        ptx::tmem_ld8(tmem_d + ((uint32_t)(q * 32) << 16) + (uint32_t)cb, v);
        ptx::tmem_ld_wait();
        if (!lvalid) continue;
        if (EPI == EPI_COUNTS) {
            uint32_t res[8];
#pragma unroll
            for (int t = 0; t < 8; ++t) {
                const int64_t pc = popC[cb + t];
                const int64_t pq = args.swap ? pc : pl, pd = args.swap ? pl : pc;
                const int64_t c = (int64_t)v[t];
                int64_t x;
                switch (args.op) {
                case 0: x = c; break;
                case 1: x = pq + pd - 2 * c; break;
                case 2: x = pq - c; break;
                default: x = pd - c; break;
                }
                res[t] = (uint32_t)x;
            }
            if (args.swap) {
                // out[j][i]: j = column row (query), i = lane row (database) -> coalesced
#pragma unroll
                for (int t = 0; t < 8; ++t) {
                    const int64_t gc = c0 + cb + t;
                    if (gc < args.nc) {
                        uint32_t *p = args.C + gc * args.ldo + gl;
                        *p = args.accumulate ? *p + res[t] : res[t];
                    }
                }
            } else {
                const int64_t gc = c0 + cb;
                uint32_t *p = args.C + gl * args.ldo + gc;
                const bool vec = gc + 8 <= args.nc && (((uintptr_t)p & 15u) == 0);
                if (vec) {
                    if (args.accumulate) {
                        const uint4 o0 = reinterpret_cast<uint4 *>(p)[0], o1 = reinterpret_cast<uint4 *>(p)[1];
                        res[0] += o0.x; res[1] += o0.y; res[2] += o0.z; res[3] += o0.w;
                        res[4] += o1.x; res[5] += o1.y; res[6] += o1.z; res[7] += o1.w;
                    }
                    reinterpret_cast<uint4 *>(p)[0] = make_uint4(res[0], res[1], res[2], res[3]);
                    reinterpret_cast<uint4 *>(p)[1] = make_uint4(res[4], res[5], res[6], res[7]);
                } else {
#pragma unroll
                    for (int t = 0; t < 8; ++t)
                        if (gc + t < args.nc) p[t] = args.accumulate ? p[t] + res[t] : res[t];
                }
            }
        } else {
            float r2v[8], dpv[8];
#pragma unroll
            for (int t = 0; t < 8; ++t) {
                const int64_t pc = popC[cb + t];
                const int64_t pa = args.swap ? pc : pl, pb = args.swap ? pl : pc;
                ld_stats(n, pa, pb, (int64_t)v[t], r2v[t], dpv[t]);
            }
            if (args.swap) {
#pragma unroll
                for (int t = 0; t < 8; ++t) {
                    const int64_t gc = c0 + cb + t;
                    if (gc < args.nc) {
                        const int64_t o = gc * args.ldo + gl;
                        args.r2[o] = r2v[t];
                        if (args.dprime) args.dprime[o] = dpv[t];
                        if (args.C) args.C[o] = v[t];
                    }
                }
            } else {
                const int64_t gc = c0 + cb;
                const int64_t o = gl * args.ldo + gc;
                const bool vec = gc + 8 <= args.nc && ((o & 3) == 0);
                if (vec) {
                    float4 *pr = reinterpret_cast<float4 *>(args.r2 + o);
                    pr[0] = make_float4(r2v[0], r2v[1], r2v[2], r2v[3]);
                    pr[1] = make_float4(r2v[4], r2v[5], r2v[6], r2v[7]);
                    if (args.dprime) {
                        float4 *pd = reinterpret_cast<float4 *>(args.dprime + o);
                        pd[0] = make_float4(dpv[0], dpv[1], dpv[2], dpv[3]);
                        pd[1] = make_float4(dpv[4], dpv[5], dpv[6], dpv[7]);
                    }
                    if (args.C) {
                        uint4 *pc = reinterpret_cast<uint4 *>(args.C + o);
                        pc[0] = make_uint4(v[0], v[1], v[2], v[3]);
                        pc[1] = make_uint4(v[4], v[5], v[6], v[7]);
                    }
                } else {
#pragma unroll
                    for (int t = 0; t < 8; ++t)
                        if (gc + t < args.nc) {
                            args.r2[o + t] = r2v[t];
                            if (args.dprime) args.dprime[o + t] = dpv[t];
                            if (args.C) args.C[o + t] = v[t];
                        }
                }
            }
        }
    }

    ptx::tc_fence_before();
    __syncthreads();
    if (warp == 0) {
        ptx::tc_fence_after();
        ptx::tmem_dealloc<C::TMEM_COLS>(tmem_d);
    }
}

template <int BN, int EPI>
cudaError_t launch_cfg(const TcArgs &t, cudaStream_t s) {
    using C = Cfg<BN>;
    auto kern = bitgemm_tc_kernel<BN, EPI>;
    cudaError_t e = ensure_dyn_smem(reinterpret_cast<const void *>(kern), (int)C::SMEM);
    if (e != cudaSuccess) return e;
    const int64_t gx = (t.nl + BM - 1) / BM;
    const int64_t gy = (t.nc + BN - 1) / BN;
    if (gx > 0x7fffffffLL || gy > 65535) return cudaErrorInvalidConfiguration;
    kern<<<dim3((unsigned)gx, (unsigned)gy), NT, C::SMEM, s>>>(t);
    count_launches(1);
    return cudaGetLastError();
}

}  // namespace

size_t tc_workspace_bytes(int64_t, int64_t, int64_t) { return 0; }

bool tc_supported(int64_t m, int64_t n, int64_t nbits) {
    const int64_t small = m < n ? m : n;
    const int bn = small <= 64 ? 64 : (small <= 128 ? 128 : 256);
    const int64_t big = m < n ? n : m;
    return nbits >= 1 && nbits < (1LL << 31) && (small + bn - 1) / bn <= 65535 && big >= 1;
}

cudaError_t launch_bitgemm_tc(const GemmArgs &a, int epi, void *, size_t, cudaStream_t s) {
    TcArgs t{};
    const bool swap = a.m < a.n;     // larger operand on TMEM lanes
    t.L = swap ? a.B : a.A;
    t.Cn = swap ? a.A : a.B;
    t.nl = swap ? a.n : a.m;
    t.nc = swap ? a.m : a.n;
    t.ldl32 = swap ? a.ldb32 : a.lda32;
    t.ldc32 = swap ? a.lda32 : a.ldb32;
    t.nbits = a.nbits;
    t.swap = swap ? 1 : 0;
    t.op = a.op;
    t.accumulate = a.accumulate;
    t.ldo = a.ldc;
    t.C = a.C;
    t.r2 = a.r2;
    t.dprime = a.dprime;
    const int64_t small = t.nc;
    if (epi == EPI_LD) {
        if (small <= 64) return launch_cfg<64, EPI_LD>(t, s);
        if (small <= 128) return launch_cfg<128, EPI_LD>(t, s);
        return launch_cfg<256, EPI_LD>(t, s);
    }
    if (small <= 64) return launch_cfg<64, EPI_COUNTS>(t, s);
    if (small <= 128) return launch_cfg<128, EPI_COUNTS>(t, s);
    return launch_cfg<256, EPI_COUNTS>(t, s);
}

}  // namespace snp
