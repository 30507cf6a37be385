// bitgemm_tc4.cu — tensor-core bit-GEMM on 4-bit expanded operands (tcgen05.mma kind::mxf4).
//
//   C[i][j] = sum_k A_ik & B_jk      (Eq. 1; the GEMM form of P:L116)
//
// Every bit becomes one e2m1 element: 1 -> 1.0 (0b0010), 0 -> 0.0, with all block
// scale factors 2^0 (ue8m0 0x7F).  A product is then exactly a_k * b_k in {0, 1} and
// the fp32 TMEM accumulator holds the exact integer count for K < 2^24 (DESIGN.md §5:
// integers below 2^24 are exact in fp32; tested bit-exact against the oracle).
// kind::mxf4 runs at twice the int8 rate and needs half the expanded bytes of the
// i8 variant (bitgemm_tc.cu), which is what bounds this kernel: expansion ALU work
// and shared-memory traffic.
//
// Structure (one persistent CTA per SM, warp-specialised, 13 warps):
//   warps 0-7  expanders: 128-bit loads of the packed 256-bit K-slice of every row of
//              the tile (prefetched 4 stages ahead in registers), popcounts, expansion
//              (w << 1 / w / w >> 1 / w >> 2) & 0x22222222 -> four words of 8 nibbles:
//                lane-side rows (A)  -> TMEM with tcgen05.st (MMA operand A from TMEM)
//                column-side rows (B) -> shared memory, K-major no-swizzle UMMA layout
//              then arrive on full[stage].
//   warp 8     TMEM allocator + MMA issuer: per stage 4 x tcgen05.mma (M=128, N=BN,
//              K=64) into one of two TMEM accumulators; commit -> empty[stage]; commit
//              after the tile's last stage -> acc_full[acc].
//   warps 9-12 epilogue: tcgen05.ld of the finished accumulator (while the MMA warp
//              already fills the other one), popcount identities / LD statistics,
//              global stores; arrive acc_empty[acc].
// The 32 bits of a packed word are permuted inside the word (nibble n of output t
// holds bit 4n + t); the same permutation is applied to both operands, so every dot
// product is unchanged.
#include "snp_internal.h"
#include "tc_ptx.cuh"

namespace snp {
namespace {

constexpr int BM = 128;            // MMA M = TMEM lanes (lane-side rows per tile)
constexpr int KBITS = 256;         // bits per pipeline stage
static_assert(KBITS == 256, "a stage is exactly the 4 K=64 MMAs of mma4_mxf4_ts_commit");
constexpr int NS = 4;              // pipeline stages
constexpr int PF = 4;              // register prefetch depth (stages)
constexpr int NEXP = 8;            // expander warps
constexpr int MMA_WARP = 8;
constexpr int EPI_WARP0 = 9;       // epilogue warps 9..12 (quarters 1,2,3,0)
constexpr int NTHREADS = 13 * 32;

template <int BN>
struct Cfg4 {
    static constexpr int B_STAGE = BN * (KBITS / 2);          // bytes of expanded B per stage
    static constexpr int ACC_COLS = BN;                       // fp32 accumulator columns
    static constexpr int A_COL0 = 2 * ACC_COLS;               // A stage s at A_COL0 + 32 s
    static constexpr int SF_COL = A_COL0 + NS * 32;           // SFA at SF_COL, SFB at SF_COL + 16
    static constexpr int TMEM_COLS = 512;
    static_assert(SF_COL + 32 <= TMEM_COLS, "TMEM budget");
    static constexpr size_t SMEM = (size_t)NS * B_STAGE + 8192;   // + barriers, tmem slot, popcounts
};

struct Tc4Args {
    const uint32_t *L;   // lane-side operand (packed rows, u32 view)
    const uint32_t *Cn;  // column-side operand
    int64_t nl, nc;
    int64_t ldl32, ldc32;
    int64_t nbits;
    int swap;            // 1: user (i, j) = (column row, lane row)
    int op;
    int accumulate;
    int64_t ldo;
    uint32_t *C;
    float *r2;
    float *dprime;
    int64_t nlb, ncb;    // lane / column blocks
    int nstages;         // stages per tile
};

__device__ __forceinline__ uint32_t word_mask(int64_t w, int64_t nbits) {
    const int64_t lo = w * 32;
    if (lo + 32 <= nbits) return 0xffffffffu;
    if (lo >= nbits) return 0u;
    return (1u << (uint32_t)(nbits - lo)) - 1u;
}

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

// Block-scaled instruction descriptor: A = B = e2m1 (MXF4 format 1), ue8m0 scales,
// K-major, dense K = 64, M = 128.
__host__ __device__ constexpr uint32_t idesc_mxf4(int M, int N) {
    return (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | (1u << 23) | ((uint32_t)(M >> 4) << 24);
}


__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t (&v)[16]) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(
            taddr),
        "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "r"(v[8]),
        "r"(v[9]), "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15])
        : "memory");
}

// packed word -> 4 words of 8 e2m1 nibbles (value 1.0 = 0b0010 where the bit is set)
__device__ __forceinline__ void expand4(uint32_t x, uint32_t &o0, uint32_t &o1, uint32_t &o2, uint32_t &o3) {
    const uint32_t M = 0x22222222u;
    o0 = (x << 1) & M;   // bits 0,4,8,...
    o1 = x & M;          // bits 1,5,9,...
    o2 = (x >> 1) & M;   // bits 2,6,10,...
    o3 = (x >> 2) & M;   // bits 3,7,11,...
}

template <int BN, int EPI>
__global__ void __launch_bounds__(NTHREADS, 1) bitgemm_tc4_kernel(const Tc4Args args) {
    using C = Cfg4<BN>;
    extern __shared__ __align__(1024) uint8_t smem[];
    uint8_t *bstage = smem;                                                    // [NS][B_STAGE]
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem + (size_t)NS * C::B_STAGE);
    uint64_t *full_bar = bars;               // [NS]   expanders -> MMA
    uint64_t *empty_bar = bars + NS;         // [NS]   MMA commit -> expanders
    uint64_t *accf_bar = bars + 2 * NS;      // [2]    MMA commit -> epilogue
    uint64_t *acce_bar = bars + 2 * NS + 2;  // [2]    epilogue -> MMA / expanders (pops)
    uint64_t *popf_bar = bars + 2 * NS + 4;  // [2]    expanders -> epilogue (pops written)
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(bars + 2 * NS + 6);
    uint32_t *popA = tmem_slot + 4;          // [2 acc][2 half][BM]
    uint32_t *popB = popA + 2 * 2 * BM;      // [2 acc][2 half][BN]

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int64_t nbits = args.nbits;
    const int nst = args.nstages;
    const int64_t ntiles = args.nlb * args.ncb;
    const int64_t my_tiles = ntiles > blockIdx.x ? (ntiles - 1 - blockIdx.x) / gridDim.x + 1 : 0;
    const int64_t total_it = my_tiles * nst;
    const int64_t nw32 = ((nbits + 127) / 128) * 4;

    if (tid == 0) {
        for (int i = 0; i < NS; ++i) {
            ptx::mbar_init(&full_bar[i], NEXP);
            ptx::mbar_init(&empty_bar[i], 1);
        }
        for (int i = 0; i < 2; ++i) {
            ptx::mbar_init(&accf_bar[i], 1);
            ptx::mbar_init(&acce_bar[i], 4);
            ptx::mbar_init(&popf_bar[i], NEXP);
        }
        ptx::fence_mbar_init();
    }
    if (warp == MMA_WARP) ptx::tmem_alloc<C::TMEM_COLS>(tmem_slot);
    ptx::tc_fence_before();
    __syncthreads();
    ptx::tc_fence_after();
    const uint32_t tmem = *tmem_slot;

    if (warp >= EPI_WARP0) {
        // scale factors: every byte 0x7F (ue8m0 2^0) in the SFA/SFB columns of all lanes
        const int q = warp & 3;
        uint32_t v[16];
#pragma unroll
        for (int i = 0; i < 16; ++i) v[i] = 0x7F7F7F7Fu;
        tmem_st16(tmem + ((uint32_t)(q * 32) << 16) + C::SF_COL, v);
        tmem_st16(tmem + ((uint32_t)(q * 32) << 16) + C::SF_COL + 16, v);
        ptx::tmem_st_wait();
    }
    ptx::tc_fence_before();
    __syncthreads();
    ptx::tc_fence_after();

    if (warp < NEXP) {
        // ------------------------------------------------------------ expanders
        const int qa = warp & 3, ha = warp >> 2;          // A unit: row 32 qa + lane, words 4 ha..
        const int arow = qa * 32 + lane;
        const bool has_b = tid < 2 * BN;
        const int brow = tid % BN, hb = tid / BN;          // B unit (if has_b)
        const int64_t full32 = nbits / 32;                 // words with no tail bits
        uint32_t popa = 0, popb = 0;

        // load cursor (runs PF iterations ahead of the consume cursor); one division
        // per tile, none per stage
        int64_t l_tl = 0;
        int l_s = 0;
        const uint32_t *la = nullptr, *lbp = nullptr;
        auto set_load_tile = [&]() {
            la = lbp = nullptr;
            if (l_tl >= my_tiles) return;
            const int64_t t = blockIdx.x + l_tl * gridDim.x;
            const int64_t lb = t % args.nlb, cb = t / args.nlb;
            const int64_t ga = lb * BM + arow;
            if (ga < args.nl) la = args.L + ga * args.ldl32 + 4 * ha;
            const int64_t gb = cb * BN + brow;
            if (has_b && gb < args.nc) lbp = args.Cn + gb * args.ldc32 + 4 * hb;
        };
        auto masked = [&](uint4 x, int64_t w) {
            if (w + 4 > full32) {
                x.x &= word_mask(w, nbits); x.y &= word_mask(w + 1, nbits);
                x.z &= word_mask(w + 2, nbits); x.w &= word_mask(w + 3, nbits);
            }
            return x;
        };
        auto load_next = [&](uint4 &ra, uint4 &rb) {
            ra = make_uint4(0, 0, 0, 0);
            rb = make_uint4(0, 0, 0, 0);
            if (l_tl >= my_tiles) return;
            const int w = l_s * (KBITS / 32);
            const int64_t wa = w + 4 * ha, wb = w + 4 * hb;
            if (la && wa < nw32) ra = masked(__ldg(reinterpret_cast<const uint4 *>(la + w)), wa);
            if (lbp && wb < nw32) rb = masked(__ldg(reinterpret_cast<const uint4 *>(lbp + w)), wb);
            if (++l_s == nst) {
                l_s = 0;
                ++l_tl;
                set_load_tile();
            }
        };

        int64_t c_tl = 0;   // consume cursor
        int c_s = 0;
        auto step = [&](int b, uint32_t use, uint4 &ra, uint4 &rb) {
            if (use > 0) ptx::mbar_wait(&empty_bar[b], (use - 1) & 1);
            // A -> TMEM columns A_COL0 + 32 b + 16 ha (two K-steps of 8 columns)
            {
                uint32_t v[16];
                const uint32_t wv[4] = {ra.x, ra.y, ra.z, ra.w};
#pragma unroll
                for (int i = 0; i < 4; ++i) {
                    popa += __popc(wv[i]);
                    expand4(wv[i], v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
                }
                tmem_st16(tmem + ((uint32_t)(qa * 32) << 16) + (uint32_t)(C::A_COL0 + 32 * b + 16 * ha), v);
            }
            if (has_b) {
                uint8_t *base = bstage + (size_t)b * C::B_STAGE + brow * 16;
                const uint32_t wv[4] = {rb.x, rb.y, rb.z, rb.w};
#pragma unroll
                for (int i = 0; i < 4; ++i) {
                    popb += __popc(wv[i]);
                    uint4 o;
                    expand4(wv[i], o.x, o.y, o.z, o.w);
                    *reinterpret_cast<uint4 *>(base + (4 * hb + i) * BN * 16) = o;   // chunk = word
                }
            }
            ptx::tmem_st_wait();
            ptx::fence_proxy_async_smem();
            ptx::tc_fence_before();
            __syncwarp();
            if (lane == 0) ptx::mbar_arrive(&full_bar[b]);
            if (++c_s == nst) {
                // tile finished: publish this thread's popcount partials
                c_s = 0;
                const int acc = (int)(c_tl & 1);
                if (c_tl >= 2) ptx::mbar_wait(&acce_bar[acc], (uint32_t)(((c_tl >> 1) - 1) & 1));
                popA[(acc * 2 + ha) * BM + arow] = popa;
                if (has_b) popB[(acc * 2 + hb) * BN + brow] = popb;
                popa = popb = 0;
                __syncwarp();
                if (lane == 0) ptx::mbar_arrive(&popf_bar[acc]);
                ++c_tl;
            }
            load_next(ra, rb);
        };

        set_load_tile();
        uint4 a0, b0, a1, b1, a2, b2, a3, b3;
        load_next(a0, b0);
        load_next(a1, b1);
        load_next(a2, b2);
        load_next(a3, b3);
        static_assert(NS == 4 && PF == 4, "stage index == register set index");
        for (int64_t it = 0; it < total_it; it += 4) {
            const uint32_t use = (uint32_t)(it >> 2);
            step(0, use, a0, b0);
            if (it + 1 < total_it) step(1, use, a1, b1);
            if (it + 2 < total_it) step(2, use, a2, b2);
            if (it + 3 < total_it) step(3, use, a3, b3);
        }
    } else if (warp == MMA_WARP) {
        // ------------------------------------------------------------ MMA issuer
        // whole warp converged; one elected lane issues a stage's 4 MMAs + commit
        constexpr uint32_t IDESC = idesc_mxf4(BM, BN);
        const uint32_t sfa = tmem + C::SF_COL, sfb = tmem + C::SF_COL + 16;
        const uint64_t bdesc0 = ptx::smem_desc_kmajor_noswizzle(ptx::smem_u32(bstage), BN * 16, 128);
        constexpr uint32_t BSTEP = (2 * BN * 16) >> 4;
        int b = 0;
        uint32_t bround = 0;
        for (int64_t tl = 0; tl < my_tiles; ++tl) {
            const int acc = (int)(tl & 1);
            if (tl >= 2) ptx::mbar_wait(&acce_bar[acc], (uint32_t)(((tl >> 1) - 1) & 1));
            ptx::tc_fence_after();
            const uint32_t d = tmem + (uint32_t)(acc * C::ACC_COLS);
            for (int s = 0; s < nst; ++s) {
                ptx::mbar_wait(&full_bar[b], bround & 1);
                ptx::tc_fence_after();
                ptx::mma4_mxf4_ts_commit(d, tmem + (uint32_t)(C::A_COL0 + 32 * b),
                                         bdesc0 + (uint64_t)((b * C::B_STAGE) >> 4), BSTEP, IDESC,
                                         s != 0 ? 1u : 0u, sfa, sfb, &empty_bar[b]);
                if (++b == NS) { b = 0; ++bround; }
            }
            ptx::mma_commit_elect(&accf_bar[acc]);
        }
        __syncwarp();
    } else {
        // ------------------------------------------------------------ epilogue
        const int q = warp & 3;
        const int li = q * 32 + lane;
        const int64_t n = nbits;
        for (int64_t tl = 0; tl < my_tiles; ++tl) {
            const int acc = (int)(tl & 1);
            const uint32_t ph = (uint32_t)((tl >> 1) & 1);
            const int64_t t = blockIdx.x + tl * gridDim.x;
            const int64_t lb = t % args.nlb, cb = t / args.nlb;
            ptx::mbar_wait(&popf_bar[acc], ph);
            ptx::mbar_wait(&accf_bar[acc], ph);
            ptx::tc_fence_after();
            const int64_t gl = lb * BM + li;
            const bool lvalid = gl < args.nl;
            const int64_t pl = (int64_t)popA[(acc * 2) * BM + li] + popA[(acc * 2 + 1) * BM + li];
            const uint32_t *pb0 = popB + (acc * 2) * BN, *pb1 = popB + (acc * 2 + 1) * BN;
            for (int cbk = 0; cbk < BN; cbk += 8) {
                uint32_t v[8];
                ptx::tmem_ld8(tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(acc * C::ACC_COLS + cbk), v);
                ptx::tmem_ld_wait();
                if (!lvalid) continue;
                uint32_t cnt[8];
#pragma unroll
                for (int u = 0; u < 8; ++u) cnt[u] = __float2uint_rn(__uint_as_float(v[u]));
                const int64_t gc0 = cb * BN + cbk;
                if (EPI == EPI_COUNTS) {
                    uint32_t res[8];
#pragma unroll
                    for (int u = 0; u < 8; ++u) {
                        const int64_t pc = (int64_t)pb0[cbk + u] + pb1[cbk + u];
                        const int64_t pq = args.swap ? pc : pl, pd = args.swap ? pl : pc;
                        const int64_t c = cnt[u];
                        int64_t x;
                        switch (args.op) {
                        case 0: x = c; break;
                        case 1: x = pq + pd - 2 * c; break;
                        case 2: x = pq - c; break;
                        default: x = pd - c; break;
                        }
                        res[u] = (uint32_t)x;
                    }
                    if (args.swap) {
#pragma unroll
                        for (int u = 0; u < 8; ++u) {
                            const int64_t gc = gc0 + u;
                            if (gc < args.nc) {
                                uint32_t *p = args.C + gc * args.ldo + gl;
                                *p = args.accumulate ? *p + res[u] : res[u];
                            }
                        }
                    } else {
                        uint32_t *p = args.C + gl * args.ldo + gc0;
                        const bool vec = gc0 + 8 <= args.nc && (((uintptr_t)p & 15u) == 0);
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
                            for (int u = 0; u < 8; ++u)
                                if (gc0 + u < args.nc) p[u] = args.accumulate ? p[u] + res[u] : res[u];
                        }
                    }
                } else {
                    float r2v[8], dpv[8];
#pragma unroll
                    for (int u = 0; u < 8; ++u) {
                        const int64_t pc = (int64_t)pb0[cbk + u] + pb1[cbk + u];
                        const int64_t pa = args.swap ? pc : pl, pbb = args.swap ? pl : pc;
                        ld_stats(n, pa, pbb, (int64_t)cnt[u], r2v[u], dpv[u]);
                    }
                    if (args.swap) {
#pragma unroll
                        for (int u = 0; u < 8; ++u) {
                            const int64_t gc = gc0 + u;
                            if (gc < args.nc) {
                                const int64_t o = gc * args.ldo + gl;
                                args.r2[o] = r2v[u];
                                if (args.dprime) args.dprime[o] = dpv[u];
                                if (args.C) args.C[o] = cnt[u];
                            }
                        }
                    } else {
                        const int64_t o = gl * args.ldo + gc0;
                        const bool vec = gc0 + 8 <= args.nc && ((o & 3) == 0);
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
                                pc[0] = make_uint4(cnt[0], cnt[1], cnt[2], cnt[3]);
                                pc[1] = make_uint4(cnt[4], cnt[5], cnt[6], cnt[7]);
                            }
                        } else {
#pragma unroll
                            for (int u = 0; u < 8; ++u)
                                if (gc0 + u < args.nc) {
                                    args.r2[o + u] = r2v[u];
                                    if (args.dprime) args.dprime[o + u] = dpv[u];
                                    if (args.C) args.C[o + u] = cnt[u];
                                }
                        }
                    }
                }
            }
            ptx::tc_fence_before();
            __syncwarp();
            if (lane == 0) ptx::mbar_arrive(&acce_bar[acc]);
        }
    }

    ptx::tc_fence_before();
    __syncthreads();
    if (warp == MMA_WARP) {
        ptx::tc_fence_after();
        ptx::tmem_dealloc<C::TMEM_COLS>(tmem);
    }
}

int g_num_sms = 0;

template <int BN, int EPI>
cudaError_t launch_cfg4(Tc4Args t, cudaStream_t s) {
    using C = Cfg4<BN>;
    auto kern = bitgemm_tc4_kernel<BN, EPI>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)C::SMEM);
    if (e != cudaSuccess) return e;
    if (g_num_sms == 0) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&g_num_sms, cudaDevAttrMultiProcessorCount, dev);
        if (g_num_sms <= 0) g_num_sms = 148;
    }
    t.nlb = (t.nl + BM - 1) / BM;
    t.ncb = (t.nc + BN - 1) / BN;
    t.nstages = (int)((t.nbits + KBITS - 1) / KBITS);
    const int64_t ntiles = t.nlb * t.ncb;
    const int grid = (int)(ntiles < g_num_sms ? ntiles : g_num_sms);
    kern<<<grid, NTHREADS, C::SMEM, s>>>(t);
    count_launches(1);
    return cudaGetLastError();
}

}  // namespace

bool tc4_supported(int64_t m, int64_t n, int64_t nbits) {
    return m >= 1 && n >= 1 && nbits >= 1 && nbits < (1LL << 24);
}

cudaError_t launch_bitgemm_tc4(const GemmArgs &a, int epi, cudaStream_t s) {
    Tc4Args t{};
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
    if (t.nc <= 64) return epi == EPI_LD ? launch_cfg4<64, EPI_LD>(t, s) : launch_cfg4<64, EPI_COUNTS>(t, s);
    return epi == EPI_LD ? launch_cfg4<128, EPI_LD>(t, s) : launch_cfg4<128, EPI_COUNTS>(t, s);
}

}  // namespace snp
