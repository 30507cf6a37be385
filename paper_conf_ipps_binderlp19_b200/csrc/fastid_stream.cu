// fastid_stream.cu — CUDA-core FastID for a handful of queries (nq <= 4) against a huge
// database: the skinny end of SURVEY §8a a3/a4 (configs[4] M = 1..4; single-profile queries
// are the common forensic case).
//
//   out[q][d] = sum_w POPC(Q[q][w] op D[d][w]),  op in {AND, XOR, ANDNOT, NOTAND}
//
// via the AND count and the popcount identities XOR = pQ + pD - 2 AND, ANDNOT = pQ - AND,
// NOTAND = pD - AND (Eqs. 1-3), plus the per-query best match
// ("no set bits ... positive match"; lowest index on ties, reading R4).
//
// Why CUDA cores here: with few queries the path is bound by streaming the database from
// HBM.  The POPC pipe (16 / clk / SM, measured: tools/alu_probe.cu) covers 16 x 32 = 512
// bit pairs per clock per SM against an HBM supply of ~180 database bits per clock per SM
// (6.55 TB/s / 148 SMs / 1.965 GHz), i.e. up to ~2.8 queries at the HBM rate (SURVEY App. A
// M*); the tcgen05 path is pinned at >= 45-50 cycles per M = 128, K = 64 MMA whatever N is
// (profiles/round2/mma_probe.txt) plus the on-chip e2m1 expansion, ~650 cycles per 128-row
// 512-bit stage measured — so for <= 4 queries this kernel is the faster one (a7 sweep).
//
// Design (one persistent CTA per SM): a TMA warp streams 256-row x 512-bit database stages
// (2-D tensor map, 64B swizzle) into a 4-deep shared-memory ring per CTA, two CTAs per SM
// (128 KB in flight per SM, and two sets of POPC dependency chains to interleave); 8
// compute warps each own 32 rows of every stage (lane = database row): 4 conflict-free
// LDS.128 for the row, the stage's query words as broadcast LDS.128, then per word and query
// one LOP3 (AND) + POPC + IADD.  At the end of a 256-row tile each lane turns its row's AND
// counts into every requested op, stores out[q][row] (coalesced: lane = consecutive rows)
// and keeps per-(op, query) running best matches (one redux.sync.min per pair and tile,
// key = count << 5 | lane); CTAs merge by 64-bit atomicMin on (count << 32 | row), the last
// warp of the grid writes (best_count, best_index).  Database popcounts are read when given
// (a resident database is prepared once), else counted from the streamed words.
#include "snp_internal.h"
#include "tc_ptx.cuh"
#include "e2m1.cuh"

namespace snp {

namespace {

constexpr int SBM = 256;                 // database rows per stage / tile
constexpr int SKW = 16;                  // 32-bit words per row per stage (512 bits)
#ifndef STREAM_NPR
#define STREAM_NPR 4
#endif
#ifndef STREAM_CTAS
#define STREAM_CTAS 2
#endif
constexpr int SNPR = STREAM_NPR;         // ring depth (16 KB stages)
constexpr int SCTAS = STREAM_CTAS;       // resident CTAs per SM (latency hiding for the POPC chains)
constexpr int NCW = 8;                   // compute warps (32 rows each)
constexpr int TMA_W = NCW;               // producer warp
constexpr int STHREADS = (NCW + 1) * 32;
constexpr int PST = SBM * SKW * 4;       // 16 KB per stage
constexpr int MAXOPS = 4;

struct StreamArgs {
    const uint32_t *Q;
    int64_t nq, ldq32;
    int64_t nd, nbits;
    int nst;
    int64_t ntiles;
    int nops;
    uint32_t cq[MAXOPS], cd[MAXOPS], cc[MAXOPS];
    uint32_t *outs[MAXOPS];
    int64_t ldo;
    int accumulate;
    int best_mask;
    unsigned long long *keys;
    unsigned int *done;
    uint32_t *best_count[MAXOPS];
    int64_t *best_index[MAXOPS];
    int64_t index_base;
    const uint32_t *popD;
};

template <int NQ>
__global__ void __launch_bounds__(STHREADS, SCTAS)
fastid_stream_kernel(const __grid_constant__ CUtensorMap tmD, const StreamArgs args) {
    extern __shared__ __align__(1024) uint8_t smem[];
    uint8_t *ring = smem;                                                     // [SNPR][PST]
    const int qw = args.nst * SKW;                                            // query words per row
    uint32_t *qs = reinterpret_cast<uint32_t *>(ring + SNPR * PST);           // [NQ][qw]
    uint64_t *pfull = reinterpret_cast<uint64_t *>(qs + NQ * qw);             // [SNPR]
    uint64_t *pempty = pfull + SNPR;                                          // [SNPR]
    uint32_t *popq = reinterpret_cast<uint32_t *>(pempty + SNPR);             // [NQ]

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int64_t nbits = args.nbits;
    const int nst = args.nst;
    const int64_t my_tiles = args.ntiles > blockIdx.x ? (args.ntiles - 1 - blockIdx.x) / gridDim.x + 1 : 0;
    if (tid == 0) {
        for (int i = 0; i < SNPR; ++i) {
            ptx::mbar_init(&pfull[i], 1);
            ptx::mbar_init(&pempty[i], NCW);
        }
        ptx::fence_mbar_init();
    }
    if (tid < NQ) popq[tid] = 0;
    if (warp == TMA_W && lane == 0) ptx::prefetch_tensormap(&tmD);
    __syncthreads();
    // programmatic dependent launch: everything above overlapped the previous kernel (the
    // key-init kernel / the caller's query packing); global data is read only after this
    asm volatile("griddepcontrol.wait;" ::: "memory");

    // ---- prologue: the queries (masked to nbits, zero rows past nq) and their popcounts
    {
        uint32_t pc[NQ];
#pragma unroll
        for (int j = 0; j < NQ; ++j) pc[j] = 0;
        for (int w = tid; w < qw; w += STHREADS) {
            const uint32_t m = word_mask(w, nbits);
#pragma unroll
            for (int j = 0; j < NQ; ++j) {
                const uint32_t x = (j < args.nq && m) ? __ldg(args.Q + j * args.ldq32 + w) & m : 0u;
                qs[j * qw + w] = x;
                pc[j] += __popc(x);
            }
        }
#pragma unroll
        for (int j = 0; j < NQ; ++j) {
#pragma unroll
            for (int o = 16; o; o >>= 1) pc[j] += __shfl_xor_sync(0xffffffffu, pc[j], o);
            if (lane == 0 && pc[j]) atomicAdd(&popq[j], pc[j]);
        }
    }
    __syncthreads();

    if (warp == TMA_W) {
        // ------------------------------------------------------------ TMA producer
        if (lane == 0) {
            int p = 0;
            uint32_t round = 0;
            for (int64_t tl = 0; tl < my_tiles; ++tl) {
                const int32_t row0 = (int32_t)((blockIdx.x + tl * gridDim.x) * SBM);
                for (int s = 0; s < nst; ++s) {
                    if (round > 0) ptx::mbar_wait(&pempty[p], (round - 1) & 1);
                    ptx::mbar_arrive_expect_tx(&pfull[p], PST);
                    ptx::tma_load_2d(ring + p * PST, &tmD, &pfull[p], s * SKW, row0);
                    if (++p == SNPR) { p = 0; ++round; }
                }
            }
        }
    } else {
        // ------------------------------------------------------------ compute warps
        const int r = warp * 32 + lane;           // row of the stage / tile
        const int sw = (r >> 1) & 3;              // TMA 64B swizzle of a 64-byte row
        const bool pre = args.popD != nullptr;
        const int64_t full32 = nbits / 32;
        uint32_t bc = 0xffffffffu, bi = 0xffffffffu;   // running best of pair `lane` (op j, query q)
        int p = 0;
        uint32_t round = 0;
        for (int64_t tl = 0; tl < my_tiles; ++tl) {
            const int64_t t = blockIdx.x + tl * gridDim.x;
            const int64_t g = t * SBM + r;       // this lane's database row
            uint32_t acc[NQ];
#pragma unroll
            for (int j = 0; j < NQ; ++j) acc[j] = 0;
            uint32_t pdv = 0;
            for (int s = 0; s < nst; ++s) {
                ptx::mbar_wait_warp(&pfull[p], round & 1);
                const uint8_t *src = ring + p * PST + r * (SKW * 4);
                uint32_t d[SKW];
#pragma unroll
                for (int c = 0; c < SKW / 4; ++c) {
                    const uint4 x = *reinterpret_cast<const uint4 *>(src + ((c ^ sw) << 4));
                    d[4 * c] = x.x; d[4 * c + 1] = x.y; d[4 * c + 2] = x.z; d[4 * c + 3] = x.w;
                }
                __syncwarp();
                if (lane == 0) ptx::mbar_arrive(&pempty[p]);   // the row words are in registers
                const int64_t w0 = (int64_t)s * SKW;
                if (w0 + SKW > full32) {
#pragma unroll
                    for (int i = 0; i < SKW; ++i) d[i] &= word_mask(w0 + i, nbits);
                }
                if (!pre) {
#pragma unroll
                    for (int i = 0; i < SKW; ++i) pdv += __popc(d[i]);
                }
#pragma unroll
                for (int j = 0; j < NQ; ++j) {
                    const uint4 *qv = reinterpret_cast<const uint4 *>(qs + j * qw + w0);   // broadcast
#pragma unroll
                    for (int c = 0; c < SKW / 4; ++c) {
                        const uint4 q = qv[c];
                        acc[j] += __popc(d[4 * c] & q.x) + __popc(d[4 * c + 1] & q.y);
                        acc[j] += __popc(d[4 * c + 2] & q.z) + __popc(d[4 * c + 3] & q.w);
                    }
                }
                if (++p == SNPR) { p = 0; ++round; }
            }
            // ---- tile epilogue: ops from the AND counts, stores, best matches
            const bool valid = g < args.nd;
            const uint32_t pd = pre ? (valid ? __ldg(args.popD + g) : 0u) : pdv;
            const uint32_t laneterm = valid ? (uint32_t)lane : 0xF0000000u;   // invalid rows never win
#pragma unroll
            for (int j = 0; j < MAXOPS; ++j) {
                if (j >= args.nops) break;
                uint32_t *out = args.outs[j];
#pragma unroll
                for (int q = 0; q < NQ; ++q) {
                    if (q >= args.nq) break;
                    const uint32_t x = args.cq[j] * popq[q] + args.cd[j] * pd + args.cc[j] * acc[q];
                    if (out && valid) {
                        uint32_t *o = out + (int64_t)q * args.ldo + g;
                        if (args.accumulate) *o += x;
                        else __stcs(o, x);
                    }
                    if ((args.best_mask >> j) & 1) {
                        const uint32_t m = __reduce_min_sync(0xffffffffu, (x << 5) + laneterm);
                        // tiles arrive in increasing row order per warp: strict < keeps the lowest row
                        if (lane == j * NQ + q && m < 0xF0000000u && (m >> 5) < bc) {
                            bc = m >> 5;
                            bi = (uint32_t)(t * SBM + warp * 32) + (m & 31u);
                        }
                    }
                }
            }
        }
        if (args.best_mask) {
            const int j = lane / NQ, q = lane % NQ;
            if (j < args.nops && q < args.nq && ((args.best_mask >> j) & 1) && bc != 0xffffffffu)
                atomicMax(args.keys + (int64_t)j * args.nq + q, ~(((unsigned long long)bc << 32) | bi));   // complemented keys
            __threadfence();
            uint32_t last = 0;
            if (lane == 0) last = atomicAdd(args.done, 1u) == gridDim.x * NCW - 1 ? 1u : 0u;
            if (__shfl_sync(0xffffffffu, last, 0)) {
                __threadfence();
                for (int jj = 0; jj < args.nops; ++jj) {
                    if (!((args.best_mask >> jj) & 1)) continue;
                    for (int i = lane; i < args.nq; i += 32) {
                        const unsigned long long k = ~__ldcg(args.keys + jj * args.nq + i);
                        args.best_count[jj][i] = k == ~0ULL ? 0xffffffffu : (uint32_t)(k >> 32);
                        args.best_index[jj][i] = k == ~0ULL ? -1 : (int64_t)(k & 0xffffffffULL) + args.index_base;
                        args.keys[jj * args.nq + i] = 0ULL;   // the workspace is left zero-filled
                    }
                }
                if (lane == 0) *args.done = 0u;
            }
        }
    }
}


size_t stream_smem(int nq_t, int64_t nbits) {
    const int64_t nst = (nbits + SKW * 32 - 1) / (SKW * 32);
    return (size_t)SNPR * PST + (size_t)nq_t * nst * SKW * 4 + 2 * SNPR * 8 + 64;
}

void stream_coefs(int op, uint32_t &cq, uint32_t &cd, uint32_t &cc) {
    switch (op) {   // x = cq pQ + cd pD + cc AND (uint32 wrap-around)
    case 0: cq = 0; cd = 0; cc = 1; break;                   // AND      Eq. (1)
    case 1: cq = 1; cd = 1; cc = (uint32_t)-2; break;        // XOR      Eq. (2)
    case 2: cq = 1; cd = 0; cc = (uint32_t)-1; break;        // ANDNOT   Eq. (3), r = query
    default: cq = 0; cd = 1; cc = (uint32_t)-1; break;       // NOTAND   Eq. (3), r = DB row
    }
}

}  // namespace

constexpr size_t STREAM_MAX_SMEM = 232448 - 1024;

bool fastid_stream_supported(int64_t nq, int64_t nd, int64_t nbits) {
    // counts < 2^27 keep the 32-bit (count << 5 | lane) reduction key exact
    if (nq < 1 || nq > 4 || nd < 1 || nd > (int64_t)0x7fffffff - SBM || nbits < 1 || nbits >= (1LL << 27))
        return false;
    return stream_smem(nq <= 1 ? 1 : nq <= 2 ? 2 : 4, nbits) <= STREAM_MAX_SMEM;   // resident query words
}

size_t fastid_stream_ws_bytes(int64_t nq, int nops) { return (((size_t)nops * nq * 8 + 255) & ~(size_t)255) + 256; }

cudaError_t launch_fastid_stream(const SearchArgs &a, cudaStream_t s) {
    StreamArgs f{};
    f.Q = a.Q; f.nq = a.nq; f.ldq32 = a.ldq32;
    f.nd = a.nd; f.nbits = a.nbits;
    f.nst = (int)((a.nbits + SKW * 32 - 1) / (SKW * 32));
    f.ntiles = (a.nd + SBM - 1) / SBM;
    f.nops = a.nops;
    f.ldo = a.ldo;
    f.accumulate = a.accumulate;
    f.popD = a.popD;
    for (int j = 0; j < a.nops; ++j) {
        stream_coefs(a.ops[j], f.cq[j], f.cd[j], f.cc[j]);
        f.outs[j] = a.counts[j];
        if (a.best_count[j]) {
            f.best_mask |= 1 << j;
            f.best_count[j] = a.best_count[j];
            f.best_index[j] = a.best_index[j];
        }
    }
    if (f.best_mask && a.accumulate) return cudaErrorInvalidValue;
    f.keys = a.keys;
    f.done = a.done;
    f.index_base = a.index_base;
    CUtensorMap tm;
    if (!make_map_u32_2d(&tm, a.D, a.nd, a.ldd32, SKW, SBM, CU_TENSOR_MAP_SWIZZLE_64B)) return cudaErrorInvalidValue;
    const int nqt = a.nq <= 1 ? 1 : a.nq <= 2 ? 2 : a.nq <= 3 ? 3 : 4;
    const size_t smem = stream_smem(nqt, a.nbits);
    using KernFn = void (*)(const CUtensorMap, const StreamArgs);
    KernFn kern = nqt == 1 ? fastid_stream_kernel<1> : nqt == 2 ? fastid_stream_kernel<2>
                : nqt == 3 ? fastid_stream_kernel<3> : fastid_stream_kernel<4>;
    if (cudaError_t e = ensure_dyn_smem(reinterpret_cast<const void *>(kern), (int)STREAM_MAX_SMEM); e != cudaSuccess)
        return e;
    const int64_t slots = (int64_t)device_sms() * (smem * SCTAS <= 232448 - 2048 ? SCTAS : 1);
    const int grid = (int)(f.ntiles < slots ? f.ntiles : slots);
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3((unsigned)STHREADS);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    cudaError_t le = cudaLaunchKernelEx(&cfg, kern, tm, f);
    count_launches(1);
    if (le != cudaSuccess) return le;
    return cudaGetLastError();
}

}  // namespace snp
