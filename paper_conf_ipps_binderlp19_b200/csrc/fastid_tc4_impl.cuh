// fastid_tc4.cu — FastID-shaped tensor-core bit-GEMM: a small query batch (<= 128
// profiles) against a huge database streamed from HBM.
//
//   out[q][d] = sum_k op(Q_qk, D_dk),  op in {AND, XOR, ANDNOT, NOTAND}  (Eqs. 1-3,
//   P:L52-78), via the AND count and the popcount identities of SURVEY §8a a4.
//
// For a few queries the path is bound by streaming the database, so this kernel is
// built around the database stream:
//   * the query batch is expanded ONCE per CTA into shared memory (e2m1 nibbles, K-major
//     no-swizzle UMMA layout, the whole K range) and stays resident — it is the MMA B
//     operand for every database tile;
//   * database tiles (128 rows) are streamed by TMA (2-D tensor map, 128 rows x 256 bits
//     per stage) into a 16-deep shared-memory ring: up to 64 KB in flight per SM without
//     spending registers;
//   * 8 expander warps turn each stage into e2m1 nibbles and write them straight into
//     TMEM (tcgen05.st) as the MMA A operand, accumulating database-row popcounts;
//   * one thread issues tcgen05.mma kind::mxf4 (M = 128 database rows, N = queries,
//     K = 64) from TMEM-A x SMEM-B into one of two TMEM accumulators;
//   * 4 epilogue warps apply the popcount identity and write out[q][d] coalesced along d
//     while the next tile is being multiplied.
// Exactness: products are in {0, 1}, fp32 sums of them are exact below 2^24.
// This file is compiled twice (fastid_tc4_k512.cu, fastid_tc4_k1024.cu) with different
// stage sizes; FASTID_FN(name) gives each instantiation's entry points a distinct name and
// fastid_tc4.cu dispatches between them per shape.
#include "snp_internal.h"
#include "tc_ptx.cuh"
#include "e2m1.cuh"
#ifndef FASTID_FN
#define FASTID_FN(name) name
#endif

#include <cuda.h>
#include <cstdlib>

namespace snp {
namespace {   // per translation unit (the file is compiled once per stage size)

// Pipeline trace (profiling aid, read with snp_debug_fastid_trace): CTA 0 records
// clock64 stamps per iteration: [0] expander before waits, [1] after pfull+empty,
// [2] before full arrive, [3] MMA after full wait.  Enabled by SNP_TRACE=1.
__device__ long long g_fastid_trace[8 * 1024];
__device__ long long g_fastid_etrace[4 * 256];   // FASTID_TRACE2: per tile, CTA 0
__device__ long long g_fastid_wtrace[4 * 1024];
__device__ long long g_fastid_wtrace2[32 * 1024]; // FASTID_TRACE2: per stage and warp qa: 8 stamps  // FASTID_TRACE2: per stage, full-arrive clock of warps qa = 0..3
__device__ long long g_fastid_cta_time[4 * 1024];   // per CTA: entry, after griddepcontrol.wait, main loop, end
__device__ long long g_fastid_launch_time[2 * 64];   // CTA 0: start / end globaltimer per launch
__device__ unsigned int g_fastid_launch_ctr;   // per CTA: start, main loop start, end (globaltimer ns)


constexpr int BM = 128;
#ifndef FASTID_KBITS
#define FASTID_KBITS 512
#endif
constexpr int KBITS = FASTID_KBITS;     // bits per stage: 512 (64-byte rows), 256 (32-byte) or 1024 (128-byte)
static_assert(KBITS == 512 || KBITS == 256 || KBITS == 1024, "stage size");
constexpr int KW = KBITS / 32;          // packed words per row per stage
constexpr int ACOLS = KW * 4;           // TMEM columns of an expanded A stage
#ifndef FASTID_NP
#define FASTID_NP 8
#endif
#ifndef FASTID_NS
#define FASTID_NS 4
#endif
#ifndef FASTID_NS32
#define FASTID_NS32 6   // TMEM A stages of the 32-wide-query instantiations (GG = 2)
#endif
// Per-half-stage full barriers (the MMA starts on the first 256 bits while the expanders
// write the second half): measured on FastID-1M, 207 -> 195 us with 4 expander groups
// (popcounts counted in-kernel) but 185 -> 191 us with 2 groups, so only for GG = 4.
#ifndef FASTID_HALF
#define FASTID_HALF 4   // the GG that uses half-stage barriers (0: none)
#endif
// tcgen05 instructions issued from one SM sub-partition execute in order, so the TMEM
// stores (tcgen05.st) of the expander warp that shares the MMA warp's sub-partition queue
// behind every MMA already issued — measured: that lane quarter finished each stage
// 1 350 - 1 560 cycles after the other three (scripts/trace_fastid2.py), which throttled
// the pipeline to 600 - 760 cycles per 400-cycle stage (the TMA warp's sub-partition shows
// a smaller lag of the same kind).  With FASTID_ISSUE_AHEAD the MMA warp issues stage s only
// after that warp has ISSUED its stores for stage s + 1, so they are queued ahead of MMA(s):
// measured, the lag halves (~800 cycles) but the MMA then waits on the look-ahead, FastID-1M
// 0.192 -> 0.200 ms, so it is off.
#ifndef FASTID_ISSUE_AHEAD
#define FASTID_ISSUE_AHEAD 0
#endif
#ifndef FASTID_ELECT_STAGE
#define FASTID_ELECT_STAGE 1   // one elect.sync per stage's block of MMAs
#endif
#ifndef FASTID_COUNT_GG2
#define FASTID_COUNT_GG2 0   // experiment: 1024-bit stages with 2 groups also counting popcounts
#endif
#ifndef FASTID_ELECT_HALF
#define FASTID_ELECT_HALF 1   // the same for the half-stage (GG = 4) instantiations
#endif
#ifndef FASTID_NACC
#define FASTID_NACC 2   // TMEM accumulators (the MMA may run NACC - 1 tiles ahead of the epilogue)
#endif
constexpr int NACC = FASTID_NACC;
constexpr int NP = FASTID_NP;           // packed TMA ring depth (64 KB in flight per SM)
constexpr int PSTAGE = BM * KBITS / 8;  // packed per stage (8 KB: 64-byte rows, 64B swizzle;
                                        // 4 KB: 32-byte rows, 32B swizzle)
#ifndef FASTID_G
#define FASTID_G 4
#endif
#ifndef FASTID_NEPI2
#define FASTID_NEPI2 8   // epilogue warps of the GG = 2 kernels
#endif
#ifndef FASTID_NEPI
#define FASTID_NEPI 8
#endif
// Warp roles for GG expander groups (group g takes stages it = g mod GG; 4 warps each, one
// per TMEM lane quarter).  GG = 4 when the expanders also count the database popcounts;
// GG = 2 when the caller gives them (fewer warps competing for issue slots: measured
// 203 vs 220 us on FastID-1M).
// The warp scheduler favours higher warp ids, so the latency-critical single-thread
// roles get the highest ids: MMA issuer last, TMA producer next, epilogue below them.
// epilogue warps: lane quarter w % 4, column block w / 4 (Roles<GG>::NEPI)
template <int GG>
struct Roles {
    static constexpr int NEPI = GG == 2 ? FASTID_NEPI2 : FASTID_NEPI;
    static constexpr int G = GG;
    static constexpr int NEXP = 4 * GG;
#ifndef FASTID_EXP_HIGH
#define FASTID_EXP_HIGH 0   // experiment: expanders above the epilogue warps (scheduler priority)
#endif
    static constexpr int EPI_WARP0 = FASTID_EXP_HIGH ? 0 : NEXP;
    static constexpr int EXP_WARP0 = FASTID_EXP_HIGH ? NEPI : 0;
#ifndef FASTID_MMA_FIRST
    static constexpr int TMA_WARP = NEXP + NEPI;
    static constexpr int MMA_WARP = NEXP + NEPI + 1;
#else   // experiment: MMA issuer on SMSP (NEXP + NEPI) % 4, TMA producer on the next one
    static constexpr int TMA_WARP = NEXP + NEPI + 1;
    static constexpr int MMA_WARP = NEXP + NEPI;
#endif
    static constexpr int NTHREADS = (NEXP + NEPI + 2) * 32;
};
constexpr size_t MAX_SMEM = 232448;     // 227 KB opt-in

template <int BN, int GG>
struct FCfg {
    // TMEM A stages (KBITS / 8 columns each), a multiple of the expander group count GG so
    // every slot belongs to one group (a group waits only for its own previous use of a slot;
    // more groups than slots per slot would let mbarrier phases alias).  A 32-wide query batch
    // frees accumulator columns for more stages with 2 groups: the lane quarter that shares
    // the MMA warp's sub-partition runs ~3.5 stages behind the others (its TMEM stores queue
    // behind the issued MMAs, scripts/trace_fastid2.py), and deeper staging keeps the MMA fed.
#if defined(FASTID_NS32_K1024)   // experiment: TMEM A stages of the 32-wide 1024-bit-stage kernels
    static constexpr int NS_PREF = (KBITS == 1024 && BN == 32) ? FASTID_NS32_K1024
                                 : FASTID_NS != 4 ? FASTID_NS : (BN == 32 ? FASTID_NS32 : 4);
#else
    static constexpr int NS_PREF = FASTID_NS != 4 ? FASTID_NS : (BN == 32 ? FASTID_NS32 : 4);
#endif
#ifdef FASTID_NS_ANY   // experiment: slot count not a multiple of the group count
    static constexpr int NS_FIT = NS_PREF;
#else
    static constexpr int NS_FIT = NS_PREF / GG * GG;
#endif
    static constexpr bool OK = NS_FIT >= GG;   // else this (BN, GG) is not instantiated for launch
    static constexpr int NS = OK ? NS_FIT : GG;
    static_assert(NP % 4 == 0, "the packed ring is shared round-robin by up to 4 groups");
    static constexpr int ACC_COLS = BN;
    static constexpr int A_COL0 = NACC * ACC_COLS;
    static constexpr int SF_COL = A_COL0 + NS * ACOLS;
    static_assert(!OK || SF_COL + 32 <= 512, "TMEM budget");
};

// Epilogue of one launch: up to 4 comparison ops, all derived from the one AND count c of
// a (query, database row) pair by  x = cq * pQ + cd * pD + cc * c:
//   AND (0,0,1), XOR (1,1,-2), ANDNOT (1,0,-1), NOTAND (0,1,-1)   [uint32 wrap-around].
// Per op, the counts are stored (outs[j] != NULL) and/or the per-query best match is
// kept (best bit j): running (min count, lowest row) per query column in registers,
// merged across warps and CTAs by a 64-bit atomicMin on (count << 32 | row) keys.
constexpr int MAXOPS = 4;

struct FArgs {
    const uint32_t *Q;   // queries (column side), packed u32 view
    int64_t nq, ldq32;
    int64_t nd;          // database rows (lane side)
    int64_t nbits;
    int nops;
    uint32_t cq[MAXOPS], cd[MAXOPS], cc[MAXOPS];
    uint32_t *outs[MAXOPS];
    int accumulate;
    int64_t ldo;
    int best_mask;                       // bit j: keep the best match of op j
    unsigned long long *keys;            // [nops][nq] ~(count << 32 | local row); zero-filled on entry and exit
    unsigned int *done;                  // epilogue-warp completion counter; zero on entry and exit
    uint32_t *best_count[MAXOPS];        // [nq] per op with a best bit
    int64_t *best_index[MAXOPS];
    int64_t index_base;
    int64_t ntiles;
    int nst;
    size_t qbytes;       // expanded query bytes in shared memory
    int trace;
    int nostore;         // profiling experiment: skip the output stores
    const uint32_t *popDg;   // database row popcounts (resident with the database), or NULL:
                             // then the expanders count them from the streamed words
};

// NOPS: ops per launch; BEST: keep best matches; ACC: accumulate into the counts.
// Everything uniform that would otherwise be tested inside the 32-column epilogue loop
// is a template parameter or folded into per-lane predicates: loop unswitching on
// runtime flags multiplied the code size (214 KB) and the instruction-cache misses
// slowed every warp role 3x.
// OPS >= 0: the ops are compile-time (op j in bits 2j..2j+1), so the epilogue key is two
// shift/add instructions per (column, op) instead of two IMADs by runtime coefficients.
// OPS = -1: coefficients from FArgs (any combination).
__host__ __device__ constexpr uint32_t op_cq(int op) { return (op == 1 || op == 2) ? 1u : 0u; }
__host__ __device__ constexpr uint32_t op_cd(int op) { return (op == 1 || op == 3) ? 1u : 0u; }
__host__ __device__ constexpr uint32_t op_cc(int op) { return op == 0 ? 1u : op == 1 ? (uint32_t)-2 : (uint32_t)-1; }

template <int BN, int NOPS, bool BEST, bool ACC, int OPS, int GG>
__global__ void __launch_bounds__(Roles<GG>::NTHREADS, 1)
fastid_tc4_kernel(const __grid_constant__ CUtensorMap tmD, const FArgs args) {
    constexpr int G = GG, NEXP = Roles<GG>::NEXP, EPI_WARP0 = Roles<GG>::EPI_WARP0, EXP_WARP0 = Roles<GG>::EXP_WARP0;
    constexpr int TMA_WARP = Roles<GG>::TMA_WARP, MMA_WARP = Roles<GG>::MMA_WARP;
    constexpr int NTHREADS = Roles<GG>::NTHREADS, NEPI = Roles<GG>::NEPI;
#ifndef FASTID_HALF1024
#define FASTID_HALF1024 0   // experiment: half-stage barriers for the 2-group 1024-bit kernels
#endif
    constexpr int NHALF = ((GG == FASTID_HALF && KBITS == 512) || (FASTID_HALF1024 && GG == 2 && KBITS == 1024)) ? 2 : 1;
    using C = FCfg<BN, GG>;
    if constexpr (!C::OK) {
        return;   // never launched (launch_f refuses this configuration)
    } else {
    constexpr int NS = C::NS;
    extern __shared__ __align__(1024) uint8_t smem[];
    uint8_t *qsm = smem;                                            // [nst*8 chunks][BN][16 B]
    uint8_t *ring = smem + args.qbytes;                             // [NP][PSTAGE]
    uint64_t *bars = reinterpret_cast<uint64_t *>(ring + NP * PSTAGE);
    uint64_t *pfull = bars;                  // [NP] TMA -> expanders
    uint64_t *pempty = pfull + NP;           // [NP] expanders -> TMA
    uint64_t *full = pempty + NP;            // [NS][NHALF] expanders -> MMA
    uint64_t *empty = full + NS * NHALF;     // [NS] MMA -> expanders
    uint64_t *accf = empty + NS;             // [NACC]
    uint64_t *acce = accf + NACC;            // [NACC]
    uint64_t *popf = acce + NACC;            // [NACC]
    uint64_t *issued = popf + NACC;          // [NS] MMA-sub-partition expander -> MMA: stores issued
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(issued + NS);
    uint32_t *popQ = tmem_slot + 4;          // [BN]
    uint32_t *popD = popQ + BN;              // [2 acc][G][BM]
    uint32_t *popQ32 = popD + NACC * G * BM; // [BN] 32 * popQ (epilogue key term)

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    __shared__ unsigned int launch_k;
    if (SNP_PROF(args.trace) && tid == 0 && blockIdx.x < 1024) g_fastid_cta_time[4 * blockIdx.x] = (long long)ptx::globaltimer_ns();
    if (SNP_PROF(args.trace) && tid == 0 && blockIdx.x == 0) {
        launch_k = atomicAdd(&g_fastid_launch_ctr, 1u) & 63u;
        g_fastid_launch_time[2 * launch_k] = (long long)ptx::globaltimer_ns();
    }
    const int64_t nbits = args.nbits;
    const int nst = args.nst;
#if defined(FASTID_TILE_GROUP)
    // measurement variant: groups of FASTID_TILE_GROUP adjacent tiles per CTA, the CTAs sweeping
    // the database together group by group
    constexpr int64_t TG = FASTID_TILE_GROUP;
    const int64_t ngroups = (args.ntiles + TG - 1) / TG;
    const int64_t my_groups = ngroups > blockIdx.x ? (ngroups - 1 - blockIdx.x) / gridDim.x + 1 : 0;
    int64_t my_tiles = my_groups * TG;
    if (my_groups > 0) {   // the last group may be ragged
        const int64_t lastg = blockIdx.x + (my_groups - 1) * gridDim.x;
        const int64_t rem = args.ntiles - lastg * TG;
        my_tiles -= TG - (rem < TG ? rem : TG);
    }
#define FASTID_TILE(tl) (((tl) / TG) * gridDim.x * TG + (int64_t)blockIdx.x * TG + (tl) % TG)
#elif !defined(FASTID_CONTIG_TILES)
    // tile tl of this CTA is blockIdx.x + tl * gridDim.x (the CTAs sweep the database together)
    const int64_t my_tiles = args.ntiles > blockIdx.x ? (args.ntiles - 1 - blockIdx.x) / gridDim.x + 1 : 0;
    const int64_t tile0 = blockIdx.x, tstep = gridDim.x;
#define FASTID_TILE(tl) (tile0 + (tl) * tstep)
#else
    // measurement variant: each CTA takes one contiguous block of tiles
    const int64_t tile0 = args.ntiles * blockIdx.x / gridDim.x, tstep = 1;
    const int64_t my_tiles = args.ntiles * (blockIdx.x + 1) / gridDim.x - tile0;
#define FASTID_TILE(tl) (tile0 + (tl) * tstep)
#endif
    const int64_t total_it = my_tiles * nst;
    const int64_t full32 = nbits / 32;

    if (tid == 0) {
        for (int i = 0; i < NP; ++i) {
            ptx::mbar_init(&pfull[i], 1);
            ptx::mbar_init(&pempty[i], 4);
        }
        for (int i = 0; i < NS; ++i) {
            for (int h = 0; h < NHALF; ++h) ptx::mbar_init(&full[i * NHALF + h], 4);
            ptx::mbar_init(&empty[i], 1);
        }
        for (int i = 0; i < NACC; ++i) {
            ptx::mbar_init(&accf[i], 1);
            ptx::mbar_init(&acce[i], NEPI);
            ptx::mbar_init(&popf[i], NEXP);
        }
        for (int i = 0; i < NS; ++i) ptx::mbar_init(&issued[i], 1);
        ptx::fence_mbar_init();
    }
    if (warp == TMA_WARP && lane == 0) ptx::prefetch_tensormap(&tmD);
    for (int r = tid; r < BN; r += NTHREADS) popQ[r] = 0;
    if (warp == MMA_WARP) ptx::tmem_alloc<512>(tmem_slot);
    ptx::tc_fence_before();
    __syncthreads();
    ptx::tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    // launched with programmatic stream serialization: everything above overlapped the
    // previous kernel in the stream (the key-init kernel); its results (and the packed
    // queries from before it) are visible after this wait
    asm volatile("griddepcontrol.wait;" ::: "memory");
#ifndef FASTID_EARLY_TMA
#define FASTID_EARLY_TMA 1
#endif
    // the first ring fill is issued before the query prologue (the ring does not depend on the
    // queries): FastID-1M 169.6 -> 168.9 us.  (With the per-MMA elect issue loop this ordering
    // measured 30 % slower; that loop was later found to be sensitive to code generation —
    // the cause was not isolated further.)
    // Only for the 2-group (database popcounts given) kernels: with 4 expander groups and
    // half-stage barriers it measured ~10 % slower (FastID-1M without popD 182 -> 200 us).
    constexpr bool EARLY = FASTID_EARLY_TMA && GG == 2;
    const int64_t n_early = EARLY ? (total_it < NP ? total_it : (int64_t)NP) : 0;
    if (EARLY && warp == TMA_WARP && lane == 0) {
        for (int64_t it = 0; it < n_early; ++it) {
            const int64_t t = FASTID_TILE(it / nst);
            const int s = (int)(it % nst);
            ptx::mbar_arrive_expect_tx(&pfull[it], PSTAGE);
            ptx::tma_load_2d(ring + it * PSTAGE, &tmD, &pfull[it], s * (KBITS / 32), (int32_t)(t * BM));
        }
    }
    if (SNP_PROF(args.trace) && tid == 0 && blockIdx.x < 1024) g_fastid_cta_time[4 * blockIdx.x + 1] = (long long)ptx::globaltimer_ns();
    // ---- prologue: expand the whole query batch once (resident MMA B operand).  A warp item
    // is 8 query rows x 16 words: lane = (row r = lane & 7, 4-word chunk c = lane >> 3), one
    // 16-byte load per lane (each row's 64 bytes in whole sectors), and every 16-byte store
    // instruction covers 8 consecutive rows of one word (128 contiguous bytes per chunk:
    // 4 wavefronts, conflict-free).  Row popcounts: reduced over the 4 chunks, one shared
    // atomic per row and item.  (Round 2's lane-per-row prologue issued 32 sectors per load
    // and took ~6 us per CTA, 3-4 % of FastID-1M.)
    {
        static_assert(KBITS % 512 == 0, "16-word items");
        const int nwb = nst * (KBITS / 32) / 16;   // 16-word blocks per row
        const int nitems = (BN / 8) * nwb;
        const int64_t nw32 = ((nbits + 127) / 128) * 4;
        const int r8 = lane & 7, c4 = lane >> 3;
        // items in batches of 4 per warp: all four loads are in flight before the first use
        constexpr int NWARPS = NTHREADS / 32;
        for (int item0 = warp; item0 < nitems; item0 += 4 * NWARPS) {
            uint4 x[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                const int item = item0 + u * NWARPS;
                const int row = (item % (BN / 8)) * 8 + r8;
                const int w = (item / (BN / 8)) * 16 + c4 * 4;
                x[u] = make_uint4(0u, 0u, 0u, 0u);
                if (item < nitems && row < args.nq && w < nw32)
                    x[u] = __ldg(reinterpret_cast<const uint4 *>(args.Q + row * args.ldq32 + w));
            }
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                const int item = item0 + u * NWARPS;
                if (item >= nitems) break;   // warp-uniform
                const int row = (item % (BN / 8)) * 8 + r8;
                const int w = (item / (BN / 8)) * 16 + c4 * 4;
                x[u].x &= word_mask(w, nbits);
                x[u].y &= word_mask(w + 1, nbits);
                x[u].z &= word_mask(w + 2, nbits);
                x[u].w &= word_mask(w + 3, nbits);
                uint32_t pc = __popc(x[u].x) + __popc(x[u].y) + __popc(x[u].z) + __popc(x[u].w);
                uint8_t *dst = qsm + (size_t)w * BN * 16 + row * 16;
                uint4 o;
                expandB(x[u].x, o.x, o.y, o.z, o.w);
                *reinterpret_cast<uint4 *>(dst) = o;
                expandB(x[u].y, o.x, o.y, o.z, o.w);
                *reinterpret_cast<uint4 *>(dst + BN * 16) = o;
                expandB(x[u].z, o.x, o.y, o.z, o.w);
                *reinterpret_cast<uint4 *>(dst + 2 * BN * 16) = o;
                expandB(x[u].w, o.x, o.y, o.z, o.w);
                *reinterpret_cast<uint4 *>(dst + 3 * BN * 16) = o;
                pc += __shfl_xor_sync(0xffffffffu, pc, 8);
                pc += __shfl_xor_sync(0xffffffffu, pc, 16);
                if (c4 == 0 && pc) atomicAdd(&popQ[row], pc);
            }
        }
    }
    if (warp >= EPI_WARP0 && warp < EPI_WARP0 + 4) {   // one warp per lane quarter
        const int q = warp & 3;
        uint32_t v[16];
#pragma unroll
        for (int i = 0; i < 16; ++i) v[i] = 0x7F7F7F7Fu;   // ue8m0 scale 2^0 in every byte
        ptx::tmem_st16(tmem + ((uint32_t)(q * 32) << 16) + C::SF_COL, v);
        ptx::tmem_st16(tmem + ((uint32_t)(q * 32) << 16) + C::SF_COL + 16, v);
        ptx::tmem_st_wait();
    }
    ptx::fence_proxy_async_smem();
    ptx::tc_fence_before();
    __syncthreads();
    ptx::tc_fence_after();
    if (warp >= EPI_WARP0 && warp < EPI_WARP0 + NEPI) {   // only the epilogue warps read it
        for (int r = tid - EPI_WARP0 * 32; r < BN; r += NEPI * 32) popQ32[r] = 32u * popQ[r];
        asm volatile("bar.sync 1, %0;" ::"r"(NEPI * 32) : "memory");
    }

    if (SNP_PROF(args.trace) && tid == 0 && blockIdx.x < 1024) g_fastid_cta_time[4 * blockIdx.x + 2] = (long long)ptx::globaltimer_ns();
    if (warp == TMA_WARP) {
        // ------------------------------------------------------------ TMA producer
        if (lane == 0) {
#ifdef FASTID_DB_EVICT_FIRST
            const uint64_t pol = ptx::l2_policy_evict_first();   // the database is read once
#endif
            int p = 0;
            uint32_t round = 0;   // how many times the ring has wrapped
            int64_t itp = 0;
            for (int64_t tl = 0; tl < my_tiles; ++tl) {
                const int64_t t = FASTID_TILE(tl);
                const int32_t row0 = (int32_t)(t * BM);
                for (int s = 0; s < nst; ++s, ++itp) {
                    if (EARLY && itp < n_early) {   // issued before the prologue
                        if (++p == NP) { p = 0; ++round; }
                        continue;
                    }
                    if (round > 0) ptx::mbar_wait(&pempty[p], (round - 1) & 1);   // lane 0 only
                    ptx::mbar_arrive_expect_tx(&pfull[p], PSTAGE);
#ifdef FASTID_DB_EVICT_FIRST
                    ptx::tma_load_2d_hint(ring + p * PSTAGE, &tmD, &pfull[p], s * (KBITS / 32), row0, pol);
#else
                    ptx::tma_load_2d(ring + p * PSTAGE, &tmD, &pfull[p], s * (KBITS / 32), row0);
#endif
                    if (++p == NP) { p = 0; ++round; }
                }
            }
        }
    } else if (warp >= EXP_WARP0 && warp < EXP_WARP0 + NEXP) {
        // ------------------------------------------------------------ expanders
        // group g = warp / 4 handles iterations it = g, g+G, ...; warp (g, q) handles the
        // 32 database rows of lane quarter q for all 256 bits of the stage.
        const int g = (warp - EXP_WARP0) >> 2, qa = warp & 3;   // EXP_WARP0 is a multiple of 4
        const int arow = qa * 32 + lane;
        uint32_t popa = 0;
        int cur_tl = 0;       // tile whose popcount partial is being accumulated
        const bool pre = args.popDg != nullptr;
        auto publish_until = [&](int upto) {
            if (pre) return;
            for (; cur_tl < upto; ++cur_tl) {
                const int acc = cur_tl % NACC;
                if (cur_tl >= NACC) ptx::mbar_wait_warp(&acce[acc], (uint32_t)((cur_tl / NACC - 1) & 1));
                popD[(acc * G + g) * BM + arow] = popa;
                popa = 0;
                __syncwarp();
                if (lane == 0) ptx::mbar_arrive(&popf[acc]);
            }
        };
        // 32-bit loop state (total_it < 2^31: fastid_tc4_supported bounds nd): the loop
        // bookkeeping is a visible share of the expander instruction stream
        int tl = g / nst;
        int s = g % nst;
        // stage it = g uses ring slot g % NP (round g / NP) and TMEM slot g % NS (round g / NS)
        int p = g % NP, b = g % NS;
        uint32_t pround = (uint32_t)(g / NP), bround = (uint32_t)(g / NS);
        const int total_it32 = (int)total_it;
        for (int it = g; it < total_it32; it += G) {
            publish_until(tl);
#if defined(FASTID_TRACE) || defined(FASTID_TRACE2)
            const bool tr = SNP_PROF(args.trace) && blockIdx.x == 0 && lane == 0 && qa == 0 && it < 1024;
#endif
#ifdef FASTID_TRACE2
            const bool trw = SNP_PROF(args.trace) && blockIdx.x == 0 && lane == 0 && it < 1024;
            long long *tw2 = g_fastid_wtrace2 + 32 * it + 8 * qa;
#endif
#if defined(FASTID_TRACE) || defined(FASTID_TRACE2)
            if (tr) g_fastid_trace[8 * it + 0] = clock64();
#ifdef FASTID_TRACE2
            if (trw) tw2[0] = clock64();
#endif
#endif
            ptx::mbar_wait_warp(&pfull[p], pround & 1);
#ifdef FASTID_TRACE2
            if (tr) g_fastid_trace[8 * it + 4] = clock64();
#ifdef FASTID_TRACE2
            if (trw) tw2[4] = clock64();
#endif
#endif
            if (bround > 0) ptx::mbar_wait_warp(&empty[b], (bround - 1) & 1);
#if defined(FASTID_TRACE) || defined(FASTID_TRACE2)
            if (tr) g_fastid_trace[8 * it + 1] = clock64();
#ifdef FASTID_TRACE2
            if (trw) tw2[1] = clock64();
#endif
#endif
            // 64-byte row of the stage; TMA 64B swizzle: 16-byte chunk c of row r sits at
            // chunk c ^ ((r >> 1) & 3)  (conflict-free LDS.128 across the warp)
            // (32-byte rows, 32B swizzle: chunk c of row r sits at c ^ ((r >> 2) & 1))
            const uint8_t *src = ring + p * PSTAGE + arow * (KBITS / 8);
            // (128-byte rows, 128B swizzle: chunk c of row r sits at c ^ (r & 7))
            const int sw = KBITS == 1024 ? (arow & 7) : KBITS == 512 ? (arow >> 1) & 3 : (arow >> 2) & 1;
            uint32_t wv[KW];
#pragma unroll
            for (int c = 0; c < KW / 4; ++c) {
                const uint4 x = *reinterpret_cast<const uint4 *>(src + ((c ^ sw) << 4));
                wv[4 * c] = x.x; wv[4 * c + 1] = x.y; wv[4 * c + 2] = x.z; wv[4 * c + 3] = x.w;
            }
            const int64_t w0 = (int64_t)s * KW;
            if (w0 + KW > full32) {   // the profile's last stage: bits past nbits are zeroed
                // 32-bit arithmetic on the bits left in this stage (0 < rem < KBITS)
                const int rem = (int)(nbits - w0 * 32);
#pragma unroll
                for (int i = 0; i < KW; ++i) {
                    const int r = rem - 32 * i;
                    wv[i] &= r >= 32 ? 0xffffffffu : r <= 0 ? 0u : (1u << r) - 1u;
                }
            }
            if (!pre) {
#pragma unroll
                for (int i = 0; i < KW; ++i) popa += __popc(wv[i]);
            }
            __syncwarp();
            if (lane == 0) ptx::mbar_arrive(&pempty[p]);
#ifdef FASTID_TRACE2
            if (tr) g_fastid_trace[8 * it + 6] = clock64();
#ifdef FASTID_TRACE2
            if (trw) tw2[6] = clock64();
#endif
#endif
            const uint32_t tbase = tmem + ((uint32_t)(qa * 32) << 16) + (uint32_t)(C::A_COL0 + ACOLS * b);
            // the last stage of a short profile: only the 256-bit groups that hold bits < nbits
            // are expanded (the MMA issues only the K-steps that cover them)
            const int hmax = (int)((nbits - w0 * 32 + 255) / 256) < KW / 8 ? (int)((nbits - w0 * 32 + 255) / 256) : KW / 8;
#pragma unroll
            for (int h = 0; h < KW / 8; ++h) {
                if (NHALF == 1 && h >= hmax) break;
                uint32_t v[32];
#pragma unroll
                for (int i = 0; i < 8; ++i)
                    expandA(wv[8 * h + i], v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
                ptx::tmem_st32(tbase + 32 * h, v);
                if (NHALF == 2 && h == KW / 16 - 1) {   // publish the first half: the MMA may start on it
                    ptx::tmem_st_wait();
                    ptx::tc_fence_before();
                    __syncwarp();
                    if (lane == 0) ptx::mbar_arrive(&full[b * NHALF]);
                }
            }
#ifdef FASTID_TRACE2
            if (tr) g_fastid_trace[8 * it + 7] = clock64();
#ifdef FASTID_TRACE2
            if (trw) tw2[7] = clock64();
#endif
#endif
            if (FASTID_ISSUE_AHEAD && qa == (MMA_WARP & 3)) {
                __syncwarp();   // every lane's tcgen05.st of this stage is issued
                if (lane == 0) ptx::mbar_arrive(&issued[b]);
            }
            ptx::tmem_st_wait();
            ptx::tc_fence_before();
            __syncwarp();
#if defined(FASTID_TRACE) || defined(FASTID_TRACE2)
            if (tr) g_fastid_trace[8 * it + 2] = clock64();
#ifdef FASTID_TRACE2
            if (trw) tw2[2] = clock64();
#endif
#endif
#ifdef FASTID_TRACE2
            if (SNP_PROF(args.trace) && blockIdx.x == 0 && lane == 0 && it < 1024) g_fastid_wtrace[4 * it + qa] = clock64();
#endif
            if (lane == 0) ptx::mbar_arrive(&full[b * NHALF + NHALF - 1]);
            s += G;
            while (s >= nst) { s -= nst; ++tl; }
            p += G;
            while (p >= NP) { p -= NP; ++pround; }
            b += G;
            while (b >= NS) { b -= NS; ++bround; }
        }
        publish_until((int)my_tiles);
    } else if (warp == MMA_WARP) {
        // ------------------------------------------------------------ MMA issuer
        // The whole warp runs the loop (converged, uniform values); the elected lane issues.
        // Descriptors are precomputed: stepping K only adds to the start-address field.
        // tmem was read from shared memory (a per-thread value to ptxas); a warp reduction
        // lands it in a uniform register so everything derived from it stays uniform.
        constexpr uint32_t IDESC = idesc_mxf4(BM, BN);
        const int kmax_last = (int)((nbits - (int64_t)(nst - 1) * KBITS + 63) / 64);   // 1 .. KBITS / 64
        const uint32_t tmu = __reduce_or_sync(0xffffffffu, tmem);
        const uint32_t sfa = tmu + C::SF_COL, sfb = tmu + C::SF_COL + 16;
        const uint64_t bdesc0 = ptx::smem_desc_kmajor_noswizzle(ptx::smem_u32(qsm), BN * 16, 128);
        constexpr uint32_t BSTEP = (2 * BN * 16) >> 4;           // one K-step = 2 chunks
        constexpr uint32_t SSTEP = ((KBITS / 32) * BN * 16) >> 4; // one stage = 16 chunks
        // Waits are warp votes, so every loop value below is warp-uniform and lives in
        // uniform registers: ~7 uniform instructions per MMA instead of ~16 with R2URs.
        int b = 0;
        uint32_t bround = 0;
        int64_t itm = 0;
        for (int64_t tl = 0; tl < my_tiles; ++tl) {
            const uint32_t tl32 = (uint32_t)tl;
            const int acc = (int)(tl32 % NACC);
#ifdef FASTID_TRACE2
            if (SNP_PROF(args.trace) && blockIdx.x == 0 && lane == 0 && tl < 256) g_fastid_etrace[4 * tl + 0] = clock64();
#endif
            if (tl32 >= NACC) ptx::mbar_wait_uniform(&acce[acc], (tl32 / NACC - 1) & 1u);
#ifdef FASTID_TRACE2
            if (SNP_PROF(args.trace) && blockIdx.x == 0 && lane == 0 && tl < 256) g_fastid_etrace[4 * tl + 1] = clock64();
#endif
            ptx::tc_fence_after();
            const uint32_t d = tmu + (uint32_t)(acc * C::ACC_COLS);
            uint64_t bd = bdesc0;
            for (int s = 0; s < nst; ++s, ++itm) {
#ifdef FASTID_TRACE2
                if (SNP_PROF(args.trace) && blockIdx.x == 0 && lane == 0 && itm < 1024) g_fastid_trace[8 * itm + 3] = clock64();
#endif
                ptx::mbar_wait_uniform(&full[b * NHALF], bround & 1);
                if (FASTID_ISSUE_AHEAD && itm + 1 < total_it) {
                    // the next stage's stores on this sub-partition go ahead of these MMAs
                    const int bn = b + 1 == NS ? 0 : b + 1;
                    const uint32_t rn = b + 1 == NS ? bround + 1 : bround;
                    ptx::mbar_wait_uniform(&issued[bn], rn & 1);
                }
                ptx::tc_fence_after();
#ifdef FASTID_TRACE2
                if (SNP_PROF(args.trace) && blockIdx.x == 0 && lane == 0 && itm < 1024) g_fastid_trace[8 * itm + 5] = clock64();
#endif
                const uint32_t a0 = tmu + (uint32_t)(C::A_COL0 + ACOLS * b);
                // K-steps of this stage that hold bits < nbits (the rest would multiply zeros:
                // a 128-SNP profile issues 2 MMAs per tile instead of KBITS / 64)
                const int kmax = s == nst - 1 ? kmax_last : KBITS / 64;
                if (NHALF == 1 && FASTID_ELECT_STAGE) {
                    // one elected lane issues the stage's MMAs back to back and commits them (one
                    // elect.sync per stage, not per MMA: the MMA issue is on the pipeline's
                    // critical path — FastID-1M 171.5 -> 169.0 us, 8 x 20M x 4096 best-only
                    // 2.34 -> 2.13 ms); a full stage has no per-MMA bound test
                    if (ptx::elect_one()) {
                        if (kmax == KBITS / 64) {
#pragma unroll
                            for (int k = 0; k < KBITS / 64; ++k)
                                ptx::mma_mxf4_ts_one(d, a0 + 8 * k, bd + (uint64_t)(k * BSTEP), IDESC,
                                                     (s | k) != 0 ? 1u : 0u, sfa, sfb);
                        } else {
#pragma unroll
                            for (int k = 0; k < KBITS / 64; ++k) {
                                if (k >= kmax) break;
                                ptx::mma_mxf4_ts_one(d, a0 + 8 * k, bd + (uint64_t)(k * BSTEP), IDESC,
                                                     (s | k) != 0 ? 1u : 0u, sfa, sfb);
                            }
                        }
                        ptx::mma_commit_one(&empty[b]);
                        if (s == nst - 1) ptx::mma_commit_one(&accf[acc]);
                    }
                    __syncwarp();
                    bd += SSTEP;
                    if (++b == NS) { b = 0; ++bround; }
                    continue;
                } else if (NHALF == 2 && FASTID_ELECT_HALF) {
                    // half-stage barriers: the same per-half elected issue (elect.sync picks the
                    // same lane both times, so the commits track both halves' MMAs)
                    constexpr int KH = KBITS / 128;
                    if (ptx::elect_one()) {
#pragma unroll
                        for (int k = 0; k < KH; ++k)
                            ptx::mma_mxf4_ts_one(d, a0 + 8 * k, bd + (uint64_t)(k * BSTEP), IDESC,
                                                 (s | k) != 0 ? 1u : 0u, sfa, sfb);
                    }
                    __syncwarp();
                    ptx::mbar_wait_uniform(&full[b * NHALF + 1], bround & 1);
                    ptx::tc_fence_after();
                    if (ptx::elect_one()) {
#pragma unroll
                        for (int k = KH; k < 2 * KH; ++k)
                            ptx::mma_mxf4_ts_one(d, a0 + 8 * k, bd + (uint64_t)(k * BSTEP), IDESC, 1u, sfa, sfb);
                        ptx::mma_commit_one(&empty[b]);
                        if (s == nst - 1) ptx::mma_commit_one(&accf[acc]);
                    }
                    __syncwarp();
                    bd += SSTEP;
                    if (++b == NS) { b = 0; ++bround; }
                    continue;
                } else {
#pragma unroll
                    for (int k = 0; k < KBITS / 64; ++k) {
                        if (NHALF == 2 && k == KBITS / 128) {   // second half of the stage
                            ptx::mbar_wait_uniform(&full[b * NHALF + 1], bround & 1);
                            ptx::tc_fence_after();
                        }
                        if (NHALF == 1 && k >= kmax) break;
                        ptx::mma_mxf4_ts(d, a0 + 8 * k, bd + (uint64_t)(k * BSTEP), IDESC, (s | k) != 0 ? 1u : 0u,
                                         sfa, sfb);
                    }
                }
                ptx::mma_commit_uniform(&empty[b]);
                bd += SSTEP;
                if (++b == NS) { b = 0; ++bround; }
            }
            if (!(NHALF == 1 ? FASTID_ELECT_STAGE : FASTID_ELECT_HALF)) ptx::mma_commit_uniform(&accf[acc]);
        }
        __syncwarp();
    } else {
        // ------------------------------------------------------------ epilogue (8 warps)
        // warp e: TMEM lane quarter e % 4 (database rows), query columns [EC h, EC h + EC)
        constexpr int EC = BN * 4 / NEPI;   // 32 (8 epilogue warps) or 16 (16 warps)
        static_assert(EC == 16 || EC == 32, "epilogue column block");
        const int e = warp - EPI_WARP0;
        const int q = e & 3, h = e >> 2;
        const int li = q * 32 + lane;
        const int c0 = EC * h;
        const int ncols = (int)(args.nq - c0 < EC ? (args.nq - c0 > 0 ? args.nq - c0 : 0) : EC);
        const int64_t ldo = args.ldo;
        // running best of column c0 + lane, per op (held by that lane only)
        uint32_t bc[NOPS], bi[NOPS];
#pragma unroll
        for (int j = 0; j < NOPS; ++j) { bc[j] = 0xffffffffu; bi[j] = 0xffffffffu; }
        for (int64_t tl = 0; tl < my_tiles; ++tl) {
            const int acc = (int)((uint32_t)tl % NACC);
            const uint32_t ph = ((uint32_t)tl / NACC) & 1u;
            const int64_t t = FASTID_TILE(tl);
            const bool pre = args.popDg != nullptr;
            const int64_t gd_l = t * BM + li;   // this lane's local database row
            uint32_t pd = 0;
            if (pre) pd = gd_l < args.nd ? __ldg(args.popDg + gd_l) : 0u;   // before the wait
            else ptx::mbar_wait_warp(&popf[acc], ph);
            ptx::mbar_wait_warp(&accf[acc], ph);
#ifdef FASTID_TRACE2
            if (SNP_PROF(args.trace) && blockIdx.x == 0 && e == 0 && lane == 0 && tl < 256) g_fastid_etrace[4 * tl + 2] = clock64();
#endif
            ptx::tc_fence_after();
            uint32_t v[EC];
            if constexpr (EC == 32) ptx::tmem_ld32(tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(acc * C::ACC_COLS + c0), v);
            else ptx::tmem_ld16(tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(acc * C::ACC_COLS + c0), v);
            if (!pre) {   // read the popcount partials BEFORE releasing the buffer pair
#pragma unroll
                for (int gg = 0; gg < G; ++gg) pd += popD[(acc * G + gg) * BM + li];
            }
            ptx::tmem_ld_wait();
            ptx::tc_fence_before();
            __syncwarp();
            if (lane == 0) ptx::mbar_arrive(&acce[acc]);   // accumulator + pops drained: reusable
            if (ncols == 0) continue;                      // nq <= 32: this column half is idle
            const int64_t row0 = t * BM + q * 32;          // local database row of lane 0
            const int64_t gd = row0 + lane;
            const bool valid = gd < args.nd;
            // Everything is computed as the 32x-scaled key of the best-match reduction:
            //   key = 32 x + lane,  x = cq pQ + cd pD + cc c  (op identity)
            // and the count c comes out of the fp32 accumulator by the 2^23 magic add
            // (fb = bits(v + 2^23) = 0x4B000000 + c for 0 <= c < 2^23; FMA pipe, no F2I):
            //   key = 32cc fb + cq (32 pQ) + [32 cd pD - 32 cc 0x4B000000 + lane]   (mod 2^32).
            // Invalid rows (past nd) get +0xF0000000 instead of lane: larger than every real
            // key (< 2^28), so they never win a reduction and are never stored.
            const uint32_t laneterm = valid ? (uint32_t)lane : 0xF0000000u;
            uint32_t L[NOPS], C32[NOPS];
            bool sv[NOPS];
            uint32_t *op_[NOPS];
#pragma unroll
            for (int j = 0; j < NOPS; ++j) {
                if (OPS >= 0) {
                    const int op = (OPS >> (2 * j)) & 3;
                    C32[j] = 32u * op_cc(op);
                    L[j] = 32u * op_cd(op) * pd - C32[j] * 0x4B000000u + laneterm;
                } else {
                    C32[j] = 32u * args.cc[j];
                    L[j] = 32u * args.cd[j] * pd - C32[j] * 0x4B000000u + laneterm;
                }
                sv[j] = valid && args.outs[j] != nullptr && !SNP_PROF(args.nostore);
                op_[j] = sv[j] ? args.outs[j] + (int64_t)c0 * ldo + gd : nullptr;
            }
            // best match: key = count << 5 | lane, so ONE redux.sync.min gives the tile
            // quarter's minimum count and, among equal counts, its lowest row; lane u keeps
            // column u's tile minimum and folds it into its running best once per tile
            uint32_t mk[NOPS];
#pragma unroll
            for (int j = 0; j < NOPS; ++j) mk[j] = 0xffffffffu;
#pragma unroll
            for (int u = 0; u < EC; ++u) {
                const uint32_t fb = __float_as_uint(__fadd_rn(__uint_as_float(v[u]), 8388608.0f));
                const uint32_t pq32 = popQ32[c0 + u];
                const bool colok = u < ncols;
#pragma unroll
                for (int j = 0; j < NOPS; ++j) {
                    uint32_t key;
                    if (OPS >= 0) {
                        const int op = (OPS >> (2 * j)) & 3;
                        const uint32_t f32 = fb << 5;
                        key = op == 0 ? f32 + L[j]                       // AND
                            : op == 1 ? pq32 + L[j] - (f32 << 1)         // XOR
                            : op == 2 ? pq32 + L[j] - f32                // ANDNOT
                                      : L[j] - f32;                      // NOTAND
                    } else {
                        key = C32[j] * fb + (args.cq[j] * pq32 + L[j]);
                    }
                    if (sv[j] && colok) {
                        const uint32_t x = key >> 5;   // valid rows: laneterm = lane < 32
                        if (ACC) *op_[j] += x;
                        else {
#ifndef FASTID_STORE_CS
                            // plain write-back store: measured 1.8-2.5 % faster on FastID-1M than the
                            // evict-first streaming store (0.1791 vs 0.1838 ms; -DFASTID_STORE_CS)
                            *op_[j] = x;
#else
                            __stcs(op_[j], x);
#endif
                        }
                    }
                    op_[j] += ldo;   // running pointer: one 64-bit add per store, not a product
                    if (BEST) {
                        const uint32_t m = __reduce_min_sync(0xffffffffu, key);
                        mk[j] = lane == u ? m : mk[j];
                    }
                }
            }
            if (BEST) {
#pragma unroll
                for (int j = 0; j < NOPS; ++j) {
                    // tiles arrive in increasing row order: strict < keeps the lowest row
                    if (mk[j] < 0xF0000000u && (mk[j] >> 5) < bc[j]) {
                        bc[j] = mk[j] >> 5;
                        bi[j] = (uint32_t)row0 + (mk[j] & 31u);
                    }
                }
            }
#ifdef FASTID_TRACE2
            if (SNP_PROF(args.trace) && blockIdx.x == 0 && e == 0 && lane == 0 && tl < 256) g_fastid_etrace[4 * tl + 3] = clock64();
#endif
        }
        if (BEST) {
#pragma unroll
            for (int j = 0; j < NOPS; ++j) {
                // keys are stored complemented and merged by atomicMax, so the zero-filled
                // workspace means "no candidate" and no init kernel runs before the search
                if (((args.best_mask >> j) & 1) && lane < ncols && bc[j] != 0xffffffffu)
                    atomicMax(args.keys + (int64_t)j * args.nq + c0 + lane,
                              ~(((unsigned long long)bc[j] << 32) | bi[j]));
            }
            // the last epilogue warp of the grid to finish turns the merged keys into
            // (best_count, best_index) (kept inside this role: a CTA-wide finalize after
            // the role branches de-uniformised the MMA issue loop)
            __threadfence();
            uint32_t last = 0;
            if (lane == 0) last = atomicAdd(args.done, 1u) == gridDim.x * NEPI - 1 ? 1u : 0u;
            if (__shfl_sync(0xffffffffu, last, 0)) {
                __threadfence();
                const int nq = (int)args.nq;   // <= 64 (fastid_tc4_supported)
#pragma unroll
                for (int j = 0; j < NOPS; ++j) {
                    if (!((args.best_mask >> j) & 1)) continue;
                    for (int i = lane; i < nq; i += 32) {
                        const unsigned long long k = ~__ldcg(args.keys + j * nq + i);
                        args.best_count[j][i] = k == ~0ULL ? 0xffffffffu : (uint32_t)(k >> 32);
                        args.best_index[j][i] = k == ~0ULL ? -1 : (int64_t)(k & 0xffffffffULL) + args.index_base;
                        args.keys[j * nq + i] = 0ULL;   // the workspace is left zero-filled
                    }
                }
                if (lane == 0) *args.done = 0u;
            }
        }
    }

    ptx::tc_fence_before();
    __syncthreads();
    if (SNP_PROF(args.trace) && tid == 0 && blockIdx.x < 1024) g_fastid_cta_time[4 * blockIdx.x + 3] = (long long)ptx::globaltimer_ns();
    if (SNP_PROF(args.trace) && tid == 0 && blockIdx.x == 0) g_fastid_launch_time[2 * launch_k + 1] = (long long)ptx::globaltimer_ns();
    if (warp == MMA_WARP) {
        ptx::tc_fence_after();
        ptx::tmem_dealloc<512>(tmem);
    }
    }   // C::OK
}

size_t smem_bytes(int bn, int64_t nbits) {
    const int64_t nst = (nbits + KBITS - 1) / KBITS;
    return (size_t)bn * (size_t)nst * (KBITS / 32) * 16 + NP * PSTAGE + 8192;   // + barriers, pops (~5 KB)
}

void op_coefs(int op, uint32_t &cq, uint32_t &cd, uint32_t &cc) {
    // x = cq pQ + cd pD + cc AND  (uint32 wrap-around for the negatives)
    switch (op) {
    case 0: cq = 0; cd = 0; cc = 1; break;                   // AND      Eq. (1)
    case 1: cq = 1; cd = 1; cc = (uint32_t)-2; break;        // XOR      Eq. (2)
    case 2: cq = 1; cd = 0; cc = (uint32_t)-1; break;        // ANDNOT   Eq. (3), r = query
    default: cq = 0; cd = 1; cc = (uint32_t)-1; break;       // NOTAND   Eq. (3), r = DB row
    }
}

template <int BN, int GG>
cudaError_t launch_f(const SearchArgs &a, cudaStream_t s) {
    // the database is the B operand of the user call (Q op D), on TMEM lanes here
    FArgs f{};
    f.Q = a.Q;
    f.nq = a.nq;
    f.ldq32 = a.ldq32;
    f.nd = a.nd;
    f.popDg = a.popD;
    f.nbits = a.nbits;
    f.nops = a.nops;
    f.accumulate = a.accumulate;
    f.ldo = a.ldo;
    for (int j = 0; j < a.nops; ++j) {
        op_coefs(a.ops[j], f.cq[j], f.cd[j], f.cc[j]);
        f.outs[j] = a.counts[j];
        if (a.best_count[j]) {
            f.best_mask |= 1 << j;
            f.best_count[j] = a.best_count[j];
            f.best_index[j] = a.best_index[j];
        }
    }
    f.keys = a.keys;
    f.done = a.done;
    f.index_base = a.index_base;
    f.ntiles = (a.nd + BM - 1) / BM;
    f.nst = (int)((a.nbits + KBITS - 1) / KBITS);
    f.qbytes = (size_t)BN * f.nst * (KBITS / 32) * 16;
#ifdef SNP_PROFILING
    static const bool trace = std::getenv("SNP_TRACE") && std::getenv("SNP_TRACE")[0] == '1';
    f.trace = trace ? 1 : 0;
    static const bool nostore = std::getenv("SNP_DEBUG_NOSTORE") && std::getenv("SNP_DEBUG_NOSTORE")[0] == '1';
    f.nostore = nostore ? 1 : 0;
#endif
    const size_t smem = smem_bytes(BN, a.nbits);

    CUtensorMap tm;
    if (!make_map_u32_2d(&tm, a.D, a.nd, a.ldd32, KBITS / 32, BM,
                         KBITS == 1024 ? CU_TENSOR_MAP_SWIZZLE_128B
                         : KBITS == 512 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B, a.dcols32))
        return cudaErrorInvalidValue;

    using KernFn = void (*)(const CUtensorMap, const FArgs);
    const bool best = f.best_mask != 0;
    KernFn kern = nullptr;
    int nthreads = Roles<GG>::NTHREADS;   // the runtime-coefficient kernels are GG = 4 only
    if (a.accumulate) {   // K-chunked searches add each chunk's counts (one or two ops per pass)
        nthreads = Roles<4>::NTHREADS;
        if (a.nops > 2 || best) return cudaErrorInvalidValue;
        kern = a.nops == 1 ? fastid_tc4_kernel<BN, 1, false, true, -1, 4> : fastid_tc4_kernel<BN, 2, false, true, -1, 4>;
    } else if (a.nops == 1) {   // compile-time op
        static KernFn k1[2][4] = {{fastid_tc4_kernel<BN, 1, false, false, 0, GG>, fastid_tc4_kernel<BN, 1, false, false, 1, GG>,
                                   fastid_tc4_kernel<BN, 1, false, false, 2, GG>, fastid_tc4_kernel<BN, 1, false, false, 3, GG>},
                                  {fastid_tc4_kernel<BN, 1, true, false, 0, GG>, fastid_tc4_kernel<BN, 1, true, false, 1, GG>,
                                   fastid_tc4_kernel<BN, 1, true, false, 2, GG>, fastid_tc4_kernel<BN, 1, true, false, 3, GG>}};
        kern = k1[best][a.ops[0] & 3];
    } else if (a.nops == 2 && a.ops[0] == 1 && a.ops[1] == 2) {   // XOR + ANDNOT (identity + mixture)
        kern = best ? fastid_tc4_kernel<BN, 2, true, false, 1 | (2 << 2), GG>
                    : fastid_tc4_kernel<BN, 2, false, false, 1 | (2 << 2), GG>;
    } else {
        nthreads = Roles<4>::NTHREADS;
        switch (a.nops * 2 + (best ? 1 : 0)) {
        case 4: kern = fastid_tc4_kernel<BN, 2, false, false, -1, 4>; break;
        case 5: kern = fastid_tc4_kernel<BN, 2, true, false, -1, 4>; break;
        case 6: kern = fastid_tc4_kernel<BN, 3, false, false, -1, 4>; break;
        case 7: kern = fastid_tc4_kernel<BN, 3, true, false, -1, 4>; break;
        case 8: kern = fastid_tc4_kernel<BN, 4, false, false, -1, 4>; break;
        case 9: kern = fastid_tc4_kernel<BN, 4, true, false, -1, 4>; break;
        default: return cudaErrorInvalidValue;
        }
    }
    // grant the whole opt-in once per (device, instantiation): the query batch's size varies per call
    // each TMEM A slot must belong to one expander group (a group waits only for its own
    // previous use of a slot; with more groups than slots an mbarrier phase could alias):
    // instantiations with fewer TMEM stages than groups refuse, and the dispatcher
    // (fastid_tc4.cu) takes the 512-bit-stage instantiation instead
    if (nthreads == Roles<4>::NTHREADS ? !FCfg<BN, 4>::OK : !FCfg<BN, 2>::OK) return cudaErrorNotSupported;
    if (cudaError_t e = ensure_dyn_smem(reinterpret_cast<const void *>(kern), (int)(MAX_SMEM - 1024)); e != cudaSuccess)
        return e;
    const int grid = (int)(f.ntiles < device_sms() ? f.ntiles : device_sms());
    // programmatic dependent launch: the kernel's setup (barriers, TMEM allocation, tensor
    // map prefetch) overlaps the preceding kernel; it waits (griddepcontrol.wait) before
    // touching any data that kernel produces
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3((unsigned)nthreads);
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

}  // namespace

// Shape filter: queries on the column side (<= 128 rows, the user's first operand),
// their whole expanded K range resident in shared memory, exact fp32 range.
// Resident query width: 64 columns while the expanded batch fits in shared memory (up to
// ~6500 SNPs), else 32 (N = 32 MMAs, up to ~9700 SNPs) for batches of <= 32 queries
// (configs[4] sweep: 1..32 queries x 20M x 8192 SNPs took the general kernel + best pass
// at 9-12 ms against a 3.1 ms database read).
int FASTID_FN(fastid_bn)(int64_t m, int64_t nbits) {
    // <= 32 queries: the 32-wide batch (N = 32 MMAs cost the same as N = 64, the epilogue
    // half, and TMEM room for 6 A stages instead of 4)
    if (m <= 32 && smem_bytes(32, nbits) <= MAX_SMEM - 1024) return 32;
    if (m <= 64 && smem_bytes(64, nbits) <= MAX_SMEM - 1024) return 64;
    return 0;
}

bool FASTID_FN(fastid_tc4_supported)(int64_t m, int64_t n, int64_t nbits) {
    // nbits < 2^23: counts leave the fp32 accumulator by the 2^23 magic add
    if (m < 1 || m > 64 || n < 1 || nbits < 1 || nbits >= (1LL << 23)) return false;
    if (n < 4 * m) return false;
    if (n > (int64_t)0x7fffffff - BM) return false;
    return FASTID_FN(fastid_bn)(m, nbits) != 0;
}

cudaError_t FASTID_FN(launch_fastid_tc4)(const GemmArgs &a, int epi, cudaStream_t s) {
    if (epi != EPI_COUNTS) return cudaErrorNotSupported;
    SearchArgs sa{};
    sa.Q = a.A; sa.nq = a.m; sa.ldq32 = a.lda32;
    sa.D = a.B; sa.nd = a.n; sa.ldd32 = a.ldb32;
    sa.popD = a.popB;   // the user's popD (NULL: counted in-kernel)
    sa.nbits = a.nbits;
    sa.nops = 1; sa.ops[0] = a.op; sa.counts[0] = a.C;
    sa.ldo = a.ldc; sa.accumulate = a.accumulate;
    // queries <= 64 (fastid_tc4_supported)
    const bool two = sa.popD || (FASTID_COUNT_GG2 && KBITS == 1024);
    if (FASTID_FN(fastid_bn)(sa.nq, sa.nbits) == 32) return two ? launch_f<32, 2>(sa, s) : launch_f<32, 4>(sa, s);
    return two ? launch_f<64, 2>(sa, s) : launch_f<64, 4>(sa, s);
}

size_t FASTID_FN(fastid_search_tc4_ws_bytes)(int64_t nq, int nops) {
    return (((size_t)nops * nq * 8 + 255) & ~(size_t)255) + 256;
}

cudaError_t FASTID_FN(launch_fastid_search_tc4)(const SearchArgs &a, cudaStream_t s) {
    const bool two = a.popD || (FASTID_COUNT_GG2 && KBITS == 1024);
    if (FASTID_FN(fastid_bn)(a.nq, a.nbits) == 32) return two ? launch_f<32, 2>(a, s) : launch_f<32, 4>(a, s);
    return two ? launch_f<64, 2>(a, s) : launch_f<64, 4>(a, s);
}

}  // namespace snp

#if defined(SNP_PROFILING)
// Profiling aid (not part of include/snp.h): copy the pipeline trace of the last
// traced fastid_tc4 launch (4 x 1024 clock64 stamps) to host memory.  The 512-bit-stage
// instantiation exports the plain names, the 1024-bit one the same names + "_k1024".
#ifdef FASTID_PRIMARY
#define FASTID_DBG(name) name
#else
#define FASTID_DBG(name) name##_k1024
#endif
extern "C" int FASTID_DBG(snp_debug_fastid_launch_times)(long long *host, int n) {
    if (n > 128) n = 128;
    return (int)cudaMemcpyFromSymbol(host, snp::g_fastid_launch_time, sizeof(long long) * n);
}

extern "C" int FASTID_DBG(snp_debug_fastid_cta_times)(long long *host, int n) {
    if (n > 4 * 1024) n = 4 * 1024;
    return (int)cudaMemcpyFromSymbol(host, snp::g_fastid_cta_time, sizeof(long long) * n);
}

extern "C" int FASTID_DBG(snp_debug_fastid_etrace)(long long *host, int n) {
    if (n > 4 * 256) n = 4 * 256;
    return (int)cudaMemcpyFromSymbol(host, snp::g_fastid_etrace, sizeof(long long) * n);
}

extern "C" int FASTID_DBG(snp_debug_fastid_wtrace2)(long long *host, int n) {
    if (n > 32 * 1024) n = 32 * 1024;
    return (int)cudaMemcpyFromSymbol(host, snp::g_fastid_wtrace2, sizeof(long long) * n);
}

extern "C" int FASTID_DBG(snp_debug_fastid_wtrace)(long long *host, int n) {
    if (n > 4 * 1024) n = 4 * 1024;
    return (int)cudaMemcpyFromSymbol(host, snp::g_fastid_wtrace, sizeof(long long) * n);
}

extern "C" int FASTID_DBG(snp_debug_fastid_trace)(long long *host, int n) {
    if (n > 8 * 1024) n = 8 * 1024;
    return (int)cudaMemcpyFromSymbol(host, snp::g_fastid_trace, sizeof(long long) * n);
}
#endif  // SNP_PROFILING
