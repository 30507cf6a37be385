/*
 * snp.h — C ABI of the B200-native SNP-comparison library (libsnp.so).
 *
 * The library computes the one data-parallel hot path of Binder, Low & Popovici,
 * "A Portable GPU Framework for SNP Comparisons" (IPDPS-W 2019): SNP comparison
 * cast as a binary matrix product (§II.A, §III)
 *
 *     C[i][j] = sum_w POPC( A[i][w]  op  B[j][w] )
 *
 * over bit-packed genotype rows, with op = AND (LD, Eq. 1),
 * XOR (FastID identity search, Eq. 2) or AND-NOT (FastID mixture
 * analysis, Eq. 3 rewritten as r & ~m).  P:Lnn is a line of the
 * paper text.
 *
 * Conventions shared by every call
 * --------------------------------
 *  - Packed layout (§III, Fig. 2): row r of a packed matrix is `ld`
 *    consecutive little-endian uint64 words; sample/SNP k of the row is bit
 *    (k % 64) of word (k / 64) (LSB first).  Bits >= nbits are IGNORED by every
 *    compute call (the kernels mask them), so padding contents never matter;
 *    snp_pack writes them as zero.  LD matrices pack along samples (rows are
 *    SNPs); FastID matrices pack along SNPs (rows are profiles).  Both operands
 *    are therefore K-contiguous and C = A . B^T.
 *  - Pointers are CUDA DEVICE pointers unless marked (host).  Matrix pointers
 *    must be 16-byte aligned and every leading dimension of a packed matrix
 *    (in uint64 words) must be even (128-bit rows), else SNP_E_ALIGN.
 *  - Every compute call is asynchronous and stream-ordered on `stream` (a
 *    cudaStream_t passed as void*; NULL = legacy default stream).  The library
 *    allocates no device memory: the caller owns every buffer, including the
 *    workspace `ws` sized by the *_workspace_bytes queries.  No pointer is kept
 *    after the call returns.
 *  - Arguments are validated synchronously before any launch; an invalid call
 *    launches nothing.  Device faults surface at the caller's next sync.
 *  - m == 0 or n == 0 is a valid no-op returning SNP_OK.
 *  - Outputs must not alias inputs.  B == A (self-LD) is allowed.
 *  - The library runs only on compute capability 10.0 (B200, sm_100a); any
 *    other device returns SNP_E_ARCH.  There is no fallback.
 *  - Calls are re-entrant and thread-safe.  Process-wide state: per-device caches
 *    (SM count, the dynamic shared-memory opt-in of each kernel, the driver's
 *    tensor-map encoder; keyed by device, guarded by atomics / a mutex) and the
 *    variant override of snp_set_variant.  Profiling hooks (pipeline traces, the
 *    snp_debug_* readers) exist only in -DSNP_PROFILING builds, not in libsnp.so.
 */
#ifndef SNP_H_
#define SNP_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    SNP_OK = 0,
    SNP_E_NULL = 1,      /* a required pointer is NULL                          */
    SNP_E_SHAPE = 2,     /* negative size, ld < ceil(nbits/64), ldc < n, nbits<1 */
    SNP_E_ALIGN = 3,     /* pointer not 16-byte aligned or odd packed ld        */
    SNP_E_OP = 4,        /* unknown snp_op / snp_variant                        */
    SNP_E_RANGE = 5,     /* nbits too large for uint32 counts, bad shard args   */
    SNP_E_WORKSPACE = 6, /* ws smaller than the workspace query returned        */
    SNP_E_ARCH = 7,      /* current device is not compute capability 10.0      */
    SNP_E_CUDA = 8       /* a CUDA runtime/launch error (see snp_last_cuda_error) */
} snp_status;

/* Bitwise comparison applied per word before POPC.  Q is the first operand
 * (query / A rows), D the second (database / B rows). */
typedef enum {
    SNP_OP_AND = 0,    /* popc(Q & D)   Eq. (1), P:L52 (LD p_AB term)                */
    SNP_OP_XOR = 1,    /* popc(Q ^ D)   Eq. (2), P:L60 (identity search, 0 = match)  */
    SNP_OP_ANDNOT = 2, /* popc(Q & ~D)  Eq. (3) with r = query, m = database row
                          ("m ... negated and stored in the database")      */
    SNP_OP_NOTAND = 3  /* popc(~Q & D)  Eq. (3) with r = database row, m = query     */
} snp_op;

/* Kernel variant selection (process-wide; default SNP_VARIANT_AUTO). */
typedef enum {
    SNP_VARIANT_AUTO = 0, /* pick per shape from the measured dispatch table    */
    SNP_VARIANT_POPC = 1, /* CUDA-core LOP3 + POPC register-blocked bit-GEMM     */
    SNP_VARIANT_TC = 2    /* tcgen05 tensor-core GEMM on bit-expanded operands: kind::mxf4
                             (bits as e2m1 nibbles, fp32 TMEM sums, exact for nbits < 2^24)
                             and kind::i8 (u8 bits, s32 sums) from nbits = 2^24 up          */
} snp_variant;

/* Recommended packed leading dimension (uint64 words) for nbits bits:
 * ceil(nbits/64) rounded up to a multiple of 8 (64-byte rows).  Any even
 * ld >= ceil(nbits/64) is accepted.  Returns 0 for nbits <= 0. */
int64_t snp_words(int64_t nbits);

/* Bytes of device workspace snp_ld_counts / snp_ld_r2 need for this shape
 * under the current variant choice (0 if none).  ws may be NULL when 0. */
size_t snp_ld_workspace_bytes(int64_t m, int64_t n, int64_t nbits);

/* Bytes of device workspace snp_fastid needs (0 if none). */
size_t snp_fastid_workspace_bytes(int64_t nq, int64_t nd, int64_t nbits, int op);

/* a1 — encode + pack (§III, Fig. 2).  g: uint8 genotypes [rows][ldg_bytes],
 * byte k of row r is sample/SNP k (non-zero = minor allele = 1, zero = major = 0).
 * packed: uint64 [rows][ldw] output; bits >= nbits and words >= ceil(nbits/64)
 * are written as 0.  g has no alignment requirement; ldg_bytes >= nbits. */
snp_status snp_pack(const uint8_t *g, int64_t rows, int64_t nbits, int64_t ldg_bytes,
                    uint64_t *packed, int64_t ldw, void *stream);

/* a1 + a2 fused — snp_pack followed by snp_row_popc in one pass over g (same
 * arguments, layout and errors as snp_pack; popc: uint32 [rows], popc[r] = set bits
 * of packed row r, the p_A / p_B of P:L44 as counts; NULL -> SNP_E_NULL). */
snp_status snp_pack_popc(const uint8_t *g, int64_t rows, int64_t nbits, int64_t ldg_bytes,
                         uint64_t *packed, int64_t ldw, uint32_t *popc, void *stream);

/* a2 — popc[r] = number of set bits among the first nbits of packed row r
 * (p_A / p_B of P:L44 as counts). */
snp_status snp_row_popc(const uint64_t *x, int64_t rows, int64_t nbits, int64_t ldw,
                        uint32_t *popc, void *stream);

/* a3 — LD counts (Eq. 1; GEMM update P:L116):
 *   C[i*ldc + j] (=|+=) sum_k A_ik & B_jk,   i < m, j < n, k < nbits.
 * A: [m][lda] packed SNP rows over samples, B: [n][ldb].  C: uint32 [m][ldc].
 * accumulate = 0 overwrites C, 1 adds (callers may split K into chunks). */
snp_status snp_ld_counts(const uint64_t *A, int64_t m, int64_t lda,
                         const uint64_t *B, int64_t n, int64_t ldb, int64_t nbits,
                         uint32_t *C, int64_t ldc, int accumulate,
                         void *ws, size_t ws_bytes, void *stream);

/* a3 + a5 — LD statistics for every SNP pair, n = nbits samples:
 *   num = n*nAB - nA*nB (= n^2 D_AB, exact), den = nA(n-nA) nB(n-nB),
 *   r2 = num^2/den (0 when den == 0, i.e. a monomorphic SNP),
 *   D' = num/Dmax, Dmax = min(nA(n-nB),(n-nA)nB) if num>0 else min(nA nB,(n-nA)(n-nB))
 *   (0 when num == 0).  num, den and Dmax are exact integers (int32 for n <= 46340, int64
 *   above); the tensor-core epilogue forms r2 and D' from them in fp32: r2 with at most 9
 *   roundings (relative error <= 9 * 2^-24 = 5.4e-7), D' with one correctly rounded
 *   division of two once-rounded integers (<= 3 * 2^-24), stored fp32; exactly 0 where
 *   the exact value is 0.  The CUDA-core variant computes them in fp64.  Both are within
 *   the 1e-6 relative bar of the fp64 oracle (north_star).
 * popA/popB: optional precomputed row popcounts (NULL = computed internally).
 * r2: float [m][ldc] (required); dprime: float [m][ldc] or NULL;
 * counts: uint32 nAB [m][ldc] or NULL. */
snp_status snp_ld_r2(const uint64_t *A, int64_t m, int64_t lda, const uint32_t *popA,
                     const uint64_t *B, int64_t n, int64_t ldb, const uint32_t *popB,
                     int64_t nbits, float *r2, float *dprime, uint32_t *counts,
                     int64_t ldc, void *ws, size_t ws_bytes, void *stream);

/* f3 — symmetric self-LD in the packed upper-triangle tile layout (LD is
 * a GEMM of one SNP matrix with itself, §II.A and Fig. 1, so C = C^T and half the
 * products are redundant).  The m x m output is cut into 128 x 128 tiles, T = ceil(m/128)
 * per side; tile t <-> (I, J), I <= J < T, in row-major upper-triangle order
 *     t = start(I) + (J - I),   start(I) = I*T - I*(I-1)/2,   snp_sym_tiles(m) = T(T+1)/2.
 * A call computes tiles tile_lo .. tile_hi-1 only (one rank's share of
 * snp_shard_plan_sym) and stores tile t as a dense row-major 128 x 128 block at element
 * offset (t - tile_lo) * 16384 of each output: element (i, j) of the block is the pair
 * (SNP 128 I + i, SNP 128 J + j).  Entries of a ragged last tile row/column (index >= m)
 * are not written.  Diagonal tiles hold both triangles of their block; the full matrix is
 * the tiles plus their mirror images (snp_sym_unpack).  Statistics as snp_ld_r2 (same
 * integers, same fp32 epilogue and bound).
 *   A: [m][lda] packed SNP rows over n = nbits samples.  popA: optional row popcounts.
 *   r2, dprime (nullable; dprime needs r2), counts (nullable): [tile_hi - tile_lo][128][128]
 *   float / float / uint32; at least one of r2, counts.  r2 == NULL gives nAB counts only.
 *   ws: snp_ld_sym_workspace_bytes(m, nbits) bytes when r2 != NULL and popA == NULL.
 * SNP_E_RANGE for tile_lo < 0, tile_hi < tile_lo or tile_hi > snp_sym_tiles(m).
 * Kernels: tcgen05 kind::mxf4 (nbits < 2^24) or the CUDA-core variant (forced, or above). */
int64_t snp_sym_tiles(int64_t m);
size_t snp_ld_sym_workspace_bytes(int64_t m, int64_t nbits);
snp_status snp_ld_sym(const uint64_t *A, int64_t m, int64_t lda, const uint32_t *popA, int64_t nbits,
                      int64_t tile_lo, int64_t tile_hi, float *r2, float *dprime, uint32_t *counts,
                      void *ws, size_t ws_bytes, void *stream);

/* f3 — scatter packed-triangle tiles tile_lo .. tile_hi-1 (4-byte elements: counts, r2 or
 * D' viewed as uint32) into the full row-major m x m matrix out[m][ldo] (ldo >= m): block
 * (I, J) and, for I != J, its transpose at (J, I).  Elements of tiles outside the range are
 * not written.  HBM-bound copy kernel. */
snp_status snp_sym_unpack(const uint32_t *tiles, int64_t m, int64_t tile_lo, int64_t tile_hi, uint32_t *out,
                          int64_t ldo, void *stream);

/* a3 + a4 — FastID comparison counts (Eqs. 2-3):
 *   out[i*ldo + j] (=|+=) sum_k op(Q_ik, D_jk)   for queries i < nq, DB rows j < nd.
 * Q: [nq][ldq] packed query profiles over SNPs, D: [nd][ldd] database profiles.
 * popQ/popD: optional exact row popcounts over nbits (snp_row_popc); may be NULL.
 * The tensor-core kernels need them for the identities XOR = pQ + pD - 2 AND,
 * ANDNOT = pQ - AND, NOTAND = pD - AND: given ones are read as they are (the FastID
 * kernel then skips counting the streamed database words), NULL ones are derived
 * in-kernel from the packed words or by a pre-pass.  The CUDA-core variant ignores
 * them (one LOP3 per op).
 * out: uint32 [nq][ldo], ldo >= nd. */
snp_status snp_fastid(const uint64_t *Q, int64_t nq, int64_t ldq, const uint32_t *popQ,
                      const uint64_t *D, int64_t nd, int64_t ldd, const uint32_t *popD,
                      int64_t nbits, int op, uint32_t *out, int64_t ldo, int accumulate,
                      void *ws, size_t ws_bytes, void *stream);

/* a6 — best match per query over a count matrix ("No set bits ...
 * signifies a positive match"; P:L62 larger = less likely):
 *   best_count[i] = min_j counts[i*ldo + j],
 *   best_index[i] = index_base + (lowest j attaining it); nd == 0 gives
 *   best_count = 0xFFFFFFFF, best_index = -1.  nd < 2^32. */
snp_status snp_fastid_best(const uint32_t *counts, int64_t nq, int64_t nd, int64_t ldo,
                           int64_t index_base, uint32_t *best_count, int64_t *best_index,
                           void *stream);

/* f1 — fused FastID search (P:L54-78 for the ops, P:L58/L62 for the
 * decision): ONE pass over the database computes, for each of the nops (1..4) ops in
 * ops[] (a HOST array of snp_op), the count matrix of snp_fastid and/or the per-query
 * best match of snp_fastid_best, without the counts being re-read (or written at all
 * when only best matches are wanted).  All ops derive from the one AND count of a
 * (query, row) pair, so XOR and ANDNOT together cost one database pass, not two.
 *   counts:     HOST array of nops device pointers (or NULL = none); counts[j] is
 *               uint32 [nq][ldo] for ops[j] as in snp_fastid (overwritten), or NULL.
 *   best_count, best_index: HOST arrays of nops device pointers (both arrays NULL =
 *               no best matches); entry j is uint32 [nq] / int64 [nq] (both NULL or
 *               both set): min count over the nd rows and index_base + lowest row
 *               attaining it (R4); nd == 0 gives 0xFFFFFFFF / -1.
 *   popD:       uint32 [nd] database row popcounts over nbits (snp_row_popc), or NULL.
 *               A database is resident and prepared once, so its popcounts
 *               can be too; given, the kernel skips counting every streamed word.
 *               They must be exact: wrong popcounts give wrong XOR/ANDNOT/NOTAND counts.
 * nd < 2^32 - 1.  ws: snp_fastid_search_workspace_bytes(nq, nd, nbits, nops) bytes
 * (never 0 when nq > 0), ZERO-FILLED before its first use by this call (e.g. one
 * cudaMemsetAsync after allocating it); every call leaves it zero-filled again when it
 * completes (the fused kernels merge best matches into it without an init launch and the
 * last CTA clears it, as a CUTLASS split-K semaphore workspace is), so a workspace is
 * cleared once and reused for any number of calls.  A workspace must not be shared by
 * calls that may run concurrently.  Kernels: the fused tcgen05 kernel for nq <= 64 (one
 * launch, + the caller's query pack); other shapes / a forced SNP_VARIANT_POPC compose
 * snp_fastid's kernels with best.cu per op, chunking the database through workspace
 * counts when counts[j] is NULL. */
size_t snp_fastid_search_workspace_bytes(int64_t nq, int64_t nd, int64_t nbits, int nops);
snp_status snp_fastid_search(const uint64_t *Q, int64_t nq, int64_t ldq,
                             const uint64_t *D, int64_t nd, int64_t ldd, const uint32_t *popD,
                             int64_t nbits,
                             int nops, const int *ops, uint32_t *const *counts, int64_t ldo,
                             uint32_t *const *best_count, int64_t *const *best_index,
                             int64_t index_base, void *ws, size_t ws_bytes, void *stream);

/* f1, threshold form — every (query, database row) pair with count <= tau for op (the
 * forensic decision of P:L58 "no set bits in the result signifies a positive match", with a
 * tolerance: tau = 0 lists exact matches; P:L62 larger counts are less likely).
 *   matches:     device array of `capacity` snp_match (16-byte aligned); the first `capacity`
 *                matches found are stored, in UNSPECIFIED order (the set is exact).
 *   match_count: device uint64 (8-byte aligned), set to the TOTAL number of matches (it may
 *                exceed capacity: the caller can re-run with a larger list).
 *   index:       index_base + database row.
 * The database is processed in row chunks through workspace counts
 * (snp_fastid_threshold_workspace_bytes), each chunk by snp_fastid's kernels and one
 * compaction pass.  nq <= 65535; SNP_E_NULL for a NULL match_count (or matches with
 * capacity > 0). */
typedef struct {
    uint32_t query;   /* query row                          */
    uint32_t count;   /* popc(Q_query op D_row) <= tau       */
    int64_t index;    /* index_base + database row           */
} snp_match;
size_t snp_fastid_threshold_workspace_bytes(int64_t nq, int64_t nd, int64_t nbits, int op);
snp_status snp_fastid_threshold(const uint64_t *Q, int64_t nq, int64_t ldq, const uint64_t *D, int64_t nd,
                                int64_t ldd, const uint32_t *popD, int64_t nbits, int op, uint32_t tau,
                                int64_t index_base, snp_match *matches, int64_t capacity, uint64_t *match_count,
                                void *ws, size_t ws_bytes, void *stream);

/* e — multi-GPU row partition (host only, no device access): rows [0, rows)
 * split into `world` contiguous ranges bounds[r] .. bounds[r+1] (bounds is a
 * HOST array of world+1 int64), each boundary a multiple of `align` (except
 * bounds clamped to rows), block counts balanced to within one.  Deterministic.
 * SNP_E_RANGE for world < 1, align < 1 or rows < 0. */
snp_status snp_shard_plan(int64_t rows, int world, int64_t align, int64_t *bounds);

/* e + f3 — triangle-area-balanced partition of the symmetric self-LD work (host only):
 * the snp_sym_tiles(m) equal-cost tiles of snp_ld_sym split into `world` contiguous ranges
 * tile_bounds[r] .. tile_bounds[r+1] (HOST array of world+1), tile_bounds[r] =
 * floor(r * total / world): every rank gets floor or ceil of total/world tiles (balanced
 * within one tile), no tile is computed twice and no exchange of mirrored blocks is needed.
 * SNP_E_RANGE for world < 1 or m < 0. */
snp_status snp_shard_plan_sym(int64_t m, int world, int64_t *tile_bounds);

/* Variant override (SNP_VARIANT_AUTO restores the dispatch table).  The
 * environment variable SNP_FORCE_VARIANT=popc|tc sets the initial value.
 * Other environment variables only steer the kernel CHOICE for A/B measurements (never the
 * results): SNP_FASTID_STREAM=0 (no CUDA-core streaming kernel), SNP_FASTID_KBITS=512|1024
 * (FastID tensor-kernel stage size), SNP_SEARCH_KCHUNK=0 / SNP_SEARCH_SLICES=0 (no K-chunked
 * or query-sliced searches), SNP_FASTID_KERNEL=0, SNP_TC_KIND=i8, SNP_GEMM_SYM=0,
 * SNP_GEMM_ORDER=0|1|2, SNP_GEMM_X2=1; SNP_SEARCH_CHUNK_ROWS sets the workspace row-chunk size
 * (tests).  Each is covered by the parity tests. */
snp_status snp_set_variant(int variant);
/* Variant used by the most recent successful compute call on this thread. */
int snp_last_variant(void);

/* Kernel family behind that variant (evidence for benchmarks and tests). */
typedef enum {
    SNP_KERNEL_NONE = 0,
    SNP_KERNEL_POPC = 1,        /* CUDA-core LOP3 + POPC                          */
    SNP_KERNEL_TC_I8 = 2,       /* tcgen05 kind::i8 on u8-expanded operands        */
    SNP_KERNEL_TC_MXF4 = 3,     /* tcgen05 kind::mxf4 on e2m1-expanded operands    */
    SNP_KERNEL_FASTID_MXF4 = 4, /* kind::mxf4, resident queries, TMA-streamed DB   */
    SNP_KERNEL_TC_MXF4_SYM = 5, /* kind::mxf4 self-LD, upper-triangle tiles + mirror (f3):
                                   executes about half of the M*N*nbits comparisons */
    SNP_KERNEL_POPC_STREAM = 6, /* CUDA-core FastID for nq <= 4: TMA-streamed database,
                                   LOP3 + POPC, all ops and best matches in one pass   */
    SNP_KERNEL_TC_MXF4_SYM_PAIR = 7, /* the whole f3 triangle on CTA pairs (tcgen05
                                   cta_group::2, M = 256 pair tiles; snp_ld_sym)       */
    SNP_KERNEL_TC_MXF4_PAIR = 8 /* kind::mxf4 on CTA pairs, general layout (opt-in)    */
} snp_kernel;
int snp_last_kernel(void);

/* Cumulative number of CUDA kernels this library has launched in this process
 * (evidence for benchmarks: every launch is one of the library's own kernels). */
int64_t snp_launch_count(void);

/* Static description of a status code. */
const char *snp_status_string(int status);
/* Text of the last CUDA error seen by a call on this thread ("" if none). */
const char *snp_last_cuda_error(void);

#ifdef __cplusplus
}
#endif
#endif /* SNP_H_ */
