// snp_internal.h — launcher declarations shared by the library's translation units.
// Not part of the public ABI (that is include/snp.h).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <math.h>

namespace snp {

// Process-wide count of kernels this library launched (snp_launch_count()).
void count_launches(int k);

// runtime.cu — per-device caches (thread-safe): SM count, dynamic shared-memory opt-in per
// (device, kernel), the driver's tensor-map encoder and 2-D uint32 tensor maps for TMA.
int device_sms();
cudaError_t ensure_dyn_smem(const void *kernel, int bytes);
typedef CUresult (*EncodeTiledFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                  const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
EncodeTiledFn tensor_map_encoder();
// cols32 > 0: the rows hold only cols32 words from `base` (a column window of a wider matrix,
// elements past it read as zero); 0: ld32
bool make_map_u32_2d(CUtensorMap *tm, const uint32_t *base, int64_t rows, int64_t ld32, uint32_t box_words,
                     uint32_t box_rows, CUtensorMapSwizzle swizzle, int64_t cols32 = 0);

// Epilogue kinds of the bit-GEMM.
enum Epi : int {
    EPI_COUNTS = 0,   // C = / += counts                       (a3, a4 direct ops)
    EPI_LD = 1        // r2 [, D'] [, counts] from nAB, nA, nB  (a5)
};

// f3 packed triangle (snp_ld_sym): the row-major upper triangle of a T x T grid of
// 128 x 128 tiles, tile t <-> (I, J), I <= J < T, t = start(I) + (J - I) with
// start(I) = I T - I (I - 1) / 2.
constexpr int SYM_TILE = 128;
__host__ __device__ __forceinline__ int64_t tri_start(int64_t T, int64_t I) { return I * T - I * (I - 1) / 2; }
__host__ __device__ __forceinline__ void tri_decode(int64_t T, int64_t t, uint32_t &I, uint32_t &J) {
    const double b = 2.0 * (double)T + 1.0;
    int64_t i = (int64_t)((b - sqrt(b * b - 8.0 * (double)t)) * 0.5);   // estimate, then exact fix-up
    if (i < 0) i = 0;
    if (i > T - 1) i = T - 1;
    while (i > 0 && tri_start(T, i) > t) --i;
    while (i + 1 < T && tri_start(T, i + 1) <= t) ++i;
    I = (uint32_t)i;
    J = (uint32_t)(i + (t - tri_start(T, i)));
}

struct GemmArgs {
    const uint32_t *A;   // [m][lda32] packed rows viewed as uint32 words
    const uint32_t *B;   // [n][ldb32]
    int64_t m, n;
    int64_t lda32, ldb32;
    int64_t nbits;
    int op;              // snp_op
    int accumulate;
    int64_t ldc;
    uint32_t *C;         // counts (EPI_COUNTS: required; EPI_LD: optional)
    float *r2;           // EPI_LD
    float *dprime;       // EPI_LD optional
    const uint32_t *popA;  // EPI_LD (and tensor identities)
    const uint32_t *popB;
    int op2 = 0;           // gemm_tc4, swapped layout (m < n) only: a second op from the same
    uint32_t *C2 = nullptr;  // AND count, written to C2 (NULL: one op)
    // f3 packed triangle (self-LD, A == B, m == n): tri_n >= 0 computes tiles tri_lo ..
    // tri_lo + tri_n - 1 only, tile u of the call stored dense at element u * 128 * 128
    // of C / r2 / dprime (row-major, ldc = 128); no mirror.
    int64_t tri_lo = 0, tri_n = -1;
    // optional scratch for the whole-triangle tensor path: the column operand pre-expanded to
    // e2m1 nibbles (gemm_tc4_bpre_bytes(m, nbits) bytes, 16-byte aligned), nullptr = off
    uint32_t *bpre = nullptr;
};

// CUDA-core LOP3 + POPC variant (bitgemm_popc.cu).
cudaError_t launch_bitgemm_popc(const GemmArgs &a, int epi, cudaStream_t s);

// pack.cu
cudaError_t launch_pack(const uint8_t *g, int64_t rows, int64_t nbits, int64_t ldg,
                        uint64_t *packed, int64_t ldw, cudaStream_t s);
cudaError_t launch_pack_popc(const uint8_t *g, int64_t rows, int64_t nbits, int64_t ldg,
                             uint64_t *packed, int64_t ldw, uint32_t *popc, cudaStream_t s);
cudaError_t launch_row_popc(const uint64_t *x, int64_t rows, int64_t nbits, int64_t ldw,
                            uint32_t *popc, cudaStream_t s);

// sym.cu — f3 packed triangle -> full symmetric matrix (4-byte elements).
cudaError_t launch_sym_unpack(const uint32_t *tiles, int64_t m, int64_t tlo, int64_t ntiles, uint32_t *out,
                              int64_t ldo, cudaStream_t s);

// best.cu — scratch is best_index reinterpreted as packed (count<<32 | j) keys.
cudaError_t launch_best(const uint32_t *counts, int64_t nq, int64_t nd, int64_t ldo,
                        int64_t index_base, uint32_t *best_count, int64_t *best_index,
                        cudaStream_t s);

// f1 fused FastID search (snp_fastid_search): one pass over the database, up to 4 ops
// derived from one AND count, each with optional counts and optional best match.
struct SearchArgs {
    const uint32_t *Q;   // [nq][ldq32] queries, packed u32 view
    int64_t nq, ldq32;
    const uint32_t *D;   // [nd][ldd32] database
    int64_t nd, ldd32;
    int64_t dcols32 = 0; // > 0: D is a column window of dcols32 words (K-chunked searches)
    const uint32_t *popD;     // [nd] database row popcounts or NULL (derived in-kernel)
    int64_t nbits;
    int nops;
    int ops[4];
    uint32_t *counts[4];      // per op [nq][ldo] or NULL
    int64_t ldo;
    int accumulate;
    uint32_t *best_count[4];  // per op [nq] or NULL (then best_index[j] is NULL too)
    int64_t *best_index[4];
    int64_t index_base;
    unsigned long long *keys; // workspace: [nops][nq] merge keys
    unsigned int *done;       // workspace: CTA completion counter
};

// Tensor-core tcgen05 variant (bitgemm_tc.cu).  ws: expanded operands.
size_t tc_workspace_bytes(int64_t m, int64_t n, int64_t nbits);
bool tc_supported(int64_t m, int64_t n, int64_t nbits);
cudaError_t launch_bitgemm_tc(const GemmArgs &a, int epi, void *ws, size_t ws_bytes,
                              cudaStream_t s);


// General tcgen05 mxf4 kernel (gemm_tc4.cu): 128x128 tiles, TMA-fed, A in TMEM.
size_t gemm_tc4_bpre_bytes(int64_t m, int64_t nbits);
bool gemm_tc4_supported(int64_t m, int64_t n, int64_t nbits);
cudaError_t launch_gemm_tc4(const GemmArgs &a, int epi, cudaStream_t s);
// Whether the most recent launch_gemm_tc4 on this thread ran the symmetric (f3) schedule.
bool gemm_tc4_last_sym();
bool gemm_tc4_last_pair();   // the last launch_gemm_tc4 of this thread ran the CTA-pair kernel

// FastID-shaped tcgen05 mxf4 kernel (fastid_tc4.cu): <= 128 queries resident in shared
// memory, database streamed by TMA.  The queries are the user's first operand.
bool fastid_tc4_supported(int64_t m, int64_t n, int64_t nbits);
int fastid_bn(int64_t m, int64_t nbits);   // resident query width (64, 32) or 0
cudaError_t launch_fastid_tc4(const GemmArgs &a, int epi, cudaStream_t s);
size_t fastid_search_tc4_ws_bytes(int64_t nq, int nops);
cudaError_t launch_fastid_search_tc4(const SearchArgs &a, cudaStream_t s);

// CUDA-core streaming FastID kernel for nq <= 4 (fastid_stream.cu): database TMA-streamed,
// LOP3 + POPC per word and query, counts and best matches of up to 4 ops in one pass.
bool fastid_stream_supported(int64_t nq, int64_t nd, int64_t nbits);
size_t fastid_stream_ws_bytes(int64_t nq, int nops);
cudaError_t launch_fastid_stream(const SearchArgs &a, cudaStream_t s);

// threshold.cu — f1 threshold form: (query, count, global index) of every count <= tau.
struct ThresholdMatch {
    uint32_t query;
    uint32_t count;
    int64_t index;
};
cudaError_t launch_threshold_compact(const uint32_t *counts, int64_t nq, int64_t rows, int64_t ldo, int64_t index0,
                                     uint32_t tau, ThresholdMatch *out, int64_t capacity, unsigned long long *total,
                                     cudaStream_t s);

// best.cu building blocks for the chunked search path: keys (count << 32 | j) are
// initialised to ~0, min-merged per count block (j offset by jbase), then finalised.
cudaError_t launch_best_init(unsigned long long *keys, int64_t n, cudaStream_t s);
cudaError_t launch_best_reduce(const uint32_t *counts, int64_t nq, int64_t nd, int64_t ldo, int64_t jbase,
                               unsigned long long *keys, cudaStream_t s);
cudaError_t launch_best_finalize(const unsigned long long *keys, int64_t nq, int64_t index_base,
                                 uint32_t *best_count, int64_t *best_index, cudaStream_t s);

}  // namespace snp
