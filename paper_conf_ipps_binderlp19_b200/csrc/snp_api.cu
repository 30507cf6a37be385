// snp_api.cu — the C ABI (include/snp.h): validation, architecture check, variant
// dispatch and launches.  Every entry point validates synchronously before any
// launch and never allocates device memory.
#include "../../include/snp.h"
#include "snp_internal.h"

#include <atomic>
#include <cstdio>
#include <cstdlib>
#include <cstring>

using namespace snp;


namespace {

thread_local char g_cuda_err[256] = "";
thread_local int g_last_variant = 0;
thread_local int g_last_kernel = 0;

std::atomic<int> g_variant{-1};   // -1: not yet read from the environment
std::atomic<long long> g_launches{0};

int current_variant() {
    int v = g_variant.load(std::memory_order_relaxed);
    if (v < 0) {
        int init = SNP_VARIANT_AUTO;
        const char *e = std::getenv("SNP_FORCE_VARIANT");
        if (e) {
            if (!std::strcmp(e, "popc")) init = SNP_VARIANT_POPC;
            else if (!std::strcmp(e, "tc")) init = SNP_VARIANT_TC;
        }
        int expected = -1;
        g_variant.compare_exchange_strong(expected, init);
        v = g_variant.load();
    }
    return v;
}

// Per-device compute-capability cache (the only other process-wide state).
std::atomic<int> g_cc[128];

snp_status set_cuda_error(cudaError_t e) {
    std::snprintf(g_cuda_err, sizeof(g_cuda_err), "%s: %s", cudaGetErrorName(e),
                  cudaGetErrorString(e));
    return SNP_E_CUDA;
}

snp_status check_arch() {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) {
        set_cuda_error(e);
        cudaGetLastError();
        return SNP_E_ARCH;
    }
    if (dev < 0 || dev >= 128) return SNP_E_ARCH;
    int cc = g_cc[dev].load(std::memory_order_relaxed);
    if (cc == 0) {
        int major = 0, minor = 0;
        if (cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev) != cudaSuccess ||
            cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev) != cudaSuccess) {
            cudaGetLastError();
            return SNP_E_ARCH;
        }
        cc = major * 10 + minor;
        g_cc[dev].store(cc);
    }
    return cc == 100 ? SNP_OK : SNP_E_ARCH;
}

inline bool aligned16(const void *p) { return ((uintptr_t)p & 15u) == 0; }
inline int64_t words_needed(int64_t nbits) { return (nbits + 63) / 64; }
inline size_t align256(size_t x) { return (x + 255) & ~(size_t)255; }

// Validation of one packed operand.
snp_status check_packed(const void *p, int64_t rows, int64_t ld, int64_t nbits) {
    if (rows < 0 || ld < 0) return SNP_E_SHAPE;
    if (rows == 0) return SNP_OK;
    if (!p) return SNP_E_NULL;
    if (ld < words_needed(nbits)) return SNP_E_SHAPE;
    if (!aligned16(p) || (ld & 1)) return SNP_E_ALIGN;
    return SNP_OK;
}

snp_status check_nbits(int64_t nbits) {
    if (nbits < 1) return SNP_E_SHAPE;
    if (nbits > 0x7fffffffLL) return SNP_E_RANGE;   // counts are uint32; LD math int64
    return SNP_OK;
}

// Some tensor-core kernel serves the shape: the persistent kind::mxf4 kernels (any m, n below
// 2^31 rows, nbits < 2^24) or the kind::i8 kernel (its grid bounds the smaller dimension).
bool tc_any_supported(int64_t m, int64_t n, int64_t nbits) {
    return fastid_tc4_supported(m, n, nbits) || gemm_tc4_supported(m, n, nbits) || tc_supported(m, n, nbits);
}

// Variant choice per shape (a7).  Measured dispatch: the tensor-core variant wins
// whenever it supports the shape (>= 15x the POPC roof); the POPC
// variant covers everything else and is kept as the forced/reference variant.
int choose_variant(int64_t m, int64_t n, int64_t nbits) {
    const int v = current_variant();
    if (v == SNP_VARIANT_POPC) return SNP_VARIANT_POPC;
    if (v == SNP_VARIANT_TC) return SNP_VARIANT_TC;
    return tc_any_supported(m, n, nbits) ? SNP_VARIANT_TC : SNP_VARIANT_POPC;
}

// a7: the CUDA-core streaming kernel serves the few-query FastID shapes in AUTO from the
// measured configs[4] sweep (profiles/round2/head/sweep/sweep_few.txt, after the tensor kernel's
// per-stage MMA issue): 1-2 queries everywhere; 3 queries only for profiles above 12,288 SNPs
// (3 x 20M x 16384: 8.2 vs 11.3 ms; 3 x 20M x 4096: tensor 2.14 vs 2.25 ms).  Any nq <= 4
// when the CUDA-core variant is forced.
bool use_stream(int64_t nq, int64_t nd, int64_t nbits) {
    const char *e = std::getenv("SNP_FASTID_STREAM");   // "0": never (A/B measurement hook)
    if (e && e[0] == '0') return false;
    if (!fastid_stream_supported(nq, nd, nbits)) return false;
    const int v = current_variant();
    if (v == SNP_VARIANT_POPC) return true;
    if (v == SNP_VARIANT_TC) return false;
    return nq <= 2 || (nq == 3 && nbits > 12288);
}

size_t pops_bytes(int64_t m, int64_t n) { return align256((size_t)m * 4) + align256((size_t)n * 4); }

// Which tensor-core kernel serves a shape (mirrors run_gemm's choice).
int tc_kernel_for(int64_t m, int64_t n, int64_t nbits, int epi) {
    const char *kind = std::getenv("SNP_TC_KIND");
    const bool want_i8 = kind && !std::strcmp(kind, "i8");
    const char *ff = std::getenv("SNP_FASTID_KERNEL");
    const bool no_fastid = ff && !std::strcmp(ff, "0");
    if (!want_i8 && !no_fastid && epi == EPI_COUNTS && fastid_tc4_supported(m, n, nbits)) return SNP_KERNEL_FASTID_MXF4;
    if (!want_i8 && gemm_tc4_supported(m, n, nbits)) return SNP_KERNEL_TC_MXF4;
    return SNP_KERNEL_TC_I8;
}

// ws layout: [popA: align256(4m)][popB: align256(4n)][kernel scratch]
snp_status run_gemm(GemmArgs &a, int epi, int variant, void *ws, size_t ws_bytes, cudaStream_t s) {
    cudaError_t e;
    if (variant == SNP_VARIANT_TC) {
        if (!tc_any_supported(a.m, a.n, a.nbits)) return SNP_E_SHAPE;
        // kind::mxf4 (2x the int8 rate, half the expanded bytes) unless K is too long
        // for exact fp32 accumulation or SNP_TC_KIND=i8 asks for the int8 kernel.
        const int kern = tc_kernel_for(a.m, a.n, a.nbits, epi);
        if (kern == SNP_KERNEL_FASTID_MXF4) {
            e = launch_fastid_tc4(a, epi, s);   // derives popcounts from the streamed words
        } else if (kern == SNP_KERNEL_TC_MXF4) {
            if (epi == EPI_LD || a.op != SNP_OP_AND || (a.C2 && a.op2 != SNP_OP_AND)) {
                // the general kernel reads row popcounts: cheap pre-pass if not given
                if (ws_bytes < pops_bytes(a.m, a.n) || !ws) return SNP_E_WORKSPACE;
                uint32_t *pa = reinterpret_cast<uint32_t *>(ws);
                uint32_t *pb = reinterpret_cast<uint32_t *>((char *)ws + align256((size_t)a.m * 4));
                const uint64_t *A64 = reinterpret_cast<const uint64_t *>(a.A);
                const uint64_t *B64 = reinterpret_cast<const uint64_t *>(a.B);
                if (!a.popA) {
                    if ((e = launch_row_popc(A64, a.m, a.nbits, a.lda32 / 2, pa, s)) != cudaSuccess) return set_cuda_error(e);
                    a.popA = pa;
                }
                if (!a.popB) {
                    if (a.B == a.A && a.n == a.m && a.ldb32 == a.lda32) {
                        a.popB = a.popA;   // self-LD (B aliases A): one popcount pass
                    } else {
                        if ((e = launch_row_popc(B64, a.n, a.nbits, a.ldb32 / 2, pb, s)) != cudaSuccess)
                            return set_cuda_error(e);
                        a.popB = pb;
                    }
                }
            }
            e = launch_gemm_tc4(a, epi, s);
        } else {
            e = launch_bitgemm_tc(a, epi, ws, ws_bytes, s);
        }
        g_last_kernel = (kern == SNP_KERNEL_TC_MXF4 && gemm_tc4_last_pair()) ? SNP_KERNEL_TC_MXF4_PAIR
                        : (kern == SNP_KERNEL_TC_MXF4 && gemm_tc4_last_sym()) ? SNP_KERNEL_TC_MXF4_SYM
                                                                               : kern;
    } else {
        e = launch_bitgemm_popc(a, epi, s);
        g_last_kernel = SNP_KERNEL_POPC;
    }
    if (e != cudaSuccess) return set_cuda_error(e);
    g_last_variant = variant;
    return SNP_OK;
}

}  // namespace

namespace snp {
void count_launches(int k) { g_launches.fetch_add(k, std::memory_order_relaxed); }
}  // namespace snp

extern "C" {

int64_t snp_words(int64_t nbits) {
    if (nbits <= 0) return 0;
    return ((words_needed(nbits) + 7) / 8) * 8;
}

size_t snp_ld_workspace_bytes(int64_t m, int64_t n, int64_t nbits) {
    if (m <= 0 || n <= 0 || nbits <= 0) return 0;
    size_t b = pops_bytes(m, n);
    if (choose_variant(m, n, nbits) == SNP_VARIANT_TC) b += tc_workspace_bytes(m, n, nbits);
    return b;
}

size_t snp_fastid_workspace_bytes(int64_t nq, int64_t nd, int64_t nbits, int op) {
    if (nq <= 0 || nd <= 0 || nbits <= 0) return 0;
    if (use_stream(nq, nd, nbits)) return 0;
    if (choose_variant(nq, nd, nbits) != SNP_VARIANT_TC) return 0;
    if (op != SNP_OP_AND && tc_kernel_for(nq, nd, nbits, EPI_COUNTS) == SNP_KERNEL_TC_MXF4)
        return pops_bytes(nq, nd);   // row popcounts for the general kernel's identities
    return tc_workspace_bytes(nq, nd, nbits);
}

snp_status snp_pack(const uint8_t *g, int64_t rows, int64_t nbits, int64_t ldg_bytes,
                    uint64_t *packed, int64_t ldw, void *stream) {
    if (rows < 0 || nbits < 0 || ldg_bytes < 0 || ldw < 0) return SNP_E_SHAPE;
    if (rows == 0) return SNP_OK;
    if (!g || !packed) return SNP_E_NULL;
    if (nbits < 1 || ldg_bytes < nbits || ldw < words_needed(nbits)) return SNP_E_SHAPE;
    if (!aligned16(packed) || (ldw & 1)) return SNP_E_ALIGN;
    snp_status st = check_arch();
    if (st != SNP_OK) return st;
    cudaError_t e = launch_pack(g, rows, nbits, ldg_bytes, packed, ldw, (cudaStream_t)stream);
    return e == cudaSuccess ? SNP_OK : set_cuda_error(e);
}

snp_status snp_pack_popc(const uint8_t *g, int64_t rows, int64_t nbits, int64_t ldg_bytes,
                         uint64_t *packed, int64_t ldw, uint32_t *popc, void *stream) {
    if (rows < 0 || nbits < 0 || ldg_bytes < 0 || ldw < 0) return SNP_E_SHAPE;
    if (rows == 0) return SNP_OK;
    if (!g || !packed || !popc) return SNP_E_NULL;
    if (nbits < 1 || ldg_bytes < nbits || ldw < words_needed(nbits)) return SNP_E_SHAPE;
    if (!aligned16(packed) || (ldw & 1)) return SNP_E_ALIGN;
    snp_status st = check_arch();
    if (st != SNP_OK) return st;
    cudaError_t e = launch_pack_popc(g, rows, nbits, ldg_bytes, packed, ldw, popc, (cudaStream_t)stream);
    return e == cudaSuccess ? SNP_OK : set_cuda_error(e);
}

snp_status snp_row_popc(const uint64_t *x, int64_t rows, int64_t nbits, int64_t ldw,
                        uint32_t *popc, void *stream) {
    snp_status st = check_nbits(nbits);
    if (rows < 0) return SNP_E_SHAPE;
    if (st != SNP_OK) return st;
    if ((st = check_packed(x, rows, ldw, nbits)) != SNP_OK) return st;
    if (rows == 0) return SNP_OK;
    if (!popc) return SNP_E_NULL;
    if ((st = check_arch()) != SNP_OK) return st;
    cudaError_t e = launch_row_popc(x, rows, nbits, ldw, popc, (cudaStream_t)stream);
    return e == cudaSuccess ? SNP_OK : set_cuda_error(e);
}

snp_status snp_ld_counts(const uint64_t *A, int64_t m, int64_t lda,
                         const uint64_t *B, int64_t n, int64_t ldb, int64_t nbits,
                         uint32_t *C, int64_t ldc, int accumulate,
                         void *ws, size_t ws_bytes, void *stream) {
    snp_status st;
    if (m < 0 || n < 0) return SNP_E_SHAPE;
    if ((st = check_nbits(nbits)) != SNP_OK) return st;
    if ((st = check_packed(A, m, lda, nbits)) != SNP_OK) return st;
    if ((st = check_packed(B, n, ldb, nbits)) != SNP_OK) return st;
    if (m == 0 || n == 0) return SNP_OK;
    if (!C) return SNP_E_NULL;
    if (ldc < n) return SNP_E_SHAPE;
    if (!aligned16(C)) return SNP_E_ALIGN;
    const int variant = choose_variant(m, n, nbits);
    const size_t need = snp_ld_workspace_bytes(m, n, nbits);
    if (ws_bytes < need || (need && !ws)) return SNP_E_WORKSPACE;
    if ((st = check_arch()) != SNP_OK) return st;
    GemmArgs a{};
    a.A = reinterpret_cast<const uint32_t *>(A);
    a.B = reinterpret_cast<const uint32_t *>(B);
    a.m = m; a.n = n; a.lda32 = 2 * lda; a.ldb32 = 2 * ldb; a.nbits = nbits;
    a.op = SNP_OP_AND; a.accumulate = accumulate ? 1 : 0; a.ldc = ldc; a.C = C;
    return run_gemm(a, EPI_COUNTS, variant, ws, ws_bytes, (cudaStream_t)stream);
}

snp_status snp_ld_r2(const uint64_t *A, int64_t m, int64_t lda, const uint32_t *popA,
                     const uint64_t *B, int64_t n, int64_t ldb, const uint32_t *popB,
                     int64_t nbits, float *r2, float *dprime, uint32_t *counts,
                     int64_t ldc, void *ws, size_t ws_bytes, void *stream) {
    snp_status st;
    if (m < 0 || n < 0) return SNP_E_SHAPE;
    if ((st = check_nbits(nbits)) != SNP_OK) return st;
    if ((st = check_packed(A, m, lda, nbits)) != SNP_OK) return st;
    if ((st = check_packed(B, n, ldb, nbits)) != SNP_OK) return st;
    if (m == 0 || n == 0) return SNP_OK;
    if (!r2) return SNP_E_NULL;
    if (ldc < n) return SNP_E_SHAPE;
    if (!aligned16(r2) || (dprime && !aligned16(dprime)) || (counts && !aligned16(counts)))
        return SNP_E_ALIGN;
    if (nbits > 0xB504F33LL) return SNP_E_RANGE;   // n^2 products must stay exact in int64/fp64
    const int variant = choose_variant(m, n, nbits);
    const size_t need = snp_ld_workspace_bytes(m, n, nbits);
    if (ws_bytes < need || !ws) return SNP_E_WORKSPACE;
    if ((st = check_arch()) != SNP_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    uint32_t *pa = reinterpret_cast<uint32_t *>(ws);
    uint32_t *pb = reinterpret_cast<uint32_t *>((char *)ws + align256((size_t)m * 4));
    cudaError_t e;
    // row popcounts (p_A, p_B of P:L44) for the r2/D' epilogue: one cheap pass over the
    // packed operands (O(m+n) vs the O(m n) GEMM)
    if (!popA) {
        if ((e = launch_row_popc(A, m, nbits, lda, pa, s)) != cudaSuccess) return set_cuda_error(e);
        popA = pa;
    }
    if (!popB) {
        if (B == A && n == m && ldb == lda) {
            popB = popA;   // self-LD (B aliases A): one popcount pass
        } else {
            if ((e = launch_row_popc(B, n, nbits, ldb, pb, s)) != cudaSuccess) return set_cuda_error(e);
            popB = pb;
        }
    }
    GemmArgs a{};
    a.A = reinterpret_cast<const uint32_t *>(A);
    a.B = reinterpret_cast<const uint32_t *>(B);
    a.m = m; a.n = n; a.lda32 = 2 * lda; a.ldb32 = 2 * ldb; a.nbits = nbits;
    a.op = SNP_OP_AND; a.accumulate = 0; a.ldc = ldc; a.C = counts;
    a.r2 = r2; a.dprime = dprime; a.popA = popA; a.popB = popB;
    return run_gemm(a, EPI_LD, variant, ws, ws_bytes, s);
}

int64_t snp_sym_tiles(int64_t m) {
    if (m <= 0) return 0;
    const int64_t T = (m + SYM_TILE - 1) / SYM_TILE;
    return T * (T + 1) / 2;
}

namespace {
// measurement hook: SNP_GEMM_BPRE=1 pre-expands the column operand of whole-triangle
// tensor-core self-LD into the workspace
bool ld_sym_bpre() {
    static const bool on = [] {
        const char *e = std::getenv("SNP_GEMM_BPRE");
        return e && e[0] == '1';
    }();
    return on;
}
}  // namespace

size_t snp_ld_sym_workspace_bytes(int64_t m, int64_t nbits) {
    if (m <= 0 || nbits <= 0) return 0;
    size_t b = align256((size_t)m * 4);   // row popcounts when popA is NULL
    if (ld_sym_bpre() && nbits < (1LL << 24)) b += align256(gemm_tc4_bpre_bytes(m, nbits));
    return b;
}

snp_status snp_ld_sym(const uint64_t *A, int64_t m, int64_t lda, const uint32_t *popA, int64_t nbits,
                      int64_t tile_lo, int64_t tile_hi, float *r2, float *dprime, uint32_t *counts,
                      void *ws, size_t ws_bytes, void *stream) {
    snp_status st;
    if (m < 0) return SNP_E_SHAPE;
    if ((st = check_nbits(nbits)) != SNP_OK) return st;
    if ((st = check_packed(A, m, lda, nbits)) != SNP_OK) return st;
    const int64_t ntot = snp_sym_tiles(m);
    if (tile_lo < 0 || tile_hi < tile_lo || tile_hi > ntot) return SNP_E_RANGE;
    if (m == 0 || tile_hi == tile_lo) return SNP_OK;
    if (!r2 && !counts) return SNP_E_NULL;
    if (dprime && !r2) return SNP_E_NULL;
    if ((r2 && !aligned16(r2)) || (dprime && !aligned16(dprime)) || (counts && !aligned16(counts)))
        return SNP_E_ALIGN;
    if (nbits > 0xB504F33LL) return SNP_E_RANGE;   // n^2 products must stay exact in int64/fp64
    const bool want_ld = r2 != nullptr;
    int variant = choose_variant(m, m, nbits);
    if (variant == SNP_VARIANT_TC && !gemm_tc4_supported(m, m, nbits)) {
        // the packed layout is produced by the mxf4 kernel (nbits < 2^24) and the CUDA-core
        // kernel; auto dispatch takes the CUDA-core one above that, a forced TC cannot
        if (current_variant() == SNP_VARIANT_TC) return SNP_E_SHAPE;
        variant = SNP_VARIANT_POPC;
    }
    const bool need_pop = want_ld && !popA;
    if (need_pop && (ws_bytes < snp_ld_sym_workspace_bytes(m, nbits) || !ws)) return SNP_E_WORKSPACE;
    if ((st = check_arch()) != SNP_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e;
    if (need_pop) {
        uint32_t *pa = reinterpret_cast<uint32_t *>(ws);
        if ((e = launch_row_popc(A, m, nbits, lda, pa, s)) != cudaSuccess) return set_cuda_error(e);
        popA = pa;
    }
    GemmArgs a{};
    a.A = a.B = reinterpret_cast<const uint32_t *>(A);
    a.m = a.n = m; a.lda32 = a.ldb32 = 2 * lda; a.nbits = nbits;
    a.op = SNP_OP_AND; a.accumulate = 0; a.ldc = SYM_TILE; a.C = counts;
    a.r2 = r2; a.dprime = dprime; a.popA = a.popB = popA;
    a.tri_lo = tile_lo; a.tri_n = tile_hi - tile_lo;
    if (variant == SNP_VARIANT_TC && ld_sym_bpre() && ws && ws_bytes >= snp_ld_sym_workspace_bytes(m, nbits))
        a.bpre = reinterpret_cast<uint32_t *>(reinterpret_cast<uint8_t *>(ws) + align256((size_t)m * 4));
    if (variant == SNP_VARIANT_TC) {
        e = launch_gemm_tc4(a, want_ld ? EPI_LD : EPI_COUNTS, s);
        g_last_kernel = gemm_tc4_last_pair() ? SNP_KERNEL_TC_MXF4_SYM_PAIR : SNP_KERNEL_TC_MXF4_SYM;
    } else {
        e = launch_bitgemm_popc(a, want_ld ? EPI_LD : EPI_COUNTS, s);
        g_last_kernel = SNP_KERNEL_POPC;
    }
    if (e != cudaSuccess) return set_cuda_error(e);
    g_last_variant = variant;
    return SNP_OK;
}

snp_status snp_sym_unpack(const uint32_t *tiles, int64_t m, int64_t tile_lo, int64_t tile_hi, uint32_t *out,
                          int64_t ldo, void *stream) {
    if (m < 0) return SNP_E_SHAPE;
    const int64_t ntot = snp_sym_tiles(m);
    if (tile_lo < 0 || tile_hi < tile_lo || tile_hi > ntot) return SNP_E_RANGE;
    if (m == 0 || tile_hi == tile_lo) return SNP_OK;
    if (!tiles || !out) return SNP_E_NULL;
    if (ldo < m) return SNP_E_SHAPE;
    snp_status st;
    if ((st = check_arch()) != SNP_OK) return st;
    cudaError_t e = launch_sym_unpack(tiles, m, tile_lo, tile_hi - tile_lo, out, ldo, (cudaStream_t)stream);
    return e == cudaSuccess ? SNP_OK : set_cuda_error(e);
}

snp_status snp_fastid(const uint64_t *Q, int64_t nq, int64_t ldq, const uint32_t *popQ,
                      const uint64_t *D, int64_t nd, int64_t ldd, const uint32_t *popD,
                      int64_t nbits, int op, uint32_t *out, int64_t ldo, int accumulate,
                      void *ws, size_t ws_bytes, void *stream) {
    snp_status st;
    if (nq < 0 || nd < 0) return SNP_E_SHAPE;
    if (op < SNP_OP_AND || op > SNP_OP_NOTAND) return SNP_E_OP;
    if ((st = check_nbits(nbits)) != SNP_OK) return st;
    if ((st = check_packed(Q, nq, ldq, nbits)) != SNP_OK) return st;
    if ((st = check_packed(D, nd, ldd, nbits)) != SNP_OK) return st;
    if (nq == 0 || nd == 0) return SNP_OK;
    if (!out) return SNP_E_NULL;
    if (ldo < nd) return SNP_E_SHAPE;
    if (!aligned16(out)) return SNP_E_ALIGN;
    const int variant = choose_variant(nq, nd, nbits);
    const size_t need = snp_fastid_workspace_bytes(nq, nd, nbits, op);
    if (ws_bytes < need || (need && !ws)) return SNP_E_WORKSPACE;
    if ((st = check_arch()) != SNP_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    GemmArgs a{};
    a.A = reinterpret_cast<const uint32_t *>(Q);
    a.B = reinterpret_cast<const uint32_t *>(D);
    a.m = nq; a.n = nd; a.lda32 = 2 * ldq; a.ldb32 = 2 * ldd; a.nbits = nbits;
    a.op = op; a.accumulate = accumulate ? 1 : 0; a.ldc = ldo; a.C = out;
    a.popA = popQ; a.popB = popD;
    if (use_stream(nq, nd, nbits)) {
        SearchArgs sa{};
        sa.Q = a.A; sa.nq = nq; sa.ldq32 = a.lda32;
        sa.D = a.B; sa.nd = nd; sa.ldd32 = a.ldb32;
        sa.popD = popD; sa.nbits = nbits;
        sa.nops = 1; sa.ops[0] = op; sa.counts[0] = out; sa.ldo = ldo; sa.accumulate = a.accumulate;
        cudaError_t e = launch_fastid_stream(sa, s);
        if (e != cudaSuccess) return set_cuda_error(e);
        g_last_variant = SNP_VARIANT_POPC;
        g_last_kernel = SNP_KERNEL_POPC_STREAM;
        return SNP_OK;
    }
    if (variant == SNP_VARIANT_TC) {
        // given popcounts are used as they are (the FastID kernel skips counting the
        // streamed database words); NULL ones are derived in-kernel or by a pre-pass
        return run_gemm(a, EPI_COUNTS, variant, ws, ws_bytes, s);
    }
    return run_gemm(a, EPI_COUNTS, variant, nullptr, 0, s);
}

snp_status snp_fastid_best(const uint32_t *counts, int64_t nq, int64_t nd, int64_t ldo,
                           int64_t index_base, uint32_t *best_count, int64_t *best_index,
                           void *stream) {
    if (nq < 0 || nd < 0) return SNP_E_SHAPE;
    if (nd > 0xfffffffeLL) return SNP_E_RANGE;
    if (nq == 0) return SNP_OK;
    if (!best_count || !best_index || (nd > 0 && !counts)) return SNP_E_NULL;
    if (ldo < nd) return SNP_E_SHAPE;
    if (((uintptr_t)best_index & 7u) || ((uintptr_t)best_count & 3u) || ((uintptr_t)counts & 3u))
        return SNP_E_ALIGN;
    snp_status st = check_arch();
    if (st != SNP_OK) return st;
    cudaError_t e = launch_best(counts, nq, nd, ldo, index_base, best_count, best_index,
                                (cudaStream_t)stream);
    return e == cudaSuccess ? SNP_OK : set_cuda_error(e);
}

}  // extern "C"

// ---------------------------------------------------------------- f1: fused search
namespace {

// Database rows per chunk of the composed (non-fused) search path when best matches are
// wanted without stored counts: <= 64 MiB of chunk counts, a multiple of 128 rows.
int64_t search_chunk_rows(int64_t nq, int64_t nd) {
    int64_t ch = ((int64_t)(64 << 20) / (4 * (nq > 0 ? nq : 1))) / 128 * 128;
    const char *e = std::getenv("SNP_SEARCH_CHUNK_ROWS");   // test hook: force small chunks
    if (e && std::atoll(e) > 0) ch = std::atoll(e);
    if (ch < 128) ch = 128;
    return ch < nd ? ch : nd;
}

bool search_fused(int64_t nq, int64_t nd, int64_t nbits) {
    return nd > 0 && choose_variant(nq, nd, nbits) == SNP_VARIANT_TC &&
           tc_kernel_for(nq, nd, nbits, EPI_COUNTS) == SNP_KERNEL_FASTID_MXF4;
}

// a7 measured dispatch (configs[4] sweeps, profiles/round1/sweep_configs4*.txt): for more than 64
// queries at nbits <= 4096 the fused FastID kernel run on 64-query slices (one database
// pass each) beats the general kernel + best pass (e.g. M = 128 x 1M x 2048: 0.28 vs
// 0.63 ms, M = 8192 x 1M x 4096: 26 vs 31 ms); above 4096 bits the general kernel wins.
// Returns the slice width (64, or 32 where only the 32-wide kernel fits: 33..64 queries at
// 6500..9700 bits, 2 x 4.9 ms vs 14.3 ms at 20M x 8192) or 0 for no slicing.
int64_t search_slice_width(int64_t nq, int64_t nd, int64_t nbits) {
    const char *e = std::getenv("SNP_SEARCH_SLICES");   // "0": never (A/B measurement hook)
    if (e && e[0] == '0') return 0;
    if (nd <= 0 || nq <= 32 || choose_variant(nq, nd, nbits) != SNP_VARIANT_TC) return 0;
    if (nq > 64 && nbits <= 4096 && fastid_bn(64, nbits) == 64 && fastid_tc4_supported(64, nd, nbits)) return 64;
    if (nq <= 64 && fastid_bn(64, nbits) == 0 && fastid_bn(32, nbits) == 32 && fastid_tc4_supported(32, nd, nbits))
        return 32;
    return 0;
}
bool search_sliced(int64_t nq, int64_t nd, int64_t nbits) { return search_slice_width(nq, nd, nbits) != 0; }
// Long profiles with <= 64 queries whose expanded batch does not fit the FastID kernel's shared
// memory: the profiles are cut into K chunks (multiples of 1024 bits) that fit, each chunk one
// pass of the FastID kernel over the database's chunk columns that ADDS its counts (every op is
// linear in the chunk-local AND count and popcounts, so the sums are exact); the
// database is read once in total instead of going to the general kernel.  Returns the chunk
// size in bits, or 0 when the path does not apply.
int64_t search_kchunk_bits(int64_t nq, int64_t nd, int64_t nbits) {
    const char *e = std::getenv("SNP_SEARCH_KCHUNK");   // "0": never (A/B measurement hook)
    if (e && e[0] == '0') return 0;
    // measured (profiles/round2/sweep_kchunk.txt, best-only 4M x 16384): 8 queries 3.43 -> 2.09 ms,
    // 16 about 8 % faster, 32 equal, 64 four times slower (the per-chunk count read-modify-write
    // grows with the query count) than the general kernel: used up to 16 queries
    if (nd <= 0 || nq < 1 || nq > 16 || nbits <= 1024 || choose_variant(nq, nd, nbits) != SNP_VARIANT_TC) return 0;
    if (fastid_tc4_supported(nq, nd, nbits) || search_slice_width(nq, nd, nbits)) return 0;
    for (int64_t cb = (nbits - 1) / 1024 * 1024; cb >= 1024; cb -= 1024)
        if (fastid_tc4_supported(nq, nd, cb)) return cb;
    return 0;
}

}  // namespace

extern "C" {

size_t snp_fastid_search_workspace_bytes(int64_t nq, int64_t nd, int64_t nbits, int nops) {
    if (nq <= 0 || nbits <= 0 || nops < 1 || nops > 4) return 0;
    if (nd < 0) return 0;
    if (nd > 0 && use_stream(nq, nd, nbits)) return fastid_stream_ws_bytes(nq, nops);
    if (search_fused(nq, nd, nbits)) return fastid_search_tc4_ws_bytes(nq, nops);
    if (search_sliced(nq, nd, nbits)) return fastid_search_tc4_ws_bytes(search_slice_width(nq, nd, nbits), nops);
    if (search_kchunk_bits(nq, nd, nbits))   // keys + per-op count chunks (for ops without stored counts)
        return align256((size_t)nops * nq * 8) + (size_t)nops * align256((size_t)nq * search_chunk_rows(nq, nd) * 4) +
               fastid_search_tc4_ws_bytes(nq, nops);
    size_t b = align256((size_t)nops * nq * 8);
    if (nd == 0) return b;
    b += align256((size_t)nq * search_chunk_rows(nq, nd) * 4);
    size_t g = 0;
    for (int op = SNP_OP_AND; op <= SNP_OP_NOTAND; ++op) {
        const size_t x = snp_fastid_workspace_bytes(nq, nd, nbits, op);
        if (x > g) g = x;
    }
    return b + g;
}

snp_status snp_fastid_search(const uint64_t *Q, int64_t nq, int64_t ldq,
                             const uint64_t *D, int64_t nd, int64_t ldd, const uint32_t *popD, int64_t nbits,
                             int nops, const int *ops, uint32_t *const *counts, int64_t ldo,
                             uint32_t *const *best_count, int64_t *const *best_index,
                             int64_t index_base, void *ws, size_t ws_bytes, void *stream) {
    snp_status st;
    if (nq < 0 || nd < 0) return SNP_E_SHAPE;
    if (nops < 1 || nops > 4) return SNP_E_OP;
    if (!ops) return SNP_E_NULL;
    for (int j = 0; j < nops; ++j)
        if (ops[j] < SNP_OP_AND || ops[j] > SNP_OP_NOTAND) return SNP_E_OP;
    if ((st = check_nbits(nbits)) != SNP_OK) return st;
    if ((st = check_packed(Q, nq, ldq, nbits)) != SNP_OK) return st;
    if ((st = check_packed(D, nd, ldd, nbits)) != SNP_OK) return st;
    if ((best_count == nullptr) != (best_index == nullptr)) return SNP_E_NULL;
    if (nd > 0xfffffffeLL) return SNP_E_RANGE;
    if (nq == 0) return SNP_OK;
    bool any_counts = false, any_best = false;
    for (int j = 0; j < nops; ++j) {
        uint32_t *c = counts ? counts[j] : nullptr;
        if (c) {
            any_counts = true;
            if (!aligned16(c)) return SNP_E_ALIGN;
        }
        if (best_count) {
            if ((best_count[j] == nullptr) != (best_index[j] == nullptr)) return SNP_E_NULL;
            if (best_count[j]) {
                any_best = true;
                if (((uintptr_t)best_count[j] & 3u) || ((uintptr_t)best_index[j] & 7u)) return SNP_E_ALIGN;
            }
        }
    }
    if (any_counts && ldo < nd) return SNP_E_SHAPE;
    if (!any_counts && !any_best) return SNP_OK;
    const size_t need = snp_fastid_search_workspace_bytes(nq, nd, nbits, nops);
    if (ws_bytes < need || !ws) return SNP_E_WORKSPACE;
    if ((st = check_arch()) != SNP_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e;

    SearchArgs a{};
    a.Q = reinterpret_cast<const uint32_t *>(Q);
    a.nq = nq; a.ldq32 = 2 * ldq;
    a.D = reinterpret_cast<const uint32_t *>(D);
    a.nd = nd; a.ldd32 = 2 * ldd;
    a.popD = popD;
    a.nbits = nbits;
    a.nops = nops;
    a.ldo = ldo;
    a.index_base = index_base;
    for (int j = 0; j < nops; ++j) {
        a.ops[j] = ops[j];
        a.counts[j] = counts ? counts[j] : nullptr;
        a.best_count[j] = best_count ? best_count[j] : nullptr;
        a.best_index[j] = best_index ? best_index[j] : nullptr;
    }
    if (nd > 0 && use_stream(nq, nd, nbits)) {
        // few queries: one CUDA-core pass over the database for every op (fastid_stream.cu)
        a.keys = reinterpret_cast<unsigned long long *>(ws);
        a.done = reinterpret_cast<unsigned int *>((char *)ws + align256((size_t)nops * nq * 8));
        if ((e = launch_fastid_stream(a, s)) != cudaSuccess) return set_cuda_error(e);
        g_last_variant = SNP_VARIANT_POPC;
        g_last_kernel = SNP_KERNEL_POPC_STREAM;
        return SNP_OK;
    }
    if (search_fused(nq, nd, nbits)) {
        // one pass over the database for every op (fastid_tc4.cu)
        a.keys = reinterpret_cast<unsigned long long *>(ws);
        a.done = reinterpret_cast<unsigned int *>((char *)ws + align256((size_t)nops * nq * 8));
        if ((e = launch_fastid_search_tc4(a, s)) != cudaSuccess) return set_cuda_error(e);
        g_last_variant = SNP_VARIANT_TC;
        g_last_kernel = SNP_KERNEL_FASTID_MXF4;
        return SNP_OK;
    }

    if (const int64_t SLICE_Q = search_slice_width(nq, nd, nbits)) {
        // 64-query slices through the fused kernel, one database pass each; the key
        // workspace is reused slice after slice (stream order; each launch re-initialises it)
        for (int64_t q0 = 0; q0 < nq; q0 += SLICE_Q) {
            SearchArgs b = a;
            b.Q = a.Q + q0 * a.ldq32;
            b.nq = nq - q0 < SLICE_Q ? nq - q0 : SLICE_Q;
            for (int j = 0; j < nops; ++j) {
                b.counts[j] = a.counts[j] ? a.counts[j] + q0 * ldo : nullptr;
                b.best_count[j] = a.best_count[j] ? a.best_count[j] + q0 : nullptr;
                b.best_index[j] = a.best_index[j] ? a.best_index[j] + q0 : nullptr;
            }
            b.keys = reinterpret_cast<unsigned long long *>(ws);
            b.done = reinterpret_cast<unsigned int *>((char *)ws + align256((size_t)nops * SLICE_Q * 8));
            if ((e = launch_fastid_search_tc4(b, s)) != cudaSuccess) return set_cuda_error(e);
        }
        g_last_variant = SNP_VARIANT_TC;
        g_last_kernel = SNP_KERNEL_FASTID_MXF4;
        return SNP_OK;
    }

    if (const int64_t KC = search_kchunk_bits(nq, nd, nbits)) {
        // K-chunked FastID kernel passes (see search_kchunk_bits): counts of every op land in
        // the caller's matrix, or — for ops without stored counts — in workspace count chunks
        // over database row blocks; best matches by best.cu from the summed counts
        unsigned long long *keys = reinterpret_cast<unsigned long long *>(ws);
        char *p = (char *)ws + align256((size_t)nops * nq * 8);
        const int64_t ch = search_chunk_rows(nq, nd);
        uint32_t *tmp[4];
        for (int j = 0; j < nops; ++j) {
            tmp[j] = reinterpret_cast<uint32_t *>(p);
            p += align256((size_t)nq * ch * 4);
        }
        for (int j = 0; j < nops; ++j)
            if (a.best_count[j] && (e = launch_best_init(keys + (int64_t)j * nq, nq, s)) != cudaSuccess)
                return set_cuda_error(e);
        bool all_stored = true;
        for (int j = 0; j < nops; ++j) all_stored = all_stored && a.counts[j] != nullptr;
        // database row blocks: the whole database when every op's counts are stored, else
        // blocks of ch rows through the workspace chunks (ops with stored counts write in place)
        const int64_t rstep = all_stored ? nd : ch;
        for (int64_t r0 = 0; r0 < nd; r0 += rstep) {
            const int64_t rows = nd - r0 < rstep ? nd - r0 : rstep;
            for (int j0 = 0; j0 < nops; j0 += 2) {
                // one pass for two ops whose counts go to the same kind of buffer, else one per op
                const int nj = nops - j0 >= 2 ? 2 : 1;
                const bool pair = nj == 2 && ((a.counts[j0] != nullptr) == (a.counts[j0 + 1] != nullptr));
                for (int g0 = j0; g0 < j0 + nj; g0 += pair ? 2 : 1) {
                    const int ng = pair ? 2 : 1;
                    const bool in_place = a.counts[g0] != nullptr;
                    for (int64_t k0 = 0; k0 < nbits; k0 += KC) {
                        SearchArgs c{};
                        c.Q = a.Q + k0 / 32; c.nq = nq; c.ldq32 = a.ldq32;
                        c.D = a.D + r0 * a.ldd32 + k0 / 32; c.nd = rows; c.ldd32 = a.ldd32;
                        c.dcols32 = a.ldd32 - k0 / 32;         // the rows' remaining words: no over-read
                        c.popD = nullptr;                      // chunk-local popcounts, counted in-kernel
                        c.nbits = nbits - k0 < KC ? nbits - k0 : KC;
                        c.nops = ng;
                        c.accumulate = k0 > 0 ? 1 : 0;
                        c.ldo = in_place ? ldo : ch;
                        for (int jj = 0; jj < ng; ++jj) {
                            c.ops[jj] = ops[g0 + jj];
                            c.counts[jj] = in_place ? a.counts[g0 + jj] + r0 : tmp[g0 + jj];
                        }
                        if ((e = launch_fastid_search_tc4(c, s)) != cudaSuccess) return set_cuda_error(e);
                    }
                }
            }
            for (int j = 0; j < nops; ++j) {
                if (!a.best_count[j]) continue;
                const uint32_t *cj = a.counts[j] ? a.counts[j] + r0 : tmp[j];
                if ((e = launch_best_reduce(cj, nq, rows, a.counts[j] ? ldo : ch, r0, keys + (int64_t)j * nq, s)) !=
                    cudaSuccess)
                    return set_cuda_error(e);
            }
        }
        for (int j = 0; j < nops; ++j)
            if (a.best_count[j] &&
                (e = launch_best_finalize(keys + (int64_t)j * nq, nq, index_base, a.best_count[j], a.best_index[j], s)) !=
                    cudaSuccess)
                return set_cuda_error(e);
        if (any_best && (e = cudaMemsetAsync(ws, 0, (size_t)nops * nq * 8, s)) != cudaSuccess)   // zero-filled again
            return set_cuda_error(e);
        g_last_variant = SNP_VARIANT_TC;
        g_last_kernel = SNP_KERNEL_FASTID_MXF4;
        return SNP_OK;
    }

    // Composed path (shapes the fused kernel does not take, or a forced variant): per op,
    // counts by snp_fastid's kernels, best by best.cu; without stored counts the database
    // is processed in chunks into workspace counts (nothing nq x nd is allocated).
    unsigned long long *keys = reinterpret_cast<unsigned long long *>(ws);
    char *p = (char *)ws + align256((size_t)nops * nq * 8);
    const int64_t ch = nd > 0 ? search_chunk_rows(nq, nd) : 0;
    uint32_t *chunk = reinterpret_cast<uint32_t *>(p);
    if (nd > 0) p += align256((size_t)nq * ch * 4);
    void *gws = p;
    const size_t gws_bytes = ws_bytes - (size_t)(p - (char *)ws);
    const int variant = choose_variant(nq, nd, nbits);
    // two ops whose counts are both stored come from ONE pass of the general tensor kernel
    // (swapped layout: database rows on TMEM lanes), which writes both identities of the
    // same AND count; the CUDA-core variant computes each op directly
    const bool pairable = variant == SNP_VARIANT_TC && nd > nq &&
                          tc_kernel_for(nq, nd, nbits, EPI_COUNTS) == SNP_KERNEL_TC_MXF4;
    for (int j = 0; j < nops; ++j) {
        const bool best = a.best_count[j] != nullptr;
        unsigned long long *kj = keys + (int64_t)j * nq;
        if (best && (e = launch_best_init(kj, nq, s)) != cudaSuccess) return set_cuda_error(e);
        if (pairable && j + 1 < nops && a.counts[j] && a.counts[j + 1] && nd > 0) {
            GemmArgs g{};
            g.A = a.Q; g.B = a.D; g.m = nq; g.n = nd; g.lda32 = a.ldq32; g.ldb32 = a.ldd32;
            g.nbits = nbits; g.op = ops[j]; g.ldc = ldo; g.C = a.counts[j]; g.popB = popD;
            g.op2 = ops[j + 1]; g.C2 = a.counts[j + 1];
            if ((st = run_gemm(g, EPI_COUNTS, variant, gws, gws_bytes, s)) != SNP_OK) return st;
            for (int jj = j; jj <= j + 1; ++jj) {
                if (!a.best_count[jj]) continue;
                unsigned long long *kk = keys + (int64_t)jj * nq;
                if (jj != j && (e = launch_best_init(kk, nq, s)) != cudaSuccess) return set_cuda_error(e);
                if ((e = launch_best_reduce(a.counts[jj], nq, nd, ldo, 0, kk, s)) != cudaSuccess)
                    return set_cuda_error(e);
                if ((e = launch_best_finalize(kk, nq, index_base, a.best_count[jj], a.best_index[jj], s)) !=
                    cudaSuccess)
                    return set_cuda_error(e);
            }
            ++j;
            continue;
        }
        if (a.counts[j] && nd > 0) {
            GemmArgs g{};
            g.A = a.Q; g.B = a.D; g.m = nq; g.n = nd; g.lda32 = a.ldq32; g.ldb32 = a.ldd32;
            g.nbits = nbits; g.op = ops[j]; g.ldc = ldo; g.C = a.counts[j]; g.popB = popD;
            if ((st = run_gemm(g, EPI_COUNTS, variant, gws, gws_bytes, s)) != SNP_OK) return st;
            if (best && (e = launch_best_reduce(a.counts[j], nq, nd, ldo, 0, kj, s)) != cudaSuccess)
                return set_cuda_error(e);
        } else if (best) {
            for (int64_t j0 = 0; j0 < nd; j0 += ch) {
                const int64_t rows = nd - j0 < ch ? nd - j0 : ch;
                const int cv = choose_variant(nq, rows, nbits);
                GemmArgs g{};
                g.A = a.Q; g.B = a.D + j0 * a.ldd32; g.m = nq; g.n = rows;
                g.lda32 = a.ldq32; g.ldb32 = a.ldd32;
                g.popB = popD ? popD + j0 : nullptr;
                g.nbits = nbits; g.op = ops[j]; g.ldc = ch; g.C = chunk;
                if ((st = run_gemm(g, EPI_COUNTS, cv, gws, gws_bytes, s)) != SNP_OK) return st;
                if ((e = launch_best_reduce(chunk, nq, rows, ch, j0, kj, s)) != cudaSuccess)
                    return set_cuda_error(e);
            }
        }
        if (best && (e = launch_best_finalize(kj, nq, index_base, a.best_count[j], a.best_index[j], s)) !=
                        cudaSuccess)
            return set_cuda_error(e);
    }
    // the key region is returned to zero (the fused kernels rely on a zero-filled workspace)
    if (any_best && (e = cudaMemsetAsync(ws, 0, (size_t)nops * nq * 8, s)) != cudaSuccess) return set_cuda_error(e);
    return SNP_OK;
}

}  // extern "C"

extern "C" {

snp_status snp_shard_plan(int64_t rows, int world, int64_t align, int64_t *bounds) {
    if (world < 1 || align < 1 || rows < 0) return SNP_E_RANGE;
    if (!bounds) return SNP_E_NULL;
    const int64_t nblocks = (rows + align - 1) / align;
    const int64_t base = nblocks / world, rem = nblocks % world;
    int64_t blk = 0;
    bounds[0] = 0;
    for (int r = 0; r < world; ++r) {
        blk += base + (r < rem ? 1 : 0);
        const int64_t b = blk * align;
        bounds[r + 1] = b < rows ? b : rows;
    }
    return SNP_OK;
}

size_t snp_fastid_threshold_workspace_bytes(int64_t nq, int64_t nd, int64_t nbits, int op) {
    if (nq <= 0 || nd <= 0 || nbits <= 0) return 0;
    const int64_t ch = search_chunk_rows(nq, nd);
    return align256((size_t)nq * ch * 4) + snp_fastid_workspace_bytes(nq, ch, nbits, op) + 256;
}

snp_status snp_fastid_threshold(const uint64_t *Q, int64_t nq, int64_t ldq, const uint64_t *D, int64_t nd,
                                int64_t ldd, const uint32_t *popD, int64_t nbits, int op, uint32_t tau,
                                int64_t index_base, snp_match *matches, int64_t capacity, uint64_t *match_count,
                                void *ws, size_t ws_bytes, void *stream) {
    snp_status st;
    if (nq < 0 || nd < 0 || capacity < 0) return SNP_E_SHAPE;
    if (op < SNP_OP_AND || op > SNP_OP_NOTAND) return SNP_E_OP;
    if ((st = check_nbits(nbits)) != SNP_OK) return st;
    if ((st = check_packed(Q, nq, ldq, nbits)) != SNP_OK) return st;
    if ((st = check_packed(D, nd, ldd, nbits)) != SNP_OK) return st;
    if (!match_count || (capacity > 0 && !matches)) return SNP_E_NULL;
    if (((uintptr_t)match_count & 7u) || ((uintptr_t)matches & 15u)) return SNP_E_ALIGN;
    if (nq > 65535) return SNP_E_RANGE;
    if ((st = check_arch()) != SNP_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e = cudaMemsetAsync(match_count, 0, sizeof(uint64_t), s);
    if (e != cudaSuccess) return set_cuda_error(e);
    if (nq == 0 || nd == 0) return SNP_OK;
    const size_t need = snp_fastid_threshold_workspace_bytes(nq, nd, nbits, op);
    if (ws_bytes < need || !ws) return SNP_E_WORKSPACE;
    // the database in row chunks: counts of one chunk into workspace (snp_fastid's dispatch:
    // the streaming, FastID or general kernel), then one compaction pass over the chunk
    const int64_t ch = search_chunk_rows(nq, nd);
    uint32_t *chunk = reinterpret_cast<uint32_t *>(ws);
    char *ws2 = (char *)ws + align256((size_t)nq * ch * 4);
    const size_t ws2_bytes = ws_bytes - align256((size_t)nq * ch * 4);
    for (int64_t j0 = 0; j0 < nd; j0 += ch) {
        const int64_t rows = nd - j0 < ch ? nd - j0 : ch;
        if ((st = snp_fastid(Q, nq, ldq, nullptr, D + j0 * ldd, rows, ldd, popD ? popD + j0 : nullptr, nbits, op,
                             chunk, ch, 0, ws2, ws2_bytes, stream)) != SNP_OK)
            return st;
        if ((e = launch_threshold_compact(chunk, nq, rows, ch, index_base + j0, tau,
                                          reinterpret_cast<ThresholdMatch *>(matches), capacity,
                                          reinterpret_cast<unsigned long long *>(match_count), s)) != cudaSuccess)
            return set_cuda_error(e);
    }
    return SNP_OK;
}

snp_status snp_shard_plan_sym(int64_t m, int world, int64_t *tile_bounds) {
    if (world < 1 || m < 0) return SNP_E_RANGE;
    if (!tile_bounds) return SNP_E_NULL;
    // equal-cost 128 x 128 tiles, so contiguous ranges of the row-major triangle balance
    // the work to within one tile: bounds[r] = floor(r * total / world)
    const int64_t total = snp_sym_tiles(m);
    for (int r = 0; r <= world; ++r) {
        // r * total can overflow int64 only for total > 2^56 (m > 2^35): not reachable (m < 2^31)
        tile_bounds[r] = (int64_t)(((__int128)r * total) / world);
    }
    return SNP_OK;
}

snp_status snp_set_variant(int variant) {
    if (variant < SNP_VARIANT_AUTO || variant > SNP_VARIANT_TC) return SNP_E_OP;
    current_variant();
    g_variant.store(variant);
    return SNP_OK;
}

int snp_last_variant(void) { return g_last_variant; }

int snp_last_kernel(void) { return g_last_kernel; }



int64_t snp_launch_count(void) { return (int64_t)g_launches.load(); }

const char *snp_status_string(int status) {
    switch (status) {
    case SNP_OK: return "SNP_OK";
    case SNP_E_NULL: return "SNP_E_NULL: a required pointer is NULL";
    case SNP_E_SHAPE: return "SNP_E_SHAPE: invalid size or leading dimension";
    case SNP_E_ALIGN: return "SNP_E_ALIGN: pointer not 16-byte aligned or odd packed leading dimension";
    case SNP_E_OP: return "SNP_E_OP: unknown op or variant";
    case SNP_E_RANGE: return "SNP_E_RANGE: value out of supported range";
    case SNP_E_WORKSPACE: return "SNP_E_WORKSPACE: workspace too small";
    case SNP_E_ARCH: return "SNP_E_ARCH: current device is not a compute capability 10.0 (B200) GPU";
    case SNP_E_CUDA: return "SNP_E_CUDA: CUDA error (see snp_last_cuda_error)";
    default: return "unknown snp_status";
    }
}

const char *snp_last_cuda_error(void) { return g_cuda_err; }

}  // extern "C"
