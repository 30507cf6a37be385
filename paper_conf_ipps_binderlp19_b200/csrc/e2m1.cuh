// e2m1.cuh — exact 1-bit products on the 4-bit tensor cores, shared by
// every kind::mxf4 kernel of the library (fastid_tc4.cu, gemm_tc4.cu) — and the tail mask
// used by every kernel that reads packed rows.
//
// sm_100a has no native 1-bit MMA, so each packed bit becomes an e2m1 nibble and the
// product is `tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32` with every scale
// factor 2^0.  Counts are Σ POPC(a & b) over the packed words (Eq. 1; γ += Σ POPC,
// P:L114-116 §III): every product of two set bits must be exactly 1.0 and every fp32
// partial sum an exact integer (measured exact to nbits = 2^23 − 1 on odd random counts,
// tests/test_gpu_exactness.py).
#pragma once
#include <stdint.h>

// Profiling instrumentation (pipeline clock stamps, the no-store and no-expand experiments,
// the snp_debug_* trace readers) exists only in builds with -DSNP_PROFILING
// (scripts/build_variant.sh); in the product library every such flag is a constant false.
#ifdef SNP_PROFILING
#define SNP_PROF(x) (x)
#else
#define SNP_PROF(x) false
#endif

namespace snp {

// Bits of 32-bit word w (0-based) of a row that lie below nbits (padding never counts:
// SURVEY §8a tail handling; the caller's padding bits are garbage by contract).
__device__ __forceinline__ uint32_t word_mask(int64_t w, int64_t nbits) {
    const int64_t lo = w * 32;
    if (lo + 32 <= nbits) return 0xffffffffu;
    if (lo >= nbits) return 0u;
    return (1u << (uint32_t)(nbits - lo)) - 1u;
}

// Bits -> e2m1 nibbles.  Output word t of input word x holds bit 4n + t in nibble n (a fixed
// K permutation shared by both operands, so every dot product is unchanged).  The two
// operands use complementary nibble positions so every product of set bits is exactly 1.0
// with as few shifts as possible (e2m1: bit0 = 0.5, bit1 = 1.0, bit2 = 2.0):
//   t:        0            1           2            3
//   A         bit0 = 0.5   bit1 = 1.0  bit2 = 2.0   bit1 = 1.0 (x >> 2)
//   B         bit2 = 2.0   bit1 = 1.0  bit0 = 0.5   bit1 = 1.0 (x >> 2)
// A: 4 LOP3 + 1 shift, B: 4 LOP3 + 2 shifts; the shifts run on the FMA pipe (IMAD.HI).
__device__ __forceinline__ void expandA(uint32_t x, uint32_t &o0, uint32_t &o1, uint32_t &o2, uint32_t &o3) {
    o0 = x & 0x11111111u;
    o1 = x & 0x22222222u;
    o2 = x & 0x44444444u;
    o3 = __umulhi(x, 0x40000000u) & 0x22222222u;   // (x >> 2) on the FMA pipe
}
__device__ __forceinline__ void expandB(uint32_t x, uint32_t &o0, uint32_t &o1, uint32_t &o2, uint32_t &o3) {
    const uint32_t y = __umulhi(x, 0x40000000u);    // x >> 2
    o0 = (x * 4u) & 0x44444444u;
    o1 = x & 0x22222222u;
    o2 = y & 0x11111111u;
    o3 = y & 0x22222222u;
}

// Instruction descriptor of kind::mxf4.block_scale (e2m1 x e2m1, fp32 accumulator,
// K-major A and B, ue8m0 scale factors): M >> 4 at bit 24, N >> 3 at bit 17.
__host__ __device__ constexpr uint32_t idesc_mxf4(int M, int N) {
    return (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | (1u << 23) | ((uint32_t)(M >> 4) << 24);
}

// ue8m0 scale factor 2^0 in every byte (written once per CTA into the scale-factor columns)
constexpr uint32_t SF_ONE_X4 = 0x7F7F7F7Fu;

// Exact count from an fp32 accumulator word holding an integer c < 2^23: bits(v + 2^23) =
// 0x4B000000 + c (one FADD, no F2I).
constexpr uint32_t MAGIC_2P23_BITS = 0x4B000000u;
__device__ __forceinline__ uint32_t acc_count_small(uint32_t v) {
    return __float_as_uint(__fadd_rn(__uint_as_float(v), 8388608.0f)) - MAGIC_2P23_BITS;
}

}  // namespace snp
