// pack.cu — a1 (encode + pack, §III, Fig. 2) and a2 (row popcounts, p_A/p_B of P:L44).
//
// Layout written by snp_pack: row r is ldw little-endian uint64 words, sample k at
// bit k%64 of word k/64; bits >= nbits and words >= ceil(nbits/64) are zero.
#include "snp_internal.h"

namespace snp {
namespace {

// One thread builds one uint64 word from 64 genotype bytes.  High bit of each
// byte of `nz` is set iff the byte is non-zero ("non-zero = minor allele").
__device__ __forceinline__ uint32_t nonzero_bits8(uint64_t x) {
    const uint64_t lo7 = 0x7F7F7F7F7F7F7F7FULL;
    uint64_t nz = (((x & lo7) + lo7) | x) & 0x8080808080808080ULL;
    // gather the 8 high bits, byte i -> bit i
    return (uint32_t)(((nz >> 7) * 0x0102040810204080ULL) >> 56);
}

__global__ void pack_vec_kernel(const uint8_t *__restrict__ g, int64_t rows, int64_t nbits,
                                int64_t ldg, uint64_t *__restrict__ packed, int64_t ldw) {
    // grid-stride over (row, word) pairs; g rows are 16-byte aligned here.
    const int64_t total = rows * ldw;
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = t / ldw, w = t - r * ldw;
        const int64_t k0 = w * 64;
        uint64_t word = 0;
        if (k0 < nbits) {
            const uint8_t *src = g + r * ldg + k0;
            const int64_t valid = nbits - k0;   // bytes of this word that are real
            if (valid >= 64) {
                const uint4 *p = reinterpret_cast<const uint4 *>(src);
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    uint4 v = __ldg(p + q);
                    uint64_t lo = ((uint64_t)v.y << 32) | v.x;
                    uint64_t hi = ((uint64_t)v.w << 32) | v.z;
                    word |= (uint64_t)nonzero_bits8(lo) << (16 * q);
                    word |= (uint64_t)nonzero_bits8(hi) << (16 * q + 8);
                }
            } else {
                for (int64_t k = 0; k < valid; ++k)
                    word |= (uint64_t)(src[k] != 0) << k;
            }
        }
        packed[r * ldw + w] = word;
    }
}

__global__ void pack_byte_kernel(const uint8_t *__restrict__ g, int64_t rows, int64_t nbits,
                                 int64_t ldg, uint64_t *__restrict__ packed, int64_t ldw) {
    const int64_t total = rows * ldw;
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = t / ldw, w = t - r * ldw;
        const int64_t k0 = w * 64;
        uint64_t word = 0;
        if (k0 < nbits) {
            const uint8_t *src = g + r * ldg + k0;
            const int64_t valid = nbits - k0 < 64 ? nbits - k0 : 64;
            for (int64_t k = 0; k < valid; ++k) word |= (uint64_t)(src[k] != 0) << k;
        }
        packed[r * ldw + w] = word;
    }
}

// a1 + a2 fused: one warp per row packs the row's words (as pack_*_kernel) and sums their
// popcounts, so the LD step reads the genotype bytes once and skips the row_popc pass.
// Bits past nbits are packed as zero, so the word popcounts need no mask.
template <bool VEC>
__global__ void pack_popc_kernel(const uint8_t *__restrict__ g, int64_t rows, int64_t nbits,
                                 int64_t ldg, uint64_t *__restrict__ packed, int64_t ldw,
                                 uint32_t *__restrict__ popc) {
    // programmatic dependent launch: the bit-GEMM (launched with PDL) may start its setup
    // now; its griddepcontrol.wait still waits for this grid to finish and flush
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const int lane = threadIdx.x & 31;
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int64_t fullw = nbits / 64;            // words entirely inside nbits
    for (int64_t r = warp; r < rows; r += nwarps) {
        uint32_t c = 0;
        int64_t w = lane;
        if (VEC) {
            // two full words per lane per round, all 8 loads issued before any is consumed
            // (memory-level parallelism: the LD step's first kernel is latency-bound otherwise)
            for (; w + 32 < fullw; w += 64) {
                const uint4 *p0 = reinterpret_cast<const uint4 *>(g + r * ldg + w * 64);
                const uint4 *p1 = reinterpret_cast<const uint4 *>(g + r * ldg + (w + 32) * 64);
                uint4 v0[4], v1[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) { v0[q] = __ldg(p0 + q); v1[q] = __ldg(p1 + q); }
                uint64_t a = 0, b = 0;
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    a |= (uint64_t)nonzero_bits8(((uint64_t)v0[q].y << 32) | v0[q].x) << (16 * q);
                    a |= (uint64_t)nonzero_bits8(((uint64_t)v0[q].w << 32) | v0[q].z) << (16 * q + 8);
                    b |= (uint64_t)nonzero_bits8(((uint64_t)v1[q].y << 32) | v1[q].x) << (16 * q);
                    b |= (uint64_t)nonzero_bits8(((uint64_t)v1[q].w << 32) | v1[q].z) << (16 * q + 8);
                }
                packed[r * ldw + w] = a;
                packed[r * ldw + w + 32] = b;
                c += __popcll(a) + __popcll(b);
            }
        }
        for (; w < ldw; w += 32) {
            const int64_t k0 = w * 64;
            uint64_t word = 0;
            if (k0 < nbits) {
                const uint8_t *src = g + r * ldg + k0;
                const int64_t valid = nbits - k0;
                if (VEC && valid >= 64) {
                    const uint4 *p = reinterpret_cast<const uint4 *>(src);
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        uint4 v = __ldg(p + q);
                        uint64_t lo = ((uint64_t)v.y << 32) | v.x;
                        uint64_t hi = ((uint64_t)v.w << 32) | v.z;
                        word |= (uint64_t)nonzero_bits8(lo) << (16 * q);
                        word |= (uint64_t)nonzero_bits8(hi) << (16 * q + 8);
                    }
                } else {
                    const int64_t nb = valid < 64 ? valid : 64;
                    for (int64_t k = 0; k < nb; ++k) word |= (uint64_t)(src[k] != 0) << k;
                }
            }
            packed[r * ldw + w] = word;
            c += __popcll(word);
        }
#pragma unroll
        for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
        if (lane == 0) popc[r] = c;
    }
}

// One warp per row; lanes stride over the row's words; last word masked.
__global__ void row_popc_kernel(const uint64_t *__restrict__ x, int64_t rows, int64_t nbits,
                                int64_t ldw, uint32_t *__restrict__ popc) {
    // programmatic dependent launch: wait for the producer of x (e.g. snp_pack), then let
    // the consumer (the bit-GEMM) start its setup while the popcounts are being computed
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const int lane = threadIdx.x & 31;
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int64_t full = nbits >> 6;          // words fully inside nbits
    const int tail = (int)(nbits & 63);
    for (int64_t r = warp; r < rows; r += nwarps) {
        const uint64_t *row = x + r * ldw;
        uint32_t c = 0;
        for (int64_t w = lane; w < full; w += 32) c += __popcll(__ldg(row + w));
        if (tail && lane == 0) c += __popcll(__ldg(row + full) & ((1ULL << tail) - 1));
#pragma unroll
        for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
        if (lane == 0) popc[r] = c;
    }
}

int grid_for(int64_t work, int threads) {
    int64_t b = (work + threads - 1) / threads;
    const int64_t cap = 148 * 32;
    if (b > cap) b = cap;
    if (b < 1) b = 1;
    return (int)b;
}

}  // namespace

cudaError_t launch_pack(const uint8_t *g, int64_t rows, int64_t nbits, int64_t ldg,
                        uint64_t *packed, int64_t ldw, cudaStream_t s) {
    const int threads = 256;
    const int blocks = grid_for(rows * ldw, threads);
    const bool vec = ((uintptr_t)g % 16 == 0) && (ldg % 16 == 0);
    if (vec)
        pack_vec_kernel<<<blocks, threads, 0, s>>>(g, rows, nbits, ldg, packed, ldw);
    else
        pack_byte_kernel<<<blocks, threads, 0, s>>>(g, rows, nbits, ldg, packed, ldw);
    count_launches(1);
    return cudaGetLastError();
}

cudaError_t launch_pack_popc(const uint8_t *g, int64_t rows, int64_t nbits, int64_t ldg,
                             uint64_t *packed, int64_t ldw, uint32_t *popc, cudaStream_t s) {
    const int threads = 256;
    const int blocks = grid_for(rows * 32, threads);
    const bool vec = ((uintptr_t)g % 16 == 0) && (ldg % 16 == 0);
    if (vec)
        pack_popc_kernel<true><<<blocks, threads, 0, s>>>(g, rows, nbits, ldg, packed, ldw, popc);
    else
        pack_popc_kernel<false><<<blocks, threads, 0, s>>>(g, rows, nbits, ldg, packed, ldw, popc);
    count_launches(1);
    return cudaGetLastError();
}

cudaError_t launch_row_popc(const uint64_t *x, int64_t rows, int64_t nbits, int64_t ldw,
                            uint32_t *popc, cudaStream_t s) {
    const int threads = 256;
    const int blocks = grid_for(rows * 32, threads);
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3((unsigned)blocks);
    cfg.blockDim = dim3((unsigned)threads);
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, row_popc_kernel, x, rows, nbits, ldw, popc);
    count_launches(1);
    if (e != cudaSuccess) return e;
    return cudaGetLastError();
}

}  // namespace snp
