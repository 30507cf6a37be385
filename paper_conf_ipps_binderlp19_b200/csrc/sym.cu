// sym.cu — f3 packed-triangle helpers (LD as a GEMM of two equal inputs,
// P:L46 §II.A, Fig. 1): scatter the dense 128 x 128 tiles of snp_ld_sym (row-major upper
// triangle of the tile grid, include/snp.h) into a full row-major m x m matrix, every
// off-diagonal tile also mirrored (all LD outputs are symmetric: nAB, r2, D').
// HBM-bound data movement: one 64 KB tile read, one or two 64 KB writes, both coalesced
// (the mirror goes through a 32 x 33 shared-memory transpose).
#include "snp_internal.h"

namespace snp {
namespace {

constexpr int T = SYM_TILE;   // 128

__global__ void __launch_bounds__(256) sym_unpack_kernel(const uint32_t *__restrict__ tiles, int64_t m,
                                                         int64_t tlo, uint32_t *__restrict__ out, int64_t ldo) {
    __shared__ uint32_t tr[8][32][33];
    const int64_t u = blockIdx.x;                // tile of the call
    uint32_t I, J;
    tri_decode((m + T - 1) / T, tlo + u, I, J);
    const int64_t r0 = (int64_t)I * T, c0 = (int64_t)J * T;
    const uint32_t *src = tiles + u * (T * T);
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    // normal orientation: warp w copies rows w, w + 8, ... (128 columns = 4 x 32 lanes)
    for (int i = w; i < T; i += 8) {
        const int64_t row = r0 + i;
        if (row >= m) break;
#pragma unroll
        for (int cc = 0; cc < T; cc += 32) {
            const int64_t col = c0 + cc + lane;
            if (col < m) out[row * ldo + col] = src[i * T + cc + lane];
        }
    }
    if (I == J) return;
    // mirror: block (bi, bj) of 32 x 32 is transposed through shared memory by warp w
    for (int blk = w; blk < 16; blk += 8) {
        const int bi = blk >> 2, bj = blk & 3;
#pragma unroll 4
        for (int i = 0; i < 32; ++i) tr[w][i][lane] = src[(bi * 32 + i) * T + bj * 32 + lane];
        __syncwarp();
        // out[c0 + bj*32 + j][r0 + bi*32 + lane] = tile[bi*32 + lane][bj*32 + j]
        for (int j = 0; j < 32; ++j) {
            const int64_t row = c0 + bj * 32 + j, col = r0 + bi * 32 + lane;
            if (row < m && col < m) out[row * ldo + col] = tr[w][lane][j];
        }
        __syncwarp();
    }
}

}  // namespace

cudaError_t launch_sym_unpack(const uint32_t *tiles, int64_t m, int64_t tlo, int64_t ntiles, uint32_t *out,
                              int64_t ldo, cudaStream_t s) {
    if (ntiles <= 0) return cudaSuccess;
    if (ntiles > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    sym_unpack_kernel<<<(unsigned)ntiles, 256, 0, s>>>(tiles, m, tlo, out, ldo);
    count_launches(1);
    return cudaGetLastError();
}

}  // namespace snp
