// best.cu — a6: per-query best match over a FastID count matrix.
//
// P:L58 (§II.B): "No set bits in the result signifies a positive match"; P:L62:
// greater counts are less likely matches.  So the decision statistic is the row
// minimum; ties go to the lowest database index (reading R4).
//
// Keys (count << 32 | j) are reduced with a 64-bit min: the smallest key is the
// smallest count and, among equal counts, the lowest j.  best_index doubles as
// the key scratch (init -> per-block atomicMin -> finalize), so nothing is
// allocated.  HBM-bound: one coalesced 128-bit read of the count matrix.
#include "snp_internal.h"

namespace snp {
namespace {

constexpr int BT = 256;
constexpr int PER_BLOCK = BT * 32;   // elements of one row per block

__global__ void best_init(int64_t nq, unsigned long long *keys) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nq;
         i += (int64_t)gridDim.x * blockDim.x)
        keys[i] = ~0ULL;
}

__device__ __forceinline__ unsigned long long kmin(unsigned long long a, unsigned long long b) {
    return a < b ? a : b;
}

__global__ void __launch_bounds__(BT) best_reduce(const uint32_t *__restrict__ c, int64_t nd,
                                                  int64_t ldo, int64_t jbase, unsigned long long *keys) {
    const int64_t i = blockIdx.y;
    const int64_t j0 = (int64_t)blockIdx.x * PER_BLOCK;
    const int64_t j1 = j0 + PER_BLOCK < nd ? j0 + PER_BLOCK : nd;
    const uint32_t *row = c + i * ldo;
    unsigned long long best = ~0ULL;
    const bool vec = (((uintptr_t)(row + j0)) % 16 == 0);
    if (vec) {
        const int64_t nv = (j1 - j0) / 4;
        const uint4 *p = reinterpret_cast<const uint4 *>(row + j0);
        for (int64_t v = threadIdx.x; v < nv; v += BT) {
            const uint4 x = __ldg(p + v);
            const unsigned long long j = (unsigned long long)(jbase + j0 + 4 * v);
            best = kmin(best, ((unsigned long long)x.x << 32) | j);
            best = kmin(best, ((unsigned long long)x.y << 32) | (j + 1));
            best = kmin(best, ((unsigned long long)x.z << 32) | (j + 2));
            best = kmin(best, ((unsigned long long)x.w << 32) | (j + 3));
        }
        for (int64_t j = j0 + 4 * nv + threadIdx.x; j < j1; j += BT)
            best = kmin(best, ((unsigned long long)row[j] << 32) | (unsigned long long)(jbase + j));
    } else {
        for (int64_t j = j0 + threadIdx.x; j < j1; j += BT)
            best = kmin(best, ((unsigned long long)row[j] << 32) | (unsigned long long)(jbase + j));
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) best = kmin(best, __shfl_xor_sync(0xffffffffu, best, o));
    __shared__ unsigned long long red[BT / 32];
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = best;
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int w = 1; w < BT / 32; ++w) best = kmin(best, red[w]);
        atomicMin(keys + i, best);
    }
}

__global__ void best_finalize(const unsigned long long *keys, int64_t nq, int64_t index_base,
                              uint32_t *best_count, int64_t *best_index) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nq;
         i += (int64_t)gridDim.x * blockDim.x) {
        const unsigned long long k = keys[i];   // read before best_index (may alias keys) is written
        if (k == ~0ULL) {
            best_count[i] = 0xffffffffu;
            best_index[i] = -1;
        } else {
            best_count[i] = (uint32_t)(k >> 32);
            best_index[i] = (int64_t)(k & 0xffffffffULL) + index_base;
        }
    }
}

int small_grid(int64_t n) { return (int)((n + 255) / 256 < 1024 ? (n + 255) / 256 : 1024); }

}  // namespace

cudaError_t launch_best_init(unsigned long long *keys, int64_t n, cudaStream_t s) {
    best_init<<<small_grid(n), 256, 0, s>>>(n, keys);
    count_launches(1);
    return cudaGetLastError();
}

cudaError_t launch_best_reduce(const uint32_t *counts, int64_t nq, int64_t nd, int64_t ldo, int64_t jbase,
                               unsigned long long *keys, cudaStream_t s) {
    if (nd <= 0) return cudaSuccess;
    const int64_t gx = (nd + PER_BLOCK - 1) / PER_BLOCK;
    int64_t done = 0;
    while (done < nq) {   // gridDim.y <= 65535
        const int64_t chunk = nq - done < 65535 ? nq - done : 65535;
        dim3 grid((unsigned)gx, (unsigned)chunk);
        best_reduce<<<grid, BT, 0, s>>>(counts + done * ldo, nd, ldo, jbase, keys + done);
        count_launches(1);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        done += chunk;
    }
    return cudaSuccess;
}

cudaError_t launch_best_finalize(const unsigned long long *keys, int64_t nq, int64_t index_base,
                                 uint32_t *best_count, int64_t *best_index, cudaStream_t s) {
    best_finalize<<<small_grid(nq), 256, 0, s>>>(keys, nq, index_base, best_count, best_index);
    count_launches(1);
    return cudaGetLastError();
}

// snp_fastid_best: best_index doubles as the key scratch, so nothing is allocated.
cudaError_t launch_best(const uint32_t *counts, int64_t nq, int64_t nd, int64_t ldo,
                        int64_t index_base, uint32_t *best_count, int64_t *best_index,
                        cudaStream_t s) {
    unsigned long long *keys = reinterpret_cast<unsigned long long *>(best_index);
    cudaError_t e = launch_best_init(keys, nq, s);
    if (e != cudaSuccess) return e;
    if ((e = launch_best_reduce(counts, nq, nd, ldo, 0, keys, s)) != cudaSuccess) return e;
    return launch_best_finalize(keys, nq, index_base, best_count, best_index, s);
}

}  // namespace snp
