// threshold.cu — f1, threshold form: every (query, database row) pair whose
// count is <= tau, the forensic decision of P:L58 ("no set bits in the result signifies a
// positive match"; larger counts are less likely matches) with a tolerance tau (tau = 0:
// exact matches only).
//
// A count block [nq][rows] (row stride ldo) is scanned once (coalesced, L2-resident when the
// caller streams the database through a workspace chunk); each warp compacts its lane hits with
// a ballot: one atomicAdd per warp and 32-element run reserves the output slots, each hit lane
// writes its (query, count, global index) triple at base + rank.  The running total keeps counting
// past `capacity`, so the caller learns how many matches exist even when the list is full.
#include "snp_internal.h"

namespace snp {
namespace {

__global__ void __launch_bounds__(256) threshold_compact(const uint32_t *__restrict__ c, int64_t nq, int64_t rows,
                                                         int64_t ldo, int64_t index0, uint32_t tau,
                                                         ThresholdMatch *__restrict__ out, int64_t capacity,
                                                         unsigned long long *__restrict__ total) {
    const int lane = threadIdx.x & 31;
    const int64_t q = blockIdx.y;
    const uint32_t *row = c + q * ldo;
    for (int64_t j0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) & ~31LL; j0 < rows;
         j0 += (int64_t)gridDim.x * blockDim.x) {
        const int64_t j = j0 + lane;
        const uint32_t x = j < rows ? __ldg(row + j) : 0xffffffffu;
        const bool hit = j < rows && x <= tau;
        const uint32_t m = __ballot_sync(0xffffffffu, hit);
        if (!m) continue;
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(total, (unsigned long long)__popc(m));
        base = __shfl_sync(0xffffffffu, base, 0);
        if (hit) {
            const unsigned long long slot = base + (unsigned long long)__popc(m & ((1u << lane) - 1u));
            if (slot < (unsigned long long)capacity) {
                ThresholdMatch t;
                t.query = (uint32_t)q;
                t.count = x;
                t.index = index0 + j;
                out[slot] = t;
            }
        }
    }
}

}  // namespace

cudaError_t launch_threshold_compact(const uint32_t *counts, int64_t nq, int64_t rows, int64_t ldo, int64_t index0,
                                     uint32_t tau, ThresholdMatch *out, int64_t capacity, unsigned long long *total,
                                     cudaStream_t s) {
    if (nq <= 0 || rows <= 0) return cudaSuccess;
    if (nq > 65535) return cudaErrorInvalidConfiguration;
    int64_t bx = (rows + 255) / 256;
    const int64_t cap = 4 * (int64_t)device_sms();   // enough blocks to cover HBM latency
    if (bx * nq > cap * 8) bx = (cap * 8 + nq - 1) / nq;
    if (bx < 1) bx = 1;
    threshold_compact<<<dim3((unsigned)bx, (unsigned)nq), 256, 0, s>>>(counts, nq, rows, ldo, index0, tau, out, capacity,
                                                                      total);
    count_launches(1);
    return cudaGetLastError();
}

}  // namespace snp
