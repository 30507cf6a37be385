// store_probe.cu — write bandwidth of the FastID count-matrix store pattern (out[q][d], lane =
// database row): each warp stores 128-byte row segments of NQ query rows `ldo` words apart, the
// CTAs sweeping the database together, as the FastID epilogues do.  Compares row strides
// (4 MB: FastID-1M; 80 MB: FastID-20M) against a dense stream to tell whether the scattered
// pattern itself caps the epilogue's store rate.  Not part of the library.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void store_kernel(uint32_t *out, int64_t ldo, int nq, int64_t ncols, int64_t tiles_per_cta, int cs) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;   // 8 warps: 4 lane quarters x 2 query halves
    const int q0 = (warp >> 2) * (nq / 2);
    for (int64_t tl = 0; tl < tiles_per_cta; ++tl) {
        const int64_t tile = blockIdx.x + tl * gridDim.x;
        const int64_t d = tile * 128 + (warp & 3) * 32 + lane;
        if (d >= ncols) break;
        uint32_t *p = out + (int64_t)q0 * ldo + d;
#pragma unroll 4
        for (int u = 0; u < nq / 2; ++u) {
            if (cs) __stcs(p, (uint32_t)(d ^ u));
            else *p = (uint32_t)(d ^ u);
            p += ldo;
        }
    }
}

int main() {
    const int nsm = 148;
    const size_t bytes = (size_t)24 << 30;   // 24 GB buffer
    uint32_t *buf;
    if (cudaMalloc(&buf, bytes) != cudaSuccess) { printf("alloc failed\n"); return 1; }
    struct Case { const char *name; int nq; int64_t ncols; };
    const Case cases[] = {{"FastID-1M-like  (64 q x 1M, 2 ops as 128 rows)", 128, 1000000},
                          {"FastID-20M-like (256 rows of 20M)", 256, 20000000},
                          {"FastID-20M-like (2048 rows of 2.5M)", 2048, 2500000}};
    for (const Case &c : cases) {
        for (int cs = 0; cs < 2; ++cs) {
            const int64_t ldo = c.ncols;
            const int64_t total = (int64_t)c.nq * ldo;
            if ((size_t)total * 4 > bytes) continue;
            const int64_t tiles = (c.ncols + 127) / 128;
            const int64_t tpc = (tiles + nsm - 1) / nsm;
            store_kernel<<<nsm, 256>>>(buf, ldo, c.nq, c.ncols, tpc, cs);
            cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
            cudaEventRecord(e0);
            for (int r = 0; r < 3; ++r) store_kernel<<<nsm, 256>>>(buf, ldo, c.nq, c.ncols, tpc, cs);
            cudaEventRecord(e1); cudaEventSynchronize(e1);
            float ms; cudaEventElapsedTime(&ms, e0, e1); ms /= 3;
            printf("%-48s %s  %.2f GB in %.3f ms = %.0f GB/s  %s\n", c.name, cs ? ".cs" : ".wb", total * 4 / 1e9, ms,
                   total * 4 / (ms * 1e6), cudaGetErrorString(cudaGetLastError()));
        }
    }
    // dense reference: the same bytes as one contiguous stream
    for (int cs = 0; cs < 2; ++cs) {
        const int64_t n = (int64_t)128 * 20000000;   // two rows of n words: 2 x 10.24 GB, each written densely
        store_kernel<<<nsm, 256>>>(buf, n, 2, n, (n / 128 + nsm - 1) / nsm, cs);
        cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
        cudaEventRecord(e0);
        store_kernel<<<nsm, 256>>>(buf, n, 2, n, (n / 128 + nsm - 1) / nsm, cs);
        cudaEventRecord(e1); cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        printf("%-48s %s  %.2f GB in %.3f ms = %.0f GB/s\n", "dense (2 rows, 128 B per warp store)", cs ? ".cs" : ".wb",
               2 * n * 4 / 1e9, ms, 2 * n * 4 / (ms * 1e6));
    }
    return 0;
}
