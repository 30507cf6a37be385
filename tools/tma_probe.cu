// tma_probe.cu — TMA load throughput per SM on B200 for the packed-operand access patterns of
// the LD kernel.  148 CTAs, one producer thread streaming 16 KB stages into
// an NP-deep ring, one consumer thread releasing them at once (no compute), from an
// L2-resident 64 MB packed matrix (32,768 rows x 2 KB, the LD-32K operand).  Modes:
//   0  two 2-D boxes {16 words, 128 rows}, 64B swizzle, 2 KB row pitch (the kernel today)
//   1  one 2-D box {32 words, 128 rows}, 128B swizzle, 2 KB pitch (128-byte rows)
//   2  two 1-D bulk copies of 8 KB from a stage-tiled copy (contiguous 128 x 64 B blocks)
//   3  two 2-D boxes {16 words, 128 rows} over the stage-tiled copy (64-byte pitch)
//   4  one 1-D bulk copy of 16 KB (stage-tiled)
// Not part of the library.  Build: see scripts/gpu_tma_probe.sh.
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>
#include "../paper_conf_ipps_binderlp19_b200/csrc/snp_internal.h"
#include "../paper_conf_ipps_binderlp19_b200/csrc/tc_ptx.cuh"
using namespace snp;

constexpr int ROWS = 32768, PITCH = 2048, NSTG = PITCH / 64, NBLK = ROWS / 128;
constexpr int SLOT = 16384;

__device__ __forceinline__ void bulk_load(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     ptx::smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(ptx::smem_u32(bar))
                 : "memory");
}

template <int MODE, int NP>
__global__ void __launch_bounds__(64, 1) probe(const __grid_constant__ CUtensorMap tm, const uint8_t *tiled, int iters,
                                              long long *out) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint64_t full[NP], empty[NP];
    if (threadIdx.x == 0) {
        for (int i = 0; i < NP; ++i) { ptx::mbar_init(&full[i], 1); ptx::mbar_init(&empty[i], 1); }
        ptx::fence_mbar_init();
    }
    __syncthreads();
    const long long t0 = clock64();
    if (threadIdx.x == 0) {
        int p = 0;
        uint32_t round = 0;
        for (int i = 0; i < iters; ++i) {
            // stage s of tile (a, b): A block a, B block b; the tile sequence strides by the grid
            const int tile = blockIdx.x + (i / NSTG) * gridDim.x, s = i % NSTG;
            const int a = (tile * 7) % NBLK, b = (tile * 13 + 5) % NBLK;
            if (round > 0) ptx::mbar_wait(&empty[p], (round - 1) & 1);
            ptx::mbar_arrive_expect_tx(&full[p], SLOT);
            uint8_t *dst = smem + p * SLOT;
            if (MODE == 0 || MODE == 3) {
                const int ya = MODE == 0 ? a * 128 : (a * NSTG + s) * 128, yb = MODE == 0 ? b * 128 : (b * NSTG + s) * 128;
                const int x = MODE == 0 ? s * 16 : 0;
                ptx::tma_load_2d(dst, &tm, &full[p], x, ya);
                ptx::tma_load_2d(dst + SLOT / 2, &tm, &full[p], x, yb);
            } else if (MODE == 1) {
                ptx::tma_load_2d(dst, &tm, &full[p], (s & ~1) * 16, a * 128);   // 128-byte rows
            } else if (MODE == 2) {
                bulk_load(dst, tiled + ((size_t)a * NSTG + s) * 8192, 8192, &full[p]);
                bulk_load(dst + 8192, tiled + ((size_t)b * NSTG + s) * 8192, 8192, &full[p]);
            } else {
                bulk_load(dst, tiled + ((size_t)a * NSTG + (s & ~1)) * 8192, 16384, &full[p]);
            }
            if (++p == NP) { p = 0; ++round; }
        }
    } else if (threadIdx.x == 32) {
        int p = 0;
        uint32_t round = 0;
        for (int i = 0; i < iters; ++i) {
            ptx::mbar_wait(&full[p], round & 1);
            ptx::mbar_arrive(&empty[p]);
            if (++p == NP) { p = 0; ++round; }
        }
        out[blockIdx.x] = clock64() - t0;
    }
}

template <int MODE, int NP>
void run(const char *name, const uint32_t *mat, const uint8_t *tiled, long long *d) {
    CUtensorMap tm;
    bool ok;
    if (MODE == 0) ok = make_map_u32_2d(&tm, mat, ROWS, PITCH / 4, 16, 128, CU_TENSOR_MAP_SWIZZLE_64B);
    else if (MODE == 1) ok = make_map_u32_2d(&tm, mat, ROWS, PITCH / 4, 32, 128, CU_TENSOR_MAP_SWIZZLE_128B);
    else ok = make_map_u32_2d(&tm, reinterpret_cast<const uint32_t *>(tiled), (int64_t)ROWS * NSTG, 16, 16, 128,
                              CU_TENSOR_MAP_SWIZZLE_64B);
    if (!ok) { printf("map failed\n"); exit(1); }
    auto k = probe<MODE, NP>;
    const int smem = NP * SLOT;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    const int iters = 32 * 64;
    k<<<148, 64, smem>>>(tm, tiled, iters, d);   // warm (L2 fill)
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0);
    k<<<148, 64, smem>>>(tm, tiled, iters, d);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    cudaError_t err = cudaGetLastError();
    if (err != cudaSuccess) { printf("%s FAILED: %s\n", name, cudaGetErrorString(err)); exit(1); }
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    long long h[148]; cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    double mx = 0; for (int i = 0; i < 148; ++i) mx = h[i] > mx ? h[i] : mx;
    const double bytes = (double)iters * SLOT;
    printf("%-44s NP=%d  %6.1f B/clk/SM (slowest CTA)  %6.0f cyc/16KB stage  chip %6.2f TB/s\n", name, NP, bytes / mx,
           mx / iters, bytes * 148 / (ms * 1e-3) / 1e12);
}

int main() {
    setvbuf(stdout, nullptr, _IONBF, 0);
    uint32_t *mat; uint8_t *tiled; long long *d;
    cudaMalloc(&mat, (size_t)ROWS * PITCH);
    cudaMalloc(&tiled, (size_t)ROWS * PITCH);
    cudaMalloc(&d, 148 * sizeof(long long));
    cudaMemset(mat, 0x5a, (size_t)ROWS * PITCH);
    cudaMemset(tiled, 0xa5, (size_t)ROWS * PITCH);
    run<0, 6>("2D box 64B rows, 2KB pitch (kernel today)", mat, tiled, d);
    run<0, 12>("2D box 64B rows, 2KB pitch (kernel today)", mat, tiled, d);
    run<1, 6>("2D box 128B rows, 2KB pitch", mat, tiled, d);
    run<2, 6>("1D bulk 2 x 8KB, stage-tiled", mat, tiled, d);
    run<3, 6>("2D box 64B rows, 64B pitch (stage-tiled)", mat, tiled, d);
    run<4, 6>("1D bulk 16KB, stage-tiled", mat, tiled, d);
    run<2, 12>("1D bulk 2 x 8KB, stage-tiled", mat, tiled, d);
    return 0;
}
