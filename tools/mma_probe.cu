// mma_probe.cu — microbenchmark of tcgen05.mma issue throughput on B200 (one CTA per SM,
// one issuing thread, back-to-back MMAs on garbage operands, clock64 around them).
// Used to pick the tensor-core kernel shapes.  Not part of the library.
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>
#include "../paper_conf_ipps_binderlp19_b200/csrc/tc_ptx.cuh"
using namespace snp;

__host__ __device__ constexpr uint32_t idesc_mxf4(int M, int N) {
    return (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | (1u << 23) | ((uint32_t)(M >> 4) << 24);
}
__device__ __forceinline__ void mma_mxf4_ss(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc, uint32_t sfa, uint32_t sfb) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], %1, %2, %3, [%5], [%6], p;\n\t}"
                 :: "r"(d), "l"(a), "l"(b), "r"(idesc), "r"(acc), "r"(sfa), "r"(sfb));
}
__device__ __forceinline__ void mma_mxf4_ts(uint32_t d, uint32_t a, uint64_t b, uint32_t idesc, uint32_t acc, uint32_t sfa, uint32_t sfb) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [%1], %2, %3, [%5], [%6], p;\n\t}"
                 :: "r"(d), "r"(a), "l"(b), "r"(idesc), "r"(acc), "r"(sfa), "r"(sfb));
}

template <int MODE, int N, int CONTEND = 0, int M = 128>   // MODE 0: mxf4 SS, 1: mxf4 TS, 2: i8 SS, 3: i8 TS
// CONTEND 1: warps 1-4 hammer tcgen05.st into other TMEM columns; 2: tcgen05.ld
__global__ void probe(int iters, long long *out) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ uint64_t bar;
    __shared__ uint32_t slot;
    if (threadIdx.x < 32) ptx::tmem_alloc<512>(&slot);
    if (threadIdx.x == 0) { ptx::mbar_init(&bar, 1); ptx::fence_mbar_init(); }
    ptx::tc_fence_before(); __syncthreads(); ptx::tc_fence_after();
    uint32_t tmem = slot;
    if (threadIdx.x == 0) {
        const uint32_t sa = ptx::smem_u32(sm), sb = sa + 128 * 32;
        const uint64_t ad = ptx::smem_desc_kmajor_noswizzle(sa, 128 * 16, 128);
        const uint64_t bd = ptx::smem_desc_kmajor_noswizzle(sb, N * 16, 128);
        long long t0 = clock64();
        for (int i = 0; i < iters; ++i) {
            if (MODE == 0) mma_mxf4_ss(tmem, ad, bd, idesc_mxf4(M, N), 1, tmem + 480, tmem + 496);
            else if (MODE == 1) mma_mxf4_ts(tmem, tmem + 256 + (i & 7) * 8, bd, idesc_mxf4(M, N), 1, tmem + 480, tmem + 496);
            else if (MODE == 4)   // B walks 8 K-steps x 3 stages of a [3][8][N x 32 B] region (the LD kernel)
                mma_mxf4_ts(tmem, tmem + 256 + (i & 7) * 8,
                            bd + (uint64_t)((((i % 24) / 8) * N * 256 + (i & 7) * N * 32) >> 4), idesc_mxf4(M, N), 1,
                            tmem + 480, tmem + 496);
            else if (MODE == 2) ptx::mma_i8_ss(tmem, ad, bd, ptx::idesc_u8_s32(M, N), 1);
            else ptx::mma_i8_ts(tmem, tmem + 256 + (i & 7) * 8, bd, ptx::idesc_u8_s32(M, N), 1);
        }
        ptx::mma_commit(&bar);
        ptx::mbar_wait(&bar, 0);
        long long t1 = clock64();
        out[blockIdx.x] = t1 - t0;
    } else if (CONTEND && threadIdx.x >= 32 && threadIdx.x < 160) {
        const int w = threadIdx.x >> 5, q = w & 3;
        uint32_t v[8] = {1, 2, 3, 4, 5, 6, 7, 8};
        for (int i = 0; i < iters / 2; ++i) {
            const uint32_t a = tmem + ((uint32_t)(q * 32) << 16) + 384 + (i & 7) * 8;
            if (CONTEND == 1) { ptx::tmem_st8(a, v); ptx::tmem_st_wait(); }
            else { ptx::tmem_ld8(a, v); ptx::tmem_ld_wait(); }
        }
    }
    ptx::tc_fence_before(); __syncthreads();
    if (threadIdx.x < 32) { ptx::tc_fence_after(); ptx::tmem_dealloc<512>(tmem); }
}

// CTA pair (cta_group::2, M = 256 across the pair, each CTA 128 rows x N/2 B rows): the
// leader CTA's thread issues; both CTAs allocate TMEM for the pair.
template <int N, bool SS, bool WALK = false>
__global__ void __cluster_dims__(2, 1, 1) probe2(int iters, long long *out) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ uint64_t bar;
    __shared__ uint32_t slot;
    uint32_t rank;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(ptx::smem_u32(&slot)) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
    }
    if (threadIdx.x == 0) { ptx::mbar_init(&bar, 1); ptx::fence_mbar_init(); }
    ptx::tc_fence_before();
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    ptx::tc_fence_after();
    const uint32_t tmem = slot;
    long long t0 = clock64();
    if (rank == 0 && threadIdx.x < 32) {
        const uint32_t sa = ptx::smem_u32(sm), sb = sa + 128 * 32;
        const uint64_t ad = ptx::smem_desc_kmajor_noswizzle(sa, 128 * 16, 128);
        const uint64_t bd = ptx::smem_desc_kmajor_noswizzle(sb, (N / 2) * 16, 128);
        const uint32_t idesc = idesc_mxf4(256, N);
        for (int i = 0; i < iters; ++i) {
            const uint32_t sfa = tmem + 480, sfb = tmem + 496;
            if (SS)
                asm volatile("{\n\t.reg .pred e, p;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 p, 1, 0;\n\t"
                             "@e tcgen05.mma.cta_group::2.kind::mxf4.block_scale.block32 [%0], %1, %2, %3, [%4], [%5], p;\n\t}"
                             ::"r"(tmem), "l"(ad), "l"(bd), "r"(idesc), "r"(sfa), "r"(sfb) : "memory");
            else
                asm volatile("{\n\t.reg .pred e, p;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 p, 1, 0;\n\t"
                             "@e tcgen05.mma.cta_group::2.kind::mxf4.block_scale.block32 [%0], [%1], %2, %3, [%4], [%5], p;\n\t}"
                             ::"r"(tmem), "r"(tmem + 256 + (i & 7) * 8),
                               "l"(WALK ? bd + (uint64_t)((((i % 24) / 8) * (N / 2) * 256 + (i & 7) * (N / 2) * 32) >> 4) : bd),
                               "r"(idesc), "r"(sfa), "r"(sfb) : "memory");
        }
        asm volatile("{\n\t.reg .pred e;\n\t.reg .b16 m;\n\tmov.b16 m, 3;\n\telect.sync _|e, 0xffffffff;\n\t"
                     "@e tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], m;\n\t}"
                     ::"r"(ptx::smem_u32(&bar)) : "memory");
    }
    if (threadIdx.x == 0) {
        ptx::mbar_wait(&bar, 0);
        out[blockIdx.x] = clock64() - t0;
    }
    ptx::tc_fence_before();
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    if (threadIdx.x < 32) {
        ptx::tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 512;" ::"r"(tmem) : "memory");
    }
}

template <int N, bool SS, bool WALK = false>
void run2(const char *name) {
    long long *d; cudaMalloc(&d, 148 * sizeof(long long));
    const int iters = 4096;
    auto k = probe2<N, SS, WALK>;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    k<<<148, 128, 200 * 1024>>>(iters, d);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0);
    k<<<148, 128, 200 * 1024>>>(iters, d);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    cudaError_t err = cudaGetLastError();
    if (err != cudaSuccess) { printf("%-14s pair M=256 N=%3d FAILED: %s\n", name, N, cudaGetErrorString(err)); exit(1); }
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    long long h[148]; cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    const double cyc = (double)h[0] / iters;
    const double macs_sm = 128.0 * N * 64;   // per SM per pair instruction
    printf("%-14s pair M=256 N=%3d  %7.1f cycles/MMA  %8.1f MAC/clk/SM  %7.0f TMAC/s (event %.3f ms)\n", name, N, cyc,
           macs_sm / cyc, macs_sm * 148 * iters / (ms * 1e-3) / 1e12, ms);
    cudaFree(d);
}

template <int MODE, int N, int CONTEND = 0, int M = 128>
void run(const char *name) {
    long long *d; cudaMalloc(&d, 148 * sizeof(long long));
    const int iters = 4096;
    auto k = probe<MODE, N, CONTEND, M>;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    k<<<148, 192, 200 * 1024>>>(iters, d);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0);
    k<<<148, 192, 200 * 1024>>>(iters, d);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    long long h[148]; cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    cudaError_t err = cudaGetLastError();
    if (err != cudaSuccess) {
        printf("%-14s M=%3d N=%3d  FAILED: %s\n", name, M, N, cudaGetErrorString(err));
        fflush(stdout);
        exit(1);   // a sticky error poisons every later launch
    }
    double cyc = (double)h[0] / iters;
    const int K = (MODE <= 1) ? 64 : 32;
    double macs = (double)M * N * K * iters * 148;
    printf("%-14s M=%3d N=%3d  %7.1f cycles/MMA  %8.1f MAC/clk/SM  %7.0f TMAC/s (event %.3f ms) %s\n", name, M, N, cyc,
           (double)M * N * K / cyc, macs / (ms * 1e-3) / 1e12, ms, err == cudaSuccess ? "" : cudaGetErrorString(err));
    cudaFree(d);
}

int main() {
    setvbuf(stdout, nullptr, _IONBF, 0);
    if (getenv("PAIR_ONLY")) {
        run2<64, false>("mxf4 TS x2"); run2<128, false>("mxf4 TS x2"); run2<256, false>("mxf4 TS x2");
        run2<128, true>("mxf4 SS x2"); run2<256, true>("mxf4 SS x2");
        run2<128, false, true>("mxf4 TS x2 walkB"); run2<256, false, true>("mxf4 TS x2 walkB");
        run<1, 128>("mxf4 TS"); run<1, 256>("mxf4 TS"); run<4, 128>("mxf4 TS walkB");
        return 0;
    }
    run<0, 64>("mxf4 SS"); run<0, 128>("mxf4 SS"); run<0, 256>("mxf4 SS");
    run<1, 64>("mxf4 TS"); run<1, 128>("mxf4 TS"); run<1, 256>("mxf4 TS");
    run<2, 64>("i8 SS"); run<2, 128>("i8 SS"); run<2, 256>("i8 SS");
    run<3, 64>("i8 TS"); run<3, 128>("i8 TS"); run<3, 256>("i8 TS");
    run<1, 64, 1>("mxf4 TS +st"); run<1, 128, 1>("mxf4 TS +st"); run<0, 64, 1>("mxf4 SS +st");
    run<1, 64, 2>("mxf4 TS +ld"); run<0, 64, 2>("mxf4 SS +ld");
    // skinny shapes (few queries): is the per-MMA cost proportional to N below 64?
    run<1, 16>("mxf4 TS"); run<1, 32>("mxf4 TS"); run<1, 48>("mxf4 TS");
    run<0, 16>("mxf4 SS"); run<0, 32>("mxf4 SS");
    run<0, 8, 0, 64>("mxf4 SS"); run<0, 16, 0, 64>("mxf4 SS"); run<0, 32, 0, 64>("mxf4 SS"); run<0, 64, 0, 64>("mxf4 SS");
    run<0, 128, 0, 64>("mxf4 SS"); run<0, 256, 0, 64>("mxf4 SS");
    run<1, 8, 0, 64>("mxf4 TS"); run<1, 16, 0, 64>("mxf4 TS"); run<1, 64, 0, 64>("mxf4 TS"); run<1, 256, 0, 64>("mxf4 TS");
    return 0;
}
