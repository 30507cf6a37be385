// alu_probe.cu — instruction-throughput microbenchmark of the CUDA-core bit-GEMM's pipes
// (POPC, LOP3, IADD3), following the paper's §V.D method: the same loop is
// run by a growing number of thread groups and
//     throughput = (#instructions in the loop x iterations) x N_T x N_grp
//                  / (clock frequency x execution time),
// with combined, non-reducible chains (c = popc(a & c), c += a & c) exposing which
// instructions share a pipeline.  Here the clock is read on the device (clock64 per
// CTA), so the result comes out directly in instructions per clock per SM, and the
// kernel bodies are checked in SASS (cuobjdump) to contain the intended mnemonics.
//
// Output: one line per mix, "<mix>  <ops/clk/SM>  <ops/s at the measured clock>", and a
// final JSON line with the POPC-pipe peak used by bench.py's CUDA-core roofline.
// Not part of the library.
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

constexpr int CHAINS = 8;      // independent dependency chains per thread (covers latency)
constexpr int UNROLL = 16;

// MIX 0: POPC only      c_i = popc(c_i ^ a)        -> 1 POPC + 1 LOP3 per step
// MIX 1: LOP3 only      c_i = (c_i & a) ^ b        -> 1 LOP3 per step (one 3-input op)
// MIX 2: IADD3 only     c_i = c_i + a + b          -> 1 IADD3 per step
// MIX 3: paper kernel   c_i += popc(x_i & c_i+1)   -> 1 LOP3 + 1 POPC + 1 IADD3 per step
//                       (the AND operand comes from another chain, so nothing folds)
template <int MIX>
__global__ void alu_kernel(int iters, uint32_t seed, uint32_t *sink, long long *cycles) {
    uint32_t c[CHAINS], x[CHAINS];
    const uint32_t a = seed * 2654435761u + threadIdx.x, b = a ^ 0x9e3779b9u;
#pragma unroll
    for (int i = 0; i < CHAINS; ++i) {
        c[i] = a + 7u * i;
        x[i] = b * (i + 3);
    }
    __syncthreads();
    const long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int u = 0; u < UNROLL; ++u) {
#pragma unroll
            for (int i = 0; i < CHAINS; ++i) {
                if (MIX == 0) {
                    c[i] = __popc(c[i] ^ x[i]);
                } else if (MIX == 1) {
                    uint32_t r;
                    asm volatile("lop3.b32 %0, %1, %2, %3, 0x6a;" : "=r"(r) : "r"(c[i]), "r"(x[i]), "r"(a));
                    c[i] = r;
                } else if (MIX == 2) {
                    asm volatile("add.u32 %0, %0, %1;\n\tadd.u32 %0, %0, %2;" : "+r"(c[i]) : "r"(x[i]), "r"(a));
                } else {
                    c[i] += __popc(x[i] & c[(i + 1) % CHAINS]);   // operand from another chain: no folding
                }
            }
        }
    }
    __syncthreads();
    const long long t1 = clock64();
    uint32_t s = 0;
#pragma unroll
    for (int i = 0; i < CHAINS; ++i) s ^= c[i] ^ x[i];
    if (s == 0x12345678u) sink[threadIdx.x] = s;   // keep the chains alive
    if (threadIdx.x == 0) cycles[blockIdx.x] = t1 - t0;
}

template <int MIX>
double run(const char *name, int nsm, int ctas_per_sm, int threads, double clk_ghz) {
    const int iters = 2048;
    const int grid = nsm * ctas_per_sm;
    uint32_t *sink;
    long long *cyc;
    cudaMalloc(&sink, 1024 * sizeof(uint32_t));
    cudaMalloc(&cyc, grid * sizeof(long long));
    alu_kernel<MIX><<<grid, threads>>>(16, 1, sink, cyc);   // warm-up
    cudaDeviceSynchronize();
    alu_kernel<MIX><<<grid, threads>>>(iters, 1, sink, cyc);
    cudaDeviceSynchronize();
    long long *h = new long long[grid];
    cudaMemcpy(h, cyc, grid * sizeof(long long), cudaMemcpyDeviceToHost);
    long long mx = 0;
    for (int i = 0; i < grid; ++i) mx = h[i] > mx ? h[i] : mx;
    delete[] h;
    cudaFree(sink);
    cudaFree(cyc);
    const double steps = (double)iters * UNROLL * CHAINS * threads * ctas_per_sm;   // per SM
    const double per_clk = steps / (double)mx;                                      // loop steps / clk / SM
    printf("%-34s %4d thr x %d CTA/SM  %7.2f steps/clk/SM  (%.3e steps/s device at %.0f MHz)\n", name, threads,
           ctas_per_sm, per_clk, per_clk * nsm * clk_ghz * 1e9, clk_ghz * 1e3);
    return per_clk;
}

int main() {
    cudaDeviceProp p;
    cudaGetDeviceProperties(&p, 0);
    const int nsm = p.multiProcessorCount;
    int clk_khz = 0;
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    const double ghz = clk_khz / 1e6;
    printf("# %s, %d SMs, max SM clock %.0f MHz\n", p.name, nsm, ghz * 1e3);
    double popc = 0, lop = 0, add = 0, mix = 0;
    // thread groups per SM from 1 warp to full occupancy (paper: N_grp up to N_cl x L_fn)
    const int thr[] = {32, 128, 256, 512, 1024};
    for (int t : thr) {
        const double v = run<0>("POPC+LOP3 chain  popc(c^x)", nsm, 1, t, ghz);
        popc = v > popc ? v : popc;
    }
    for (int t : thr) {
        const double v = run<1>("LOP3 chain  (c&x)^a", nsm, 1, t, ghz);
        lop = v > lop ? v : lop;
    }
    for (int t : thr) {
        const double v = run<2>("IADD3 chain  c+x+a", nsm, 1, t, ghz);
        add = v > add ? v : add;
    }
    for (int t : thr) {
        const double v = run<3>("kernel mix  c+=popc(x&c')", nsm, 1, t, ghz);
        mix = v > mix ? v : mix;
    }
    // POPC-chain steps are (1 POPC + 1 LOP3); the POPC pipe rate is the step rate while
    // LOP3 has spare throughput (checked by the LOP3-only line).
    printf("{\"popc_per_clk_sm\": %.2f, \"lop3_per_clk_sm\": %.2f, \"iadd_pairs_per_clk_sm\": %.2f, "
           "\"kernel_mix_steps_per_clk_sm\": %.2f, \"sms\": %d, \"sm_max_mhz\": %.0f, "
           "\"popc_cmp_per_s_at_max\": %.4e}\n",
           popc, lop, add, mix, nsm, ghz * 1e3, popc * 32.0 * nsm * ghz * 1e9);
    return 0;
}
