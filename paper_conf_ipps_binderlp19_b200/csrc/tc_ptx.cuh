// tc_ptx.cuh — thin inline-PTX wrappers for sm_100a tcgen05 / TMEM / mbarrier.
// Hand-written (no CUTLASS/CuTe); descriptor bit layouts follow the PTX ISA
// "shared memory matrix descriptor" and "instruction descriptor" for tcgen05.mma.
#pragma once
#include <stdint.h>

namespace snp {
namespace ptx {

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}

// ---------------------------------------------------------------- mbarrier
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t *bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}
// try_wait with a suspend-time hint: the thread sleeps (issuing nothing) until the phase
// completes or ~hint_ns pass, so waiting warps do not steal issue slots from working ones.
__device__ __forceinline__ bool mbar_try_wait_sleep(uint64_t *bar, uint32_t parity, uint32_t hint_ns) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity), "r"(hint_ns)
        : "memory");
    return ok != 0;
}
__device__ __forceinline__ uint64_t globaltimer_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
// Watchdog record (debug aid, one copy per translation unit): [0] fired, [1] block,
// [2] thread, [3] smem address of the barrier, [4] parity.
static __device__ int g_snp_watchdog[8];
static __device__ int g_snp_watchdog_mode;   // 0: trap, 1: record and release all waits

// Wait for the phase with the given parity to complete.  A wait longer than ~4 s
// means a broken pipeline: trap (a launch error) instead of hanging the GPU.
static __device__ __noinline__ void mbar_wait_slow(uint64_t *bar, uint32_t parity) {
    const uint64_t t0 = globaltimer_ns();
    const int mode = g_snp_watchdog_mode;   // read once: no global load per poll
    for (;;) {
#pragma unroll 1
        for (int i = 0; i < 16; ++i)
            if (mbar_try_wait_sleep(bar, parity, 100000u)) return;
        if (globaltimer_ns() - t0 > 4000000000ull) {
            if (mode == 0) __trap();
            if (atomicCAS(&g_snp_watchdog[0], 0, 1) == 0) {
                g_snp_watchdog[1] = blockIdx.x;
                g_snp_watchdog[2] = threadIdx.x;
                g_snp_watchdog[3] = (int)smem_u32(bar);
                g_snp_watchdog[4] = (int)parity;
            }
            return;
        }
        if (mode && *(volatile int *)&g_snp_watchdog[0]) return;
    }
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    if (mbar_try_wait(bar, parity)) return;
    mbar_wait_slow(bar, parity);
}
// Same, for a whole warp that continues with warp-collective (.sync.aligned) tcgen05
// instructions: every lane waits, then the warp is re-converged explicitly.
__device__ __forceinline__ void mbar_wait_warp(uint64_t *bar, uint32_t parity) {
    mbar_wait(bar, parity);
    __syncwarp();
}
// Warp-uniform wait for MMA-issuing warps: the exit condition is a warp vote, so ptxas
// keeps the issuing loop's counters, TMEM addresses and descriptors in uniform registers
// (no per-MMA R2UR conversions; the tcgen05.mma issue path stays on the uniform datapath).
static __device__ __noinline__ void mbar_wait_uniform_slow(uint64_t *bar, uint32_t parity) {
    const uint64_t t0 = globaltimer_ns();
    for (;;) {
#pragma unroll 1
        for (int i = 0; i < 16; ++i)
            if (__all_sync(0xffffffffu, mbar_try_wait_sleep(bar, parity, 100000u))) return;
        if (__any_sync(0xffffffffu, globaltimer_ns() - t0 > 4000000000ull)) __trap();
    }
}
__device__ __forceinline__ void mbar_wait_uniform(uint64_t *bar, uint32_t parity) {
    if (__all_sync(0xffffffffu, mbar_try_wait(bar, parity))) return;
    mbar_wait_uniform_slow(bar, parity);
}
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("{\n\t.reg .b64 st;\n\tmbarrier.arrive.shared::cta.b64 st, [%0];\n\t}" ::"r"(smem_u32(bar))
                 : "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%1], %0;" ::"r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}

// ---------------------------------------------------------------- TMA
__device__ __forceinline__ void prefetch_tensormap(const void *tmap) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(tmap)) : "memory");
}
// 2-D tiled TMA load global -> shared, completion counted on an mbarrier (bytes).
// L2 eviction-priority policy for data read exactly once (a streamed database): evict_first
__device__ __forceinline__ uint64_t l2_policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ void tma_load_2d_hint(void *smem_dst, const void *tmap, uint64_t *bar, int32_t c0,
                                                 int32_t c1, uint64_t policy) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
        " [%0], [%1, {%3, %4}], [%2], %5;" ::"r"(smem_u32(smem_dst)),
        "l"(reinterpret_cast<uint64_t>(tmap)), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "l"(policy)
        : "memory");
}
__device__ __forceinline__ void tma_load_2d(void *smem_dst, const void *tmap, uint64_t *bar, int32_t c0,
                                            int32_t c1) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(
            smem_u32(smem_dst)),
        "l"(reinterpret_cast<uint64_t>(tmap)), "r"(smem_u32(bar)), "r"(c0), "r"(c1)
        : "memory");
}

// ---------------------------------------------------------------- fences
// generic-proxy smem writes -> visible to the async proxy (tensor core reads)
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_before() {
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_after() {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}

// ---------------------------------------------------------------- TMEM
template <int NCOLS>
__device__ __forceinline__ void tmem_alloc(uint32_t *dst_smem) {   // whole warp
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(dst_smem)),
                 "r"(NCOLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::);
}
template <int NCOLS>
__device__ __forceinline__ void tmem_dealloc(uint32_t taddr) {      // whole warp
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(NCOLS));
}

// 32 lanes x 32 bit, 8 consecutive columns: thread t of the warp gets lane (base+t).
__device__ __forceinline__ void tmem_ld8(uint32_t taddr, uint32_t (&v)[8]) {
    __syncwarp();   // warp-collective (.sync.aligned): converge first
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
                   "=r"(v[7])
                 : "r"(taddr));
}
__device__ __forceinline__ void tmem_ld_wait() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

// 32 lanes x 32 bit, 8 consecutive columns written from 8 registers per thread.
__device__ __forceinline__ void tmem_st8(uint32_t taddr, const uint32_t (&v)[8]) {
    __syncwarp();   // warp-collective (.sync.aligned): converge first
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(taddr),
                 "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7])
                 : "memory");
}
__device__ __forceinline__ void tmem_st_wait() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

// 16 / 32 consecutive columns (the kernels' expander and epilogue widths).
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t (&v)[16]) {
    __syncwarp();   // warp-collective (.sync.aligned): converge first
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(
            taddr),
        "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "r"(v[8]),
        "r"(v[9]), "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15])
        : "memory");
}

__device__ __forceinline__ void tmem_st32(uint32_t taddr, const uint32_t (&v)[32]) {
    __syncwarp();   // warp-collective (.sync.aligned): converge first
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
        "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr),
        "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "r"(v[8]),
        "r"(v[9]), "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15]), "r"(v[16]),
        "r"(v[17]), "r"(v[18]), "r"(v[19]), "r"(v[20]), "r"(v[21]), "r"(v[22]), "r"(v[23]), "r"(v[24]),
        "r"(v[25]), "r"(v[26]), "r"(v[27]), "r"(v[28]), "r"(v[29]), "r"(v[30]), "r"(v[31])
        : "memory");
}

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&v)[16]) {
    __syncwarp();   // warp-collective (.sync.aligned): converge first
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
        : "r"(taddr));
}

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&v)[32]) {
    __syncwarp();   // warp-collective (.sync.aligned): converge first
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,"
        "%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]),
          "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]),
          "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
        : "r"(taddr));
}

// ---------------------------------------------------------------- descriptors
// Shared-memory matrix descriptor, K-major, no swizzle ("interleaved" canonical
// layout): core matrices of 8 rows x 16 bytes (rows 16 B apart, 128 B contiguous);
// LBO = byte distance between the two 16-byte K halves of one MMA K-step,
// SBO = byte distance between consecutive 8-row groups.  version = 1 (sm_100).
__device__ __forceinline__ uint64_t smem_desc_kmajor_noswizzle(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    return (uint64_t)((saddr >> 4) & 0x3FFFu) | ((uint64_t)((lbo >> 4) & 0x3FFFu) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFFu) << 32) | (1ull << 46);
}

// Instruction descriptor for kind::i8: D = s32, A = B = u8, both K-major, dense.
// K-major operand in 128B-swizzled rows (TMA SWIZZLE_128B tiles: 8-row groups of 1024 bytes);
// the K offset inside a swizzle atom is added to the start address.  Layout type 2 at bit 61,
// stride (8-row group) 1024 B, version 1 (sm_100).
__device__ __forceinline__ uint64_t smem_desc_kmajor_sw128(uint32_t saddr) {
    return (uint64_t)((saddr >> 4) & 0x3FFFu) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) | (1ull << 46) |
           (2ull << 61);
}

__host__ __device__ constexpr uint32_t idesc_u8_s32(int M, int N) {
    return (2u << 4)                       // c_format = S32
           | (0u << 7) | (0u << 10)        // a/b format = unsigned 8-bit
           | ((uint32_t)(N >> 3) << 17)    // N / 8
           | ((uint32_t)(M >> 4) << 24);   // M / 16
}

// D[tmem] (+)= A[smem desc] * B[smem desc]^T, u8 x u8 -> s32, one CTA.
__device__ __forceinline__ void mma_i8_ss(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                          uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, {%5, %6, %7, %8}, p;\n\t}" ::"r"(tmem_d),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate), "r"(0), "r"(0), "r"(0), "r"(0));
}
// Same with A read from TMEM (tcgen05.mma ... [a_tmem]).
__device__ __forceinline__ void mma_i8_ts(uint32_t tmem_d, uint32_t tmem_a, uint64_t bdesc, uint32_t idesc,
                                          uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, {%5, %6, %7, %8}, p;\n\t}" ::"r"(tmem_d),
        "r"(tmem_a), "l"(bdesc), "r"(idesc), "r"(accumulate), "r"(0), "r"(0), "r"(0), "r"(0));
}

// Four K-steps of tcgen05.mma kind::mxf4 (block32 scales) with A from TMEM, then a
// commit to `bar`, issued by the elect.sync leader of a converged warp (the whole warp
// must call it; the wrapper re-converges first, so the leader is always the same lane:
// tcgen05.commit only tracks the async operations of the thread that executes it).  K-step i uses A columns a0 + 8 i and B descriptor b0 + i * bstep
// (descriptor start-address field, 16-byte units).  The first MMA accumulates iff
// `accumulate`; the other three always accumulate.
__device__ __forceinline__ void mma4_mxf4_ts_commit(uint32_t d, uint32_t a0, uint64_t b0, uint32_t bstep,
                                                    uint32_t idesc, uint32_t accumulate, uint32_t sfa,
                                                    uint32_t sfb, uint64_t *bar) {
    __syncwarp();   // warp-collective (.sync.aligned / elect.sync): converge first
    const uint64_t b1 = b0 + bstep, b2 = b0 + 2 * bstep, b3 = b0 + 3 * bstep;
    asm volatile(
        "{\n\t.reg .pred e, p, t;\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "setp.ne.b32 p, %9, 0;\n\t"
        "setp.eq.b32 t, 0, 0;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [%1], %5, %10, [%11], [%12], p;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [%2], %6, %10, [%11], [%12], t;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [%3], %7, %10, [%11], [%12], t;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [%4], %8, %10, [%11], [%12], t;\n\t"
        "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%13];\n\t}" ::"r"(d),
        "r"(a0), "r"(a0 + 8), "r"(a0 + 16), "r"(a0 + 24), "l"(b0), "l"(b1), "l"(b2), "l"(b3), "r"(accumulate),
        "r"(idesc), "r"(sfa), "r"(sfb), "r"(smem_u32(bar))
        : "memory");
}
// Eight K-steps (K = 512 nibbles) of tcgen05.mma kind::mxf4 with A from TMEM (columns
// a0 + 8 i) and B descriptors b0 + i * bstep, then a commit to `bar`; one elected lane.
__device__ __forceinline__ void mma8_mxf4_ts_commit(uint32_t d, uint32_t a0, uint64_t b0, uint32_t bstep,
                                                    uint32_t idesc, uint32_t accumulate, uint32_t sfa,
                                                    uint32_t sfb, uint64_t *bar) {
    __syncwarp();   // warp-collective (.sync.aligned / elect.sync): converge first
    asm volatile(
        "{\n\t.reg .pred e, p, t;\n\t.reg .b64 bd;\n\t.reg .b32 ad;\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "setp.ne.b32 p, %5, 0;\n\t"
        "setp.eq.b32 t, 0, 0;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [%1], %2, %4, [%6], [%7], p;\n\t"
        "add.u32 ad, %1, 8;  add.u64 bd, %2, %3;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [ad], bd, %4, [%6], [%7], t;\n\t"
        "add.u32 ad, ad, 8;  add.u64 bd, bd, %3;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [ad], bd, %4, [%6], [%7], t;\n\t"
        "add.u32 ad, ad, 8;  add.u64 bd, bd, %3;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [ad], bd, %4, [%6], [%7], t;\n\t"
        "add.u32 ad, ad, 8;  add.u64 bd, bd, %3;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [ad], bd, %4, [%6], [%7], t;\n\t"
        "add.u32 ad, ad, 8;  add.u64 bd, bd, %3;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [ad], bd, %4, [%6], [%7], t;\n\t"
        "add.u32 ad, ad, 8;  add.u64 bd, bd, %3;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [ad], bd, %4, [%6], [%7], t;\n\t"
        "add.u32 ad, ad, 8;  add.u64 bd, bd, %3;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [ad], bd, %4, [%6], [%7], t;\n\t"
        "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%8];\n\t}" ::"r"(d),
        "r"(a0), "l"(b0), "l"((uint64_t)bstep), "r"(idesc), "r"(accumulate), "r"(sfa), "r"(sfb),
        "r"(smem_u32(bar))
        : "memory");
}

// Four K-steps of tcgen05.mma kind::mxf4 (A from TMEM) without a commit; one elected lane.
__device__ __forceinline__ void mma4_mxf4_ts(uint32_t d, uint32_t a0, uint64_t b0, uint32_t bstep, uint32_t idesc,
                                             uint32_t accumulate, uint32_t sfa, uint32_t sfb) {
    __syncwarp();   // warp-collective (.sync.aligned / elect.sync): converge first
    const uint64_t b1 = b0 + bstep, b2 = b0 + 2 * bstep, b3 = b0 + 3 * bstep;
    asm volatile(
        "{\n\t.reg .pred e, p, t;\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "setp.ne.b32 p, %9, 0;\n\t"
        "setp.eq.b32 t, 0, 0;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [%1], %5, %10, [%11], [%12], p;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [%2], %6, %10, [%11], [%12], t;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [%3], %7, %10, [%11], [%12], t;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [%4], %8, %10, [%11], [%12], t;\n\t}" ::"r"(d),
        "r"(a0), "r"(a0 + 8), "r"(a0 + 16), "r"(a0 + 24), "l"(b0), "l"(b1), "l"(b2), "l"(b3), "r"(accumulate),
        "r"(idesc), "r"(sfa), "r"(sfb)
        : "memory");
}

// One tcgen05.mma kind::mxf4 (block32 scales, A from TMEM) issued by the elect.sync
// leader of a converged warp; with warp-uniform operands ptxas emits a single uniform
// UTCOMMA.  accumulate = 0 overwrites D.
__device__ __forceinline__ void mma_mxf4_ts(uint32_t d, uint32_t a, uint64_t b, uint32_t idesc, uint32_t accumulate,
                                            uint32_t sfa, uint32_t sfb) {
    asm volatile(
        "{\n\t.reg .pred e, p;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [%1], %2, %3, [%5], [%6], p;\n\t}" ::"r"(d),
        "r"(a), "l"(b), "r"(idesc), "r"(accumulate), "r"(sfa), "r"(sfb)
        : "memory");
}
// The same MMA without its own elect.sync: for a block of MMAs issued by one already-elected
// lane (one elect per stage instead of one per instruction).
__device__ __forceinline__ void mma_mxf4_ts_one(uint32_t d, uint32_t a, uint64_t b, uint32_t idesc, uint32_t accumulate,
                                                uint32_t sfa, uint32_t sfb) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::mxf4.block_scale.block32 [%0], [%1], %2, %3, [%5], [%6], p;\n\t}" ::"r"(d),
        "r"(a), "l"(b), "r"(idesc), "r"(accumulate), "r"(sfa), "r"(sfb)
        : "memory");
}
// tcgen05.commit by the calling thread alone (the thread that issued the MMAs it tracks).
__device__ __forceinline__ void mma_commit_one(uint64_t *bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
                 : "memory");
}
// elect.sync: true in exactly one lane of the (converged) warp.
__device__ __forceinline__ bool elect_one() {
    uint32_t r;
    asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\tselp.u32 %0, 1, 0, e;\n\t}" : "=r"(r));
    return r != 0;
}
// tcgen05.commit to an mbarrier by the elect.sync leader (uniform UTCBAR).
__device__ __forceinline__ void mma_commit_uniform(uint64_t *bar) {
    asm volatile(
        "{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(smem_u32(bar))
        : "memory");
}

// Commit by one elected lane of a converged warp.
__device__ __forceinline__ void mma_commit_elect(uint64_t *bar) {
    __syncwarp();   // warp-collective (.sync.aligned / elect.sync): converge first
    asm volatile(
        "{\n\t.reg .pred e;\n\t{ .reg .b32 ln; mov.u32 ln, %%laneid; setp.eq.u32 e, ln, 0; }\n\t"
        "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(smem_u32(bar))
        : "memory");
}

// Arrive on an mbarrier when all previously issued tcgen05.mma of this thread finish.
__device__ __forceinline__ void mma_commit(uint64_t *bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                     smem_u32(bar))
                 : "memory");
}

}  // namespace ptx
}  // namespace snp
