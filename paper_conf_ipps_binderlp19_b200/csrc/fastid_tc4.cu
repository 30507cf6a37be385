// fastid_tc4.cu — shape dispatch between the two stage sizes of the FastID tcgen05 kernel
// (fastid_tc4_impl.cuh, compiled as fastid_tc4_k512.cu and fastid_tc4_k1024.cu): a7 of
// SURVEY §8a, from the measured sweep (profiles/round2/sweep_kbits.txt).
#include "snp_internal.h"

#include <cstdlib>
#include <cstring>

namespace snp {

int fastid_bn_k512(int64_t m, int64_t nbits);
bool fastid_tc4_supported_k512(int64_t m, int64_t n, int64_t nbits);
cudaError_t launch_fastid_tc4_k512(const GemmArgs &a, int epi, cudaStream_t s);
size_t fastid_search_tc4_ws_bytes_k512(int64_t nq, int nops);
cudaError_t launch_fastid_search_tc4_k512(const SearchArgs &a, cudaStream_t s);
int fastid_bn_k1024(int64_t m, int64_t nbits);
bool fastid_tc4_supported_k1024(int64_t m, int64_t n, int64_t nbits);
cudaError_t launch_fastid_tc4_k1024(const GemmArgs &a, int epi, cudaStream_t s);
cudaError_t launch_fastid_search_tc4_k1024(const SearchArgs &a, cudaStream_t s);

namespace {
// 1024-bit stages wherever they fit: measured equal (FastID-1M, counts + best, 64 queries:
// 0.1833 vs 0.1840 ms) or 10-30 % faster (few-query searches) than 512-bit stages
// (profiles/round2/sweep_kbits.txt).  SNP_FASTID_KBITS=512|1024 forces one (A/B hook).
bool use_k1024(int64_t nq, int64_t nbits, bool writes_counts) {
    const char *e = std::getenv("SNP_FASTID_KBITS");
    if (e && !std::strcmp(e, "512")) return false;
    const bool ok = fastid_tc4_supported_k1024(nq, 1 << 20, nbits);
    if (e && !std::strcmp(e, "1024")) return ok;
    (void)writes_counts;
    return ok;
}
}  // namespace

int fastid_bn(int64_t m, int64_t nbits) { return fastid_bn_k512(m, nbits); }

bool fastid_tc4_supported(int64_t m, int64_t n, int64_t nbits) { return fastid_tc4_supported_k512(m, n, nbits); }

// The 1024-bit instantiation has 2 TMEM A stages, so only its 2-expander-group kernels
// (database popcounts given, compile-time ops) exist; it answers cudaErrorNotSupported
// (before launching anything) for the others, which then run with 512-bit stages.
cudaError_t launch_fastid_tc4(const GemmArgs &a, int epi, cudaStream_t s) {
    if (use_k1024(a.m, a.nbits, true) && fastid_tc4_supported_k1024(a.m, a.n, a.nbits)) {
        const cudaError_t e = launch_fastid_tc4_k1024(a, epi, s);
        if (e != cudaErrorNotSupported) return e;
    }
    return launch_fastid_tc4_k512(a, epi, s);
}

size_t fastid_search_tc4_ws_bytes(int64_t nq, int nops) { return fastid_search_tc4_ws_bytes_k512(nq, nops); }

cudaError_t launch_fastid_search_tc4(const SearchArgs &a, cudaStream_t s) {
    bool counts = false;
    for (int j = 0; j < a.nops; ++j) counts = counts || a.counts[j] != nullptr;
    if (use_k1024(a.nq, a.nbits, counts) && fastid_tc4_supported_k1024(a.nq, a.nd, a.nbits)) {
        const cudaError_t e = launch_fastid_search_tc4_k1024(a, s);
        if (e != cudaErrorNotSupported) return e;
    }
    return launch_fastid_search_tc4_k512(a, s);
}

}  // namespace snp
