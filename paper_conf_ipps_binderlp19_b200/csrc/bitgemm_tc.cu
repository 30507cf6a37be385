// bitgemm_tc.cu — tcgen05 kind::i8 tensor-core variant (placeholder until implemented).
#include "snp_internal.h"

namespace snp {
size_t tc_workspace_bytes(int64_t, int64_t, int64_t) { return 0; }
bool tc_supported(int64_t, int64_t, int64_t) { return false; }
cudaError_t launch_bitgemm_tc(const GemmArgs &, int, void *, size_t, cudaStream_t) {
    return cudaErrorNotSupported;
}
}  // namespace snp
