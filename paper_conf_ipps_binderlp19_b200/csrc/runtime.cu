// runtime.cu — per-device host state of the library (include/snp.h: "the only global state
// is a cached device-property record per device"), shared by every launcher:
//   * the SM count of each device (persistent grids are sized to it);
//   * the dynamic shared-memory opt-in of each (device, kernel) pair — a function attribute
//     lives in the device's context, so a second device must be granted it again;
//   * the driver's cuTensorMapEncodeTiled entry point and the 2-D tensor maps (TMA) the
//     tensor-core kernels stream packed rows with.
// All of it is thread-safe (atomics / one mutex around the attribute table).
#include "snp_internal.h"

#include <atomic>
#include <map>
#include <mutex>
#include <utility>

namespace snp {

namespace {
constexpr int MAX_DEVICES = 64;
std::atomic<int> g_sms[MAX_DEVICES];
std::mutex g_attr_mu;
std::map<std::pair<int, const void *>, int> g_attr;   // (device, kernel) -> granted bytes
std::atomic<EncodeTiledFn> g_encode{nullptr};

int current_device() {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0) dev = 0;
    return dev;
}
}  // namespace

int device_sms() {
    const int dev = current_device();
    if (dev >= MAX_DEVICES) {
        int n = 0;
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        return n > 0 ? n : 148;
    }
    int n = g_sms[dev].load(std::memory_order_relaxed);
    if (n <= 0) {
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (n <= 0) n = 148;
        g_sms[dev].store(n, std::memory_order_relaxed);
    }
    return n;
}

cudaError_t ensure_dyn_smem(const void *kernel, int bytes) {
    const std::pair<int, const void *> key{current_device(), kernel};
    std::lock_guard<std::mutex> lock(g_attr_mu);
    auto it = g_attr.find(key);
    if (it != g_attr.end() && it->second >= bytes) return cudaSuccess;
    cudaError_t e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e != cudaSuccess) return e;
    g_attr[key] = bytes;
    return cudaSuccess;
}

EncodeTiledFn tensor_map_encoder() {
    EncodeTiledFn fn = g_encode.load(std::memory_order_acquire);
    if (!fn) {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess) {
            fn = reinterpret_cast<EncodeTiledFn>(p);
            g_encode.store(fn, std::memory_order_release);
        }
    }
    return fn;
}

bool make_map_u32_2d(CUtensorMap *tm, const uint32_t *base, int64_t rows, int64_t ld32, uint32_t box_words,
                     uint32_t box_rows, CUtensorMapSwizzle swizzle, int64_t cols32) {
    EncodeTiledFn enc = tensor_map_encoder();
    if (!enc) return false;
    const cuuint64_t dims[2] = {(cuuint64_t)(cols32 > 0 ? cols32 : ld32), (cuuint64_t)rows};
    const cuuint64_t strides[1] = {(cuuint64_t)ld32 * 4};
    const cuuint32_t box[2] = {box_words, box_rows};
    const cuuint32_t estr[2] = {1, 1};
    return enc(tm, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, const_cast<uint32_t *>(base), dims, strides, box, estr,
               CU_TENSOR_MAP_INTERLEAVE_NONE, swizzle,
#ifdef SNP_TMA_L2_PROMO_NONE
               CU_TENSOR_MAP_L2_PROMOTION_NONE,   // measurement variant
#else
               CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
#endif
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

}  // namespace snp
