// scan_launch.cu -- per-device launch facts shared by every launcher of the library.
//
// cudaFuncSetAttribute (the opt-in to > 48 KiB of dynamic shared memory, non-portable
// cluster sizes) applies to the CURRENT device's context, and SM counts / occupancies are
// device properties, so nothing here may be cached process-wide: a process that drives two
// GPUs (scan_multi.cu's same-process peer path, or a user thread per device) must get the
// opt-in on each of them.  Both caches are keyed by device and guarded by one mutex.
#include <cuda_runtime.h>

#include <cstdlib>
#include <map>
#include <mutex>
#include <utility>

#include "scan_internal.h"

namespace scanb200 {

namespace {
std::mutex g_launch_mu;
std::map<int, int> g_sms;                                    // device -> SM count
std::map<std::pair<int, const void*>, int> g_occ;            // (device, kernel) -> CTAs per SM
}  // namespace

cudaError_t current_device_sms(int* sms) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    std::lock_guard<std::mutex> lk(g_launch_mu);
    auto it = g_sms.find(dev);
    if (it == g_sms.end()) {
        int n = 0;
        e = cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (e != cudaSuccess) return e;
        if (n <= 0) return cudaErrorInvalidDevice;
        it = g_sms.emplace(dev, n).first;
    }
    *sms = it->second;
    return cudaSuccess;
}

cudaError_t kernel_prepare(const void* func, int threads, size_t dyn_smem, bool nonportable_cluster, int* occ) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    std::lock_guard<std::mutex> lk(g_launch_mu);
    const auto key = std::make_pair(dev, func);
    auto it = g_occ.find(key);
    if (it == g_occ.end()) {
        if (dyn_smem > 48 * 1024) {
            e = cudaFuncSetAttribute(func, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dyn_smem);
            if (e != cudaSuccess) return e;
        }
        if (nonportable_cluster) {
            e = cudaFuncSetAttribute(func, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
            if (e != cudaSuccess) return e;
        }
        int o = 0;
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, func, threads, dyn_smem);
        if (e != cudaSuccess) return e;
        if (o < 1) return cudaErrorInvalidConfiguration;
        it = g_occ.emplace(key, o).first;
    }
    if (occ) *occ = it->second;
    return cudaSuccess;
}

cudaError_t launch_persistent(const void* func, void** args, int64_t tiles, int threads, size_t dyn_smem,
                              bool pdl, cudaStream_t s) {
    int occ = 0, sms = 0;
    cudaError_t e = kernel_prepare(func, threads, dyn_smem, false, &occ);
    if (e != cudaSuccess) return e;
    e = current_device_sms(&sms);
    if (e != cudaSuccess) return e;
    if (tiles > 0x7FFFFFFF) return cudaErrorInvalidConfiguration;
    int64_t grid = (int64_t)occ * sms;
    if (grid > tiles) grid = tiles;
    if (grid < 1) return cudaSuccess;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid, 1, 1);
    cfg.blockDim = dim3((unsigned)threads, 1, 1);
    cfg.dynamicSmemBytes = dyn_smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[2];
    int n = 0;
    // the static round robin makes CTA b wait on tiles owned by CTAs of higher index:
    // a cooperative launch guarantees that the whole grid is co-resident (or the launch
    // fails loudly, e.g. inside an SM-limited MPS / green context) instead of relying on
    // nothing else occupying the SMs
    static const bool coop = std::getenv("SCANB200_NO_COOP") == nullptr;   // A/B switch
    if (coop) {
        attr[n].id = cudaLaunchAttributeCooperative;
        attr[n].val.cooperative = 1;
        ++n;
    }
    if (pdl) {
        attr[n].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        attr[n].val.programmaticStreamSerializationAllowed = 1;
        ++n;
    }
    cfg.attrs = attr;
    cfg.numAttrs = n;
    return cudaLaunchKernelExC(&cfg, func, args);
}

}  // namespace scanb200
