// spp_internal.h — launcher interface between the C ABI (api.cu) and the
// format-specific kernel files (cosmo.cu, deepcam.cu).
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

#include <atomic>

#include "spp.h"

namespace spp {

// device properties of the current device (cached per device id)
constexpr int kMaxDevices = 64;
struct DeviceProps {
    int dev = 0;            // device ordinal (< kMaxDevices)
    int sms = 0;
    int smem_optin = 0;     // max dynamic shared memory per CTA (opt-in)
    int smem_per_sm = 0;    // shared memory per SM
    int smem_reserved = 0;  // shared memory the runtime reserves per CTA
    int cc_major = 0, cc_minor = 0;
};
spp_status current_device_props(DeviceProps *out);

// CosmoFlow (cosmo.cu)
size_t cosmo_workspace_bytes(int n);
spp_status cosmo_decode(const void *const *d_src, int n, void *d_dst, const spp_decode_opts &o,
                        cudaStream_t stream);
constexpr int kCosmoLaunches = 2;  // KC0 (unique-value transform) + KC (fused LUT expansion)

// DeepCAM (deepcam.cu)
size_t deepcam_workspace_bytes(int n);
spp_status deepcam_decode(const void *const *d_src, int n, void *d_dst, const spp_decode_opts &o,
                          cudaStream_t stream);
constexpr int kDeepcamLaunches = 2;  // KD0 (header/directory parse) + KD (warp-per-line decode)

// The dynamic shared-memory opt-in is a per-device function attribute: set it
// once per (kernel instance, device), thread-safe (the call is idempotent, so a
// race only repeats it).  Keyed by the kernel itself (a template argument), so
// every kernel instance has its own per-device record.
template <auto Kern>
spp_status set_smem_attr(int smem, const DeviceProps &dp) {
    static std::atomic<int> done[kMaxDevices];
    const auto kern = Kern;
    if (done[dp.dev].load(std::memory_order_acquire) >= smem) return SPP_OK;
    if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess)
        return SPP_ERR_CUDA;
    int prev = done[dp.dev].load(std::memory_order_acquire);
    while (prev < smem && !done[dp.dev].compare_exchange_weak(prev, smem, std::memory_order_acq_rel)) {
    }
    return SPP_OK;
}

// Labels (labels.cu, FORMAT.md 3)
spp_status labels_decode(int kind, const void *const *d_src, const uint64_t *src_bytes, int n, void *d_dst, int H,
                         int W, uint32_t *status, cudaStream_t stream);

inline size_t out_elem_bytes(int out) { return out == SPP_OUT_F32 ? 4 : 2; }

}  // namespace spp
