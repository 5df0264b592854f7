// spp_internal.h — launcher interface between the C ABI (api.cu) and the
// format-specific kernel files (cosmo.cu, deepcam.cu).
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

#include "spp.h"

namespace spp {

// device properties of the current device (cached per device id)
struct DeviceProps {
    int sms = 0;
    int smem_optin = 0;
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

inline size_t out_elem_bytes(int out) { return out == SPP_OUT_F32 ? 4 : 2; }

}  // namespace spp
