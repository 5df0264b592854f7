// api.cu — the C ABI of libspp (include/spp.h): argument validation, device
// properties, dispatch to the format kernels, host-side stream parsing.
#include <cuda_runtime.h>
#include <stdint.h>
#include <string.h>

#include <mutex>

#include "spp.h"
#include "spp_format.h"
#include "spp_internal.h"

namespace spp {

spp_status current_device_props(DeviceProps *out) {
    static std::mutex mu;
    static DeviceProps cache[kMaxDevices];
    static bool have[kMaxDevices] = {false};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= kMaxDevices) return SPP_ERR_CUDA;
    std::lock_guard<std::mutex> lock(mu);
    if (!have[dev]) {
        DeviceProps p;
        p.dev = dev;
        if (cudaDeviceGetAttribute(&p.smem_per_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev) != cudaSuccess ||
            cudaDeviceGetAttribute(&p.smem_reserved, cudaDevAttrReservedSharedMemoryPerBlock, dev) != cudaSuccess)
            return SPP_ERR_CUDA;
        if (cudaDeviceGetAttribute(&p.sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) return SPP_ERR_CUDA;
        if (cudaDeviceGetAttribute(&p.smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev) != cudaSuccess)
            return SPP_ERR_CUDA;
        cudaDeviceGetAttribute(&p.cc_major, cudaDevAttrComputeCapabilityMajor, dev);
        cudaDeviceGetAttribute(&p.cc_minor, cudaDevAttrComputeCapabilityMinor, dev);
        if (p.cc_major != 10) return SPP_ERR_CUDA;  // built for sm_100a only; no fallback
        cache[dev] = p;
        have[dev] = true;
    }
    *out = cache[dev];
    return SPP_OK;
}

static bool dims_ok(spp_format fmt, const spp_decode_opts &o) {
    if (fmt == SPP_FMT_COSMO)
        return o.C == 4 && o.D >= 1 && o.H >= 1 && o.W >= 1 && o.D <= 65535 && o.H <= 65535 && o.W <= 65535;
    if (fmt == SPP_FMT_DEEPCAM)
        return o.C >= 1 && o.H >= 1 && o.W >= 1 && o.C <= 65535 && o.H <= 65535 && o.W <= 65535;
    return false;
}

}  // namespace spp

using namespace spp;

extern "C" {

void spp_decode_opts_init(spp_decode_opts *o, spp_format fmt, int C, int D, int H, int W) {
    if (!o) return;
    memset(o, 0, sizeof(*o));
    o->out = SPP_OUT_F16;
    o->transform = fmt == SPP_FMT_COSMO ? 1 : 0;
    o->C = C;
    o->D = fmt == SPP_FMT_COSMO ? D : 1;
    o->H = H;
    o->W = W;
}

size_t spp_decode_workspace_size(spp_format fmt, int n, const spp_decode_opts *opts) {
    (void)opts;
    if (n <= 0) return 0;
    if (fmt == SPP_FMT_COSMO) return cosmo_workspace_bytes(n);
    if (fmt == SPP_FMT_DEEPCAM) return deepcam_workspace_bytes(n);
    return 0;
}

size_t spp_decoded_sample_bytes(spp_format fmt, const spp_decode_opts *o) {
    if (!o || !dims_ok(fmt, *o)) return 0;
    const size_t eb = out_elem_bytes(o->out);
    if (fmt == SPP_FMT_COSMO) return (size_t)o->C * o->D * o->H * o->W * eb;
    return (size_t)o->C * o->H * o->W * eb;
}

int spp_decode_launches(spp_format fmt) {
    return fmt == SPP_FMT_COSMO ? kCosmoLaunches : (fmt == SPP_FMT_DEEPCAM ? kDeepcamLaunches : 0);
}

spp_status spp_decode_batch(spp_format fmt, const void *const *d_src, int n, void *d_dst,
                            const spp_decode_opts *opts, spp_stream_t stream) {
    if (!opts || n < 0) return SPP_ERR_INVALID_ARG;
    const spp_decode_opts &o = *opts;
    if (fmt != SPP_FMT_COSMO && fmt != SPP_FMT_DEEPCAM) return SPP_ERR_INVALID_ARG;
    if (!dims_ok(fmt, o)) return SPP_ERR_INVALID_ARG;
    if (o.out != SPP_OUT_F16 && o.out != SPP_OUT_F32 && o.out != SPP_OUT_I16) return SPP_ERR_INVALID_ARG;
    if (o.out == SPP_OUT_I16 && (fmt != SPP_FMT_COSMO || o.transform != 0)) return SPP_ERR_INVALID_ARG;
    if (fmt == SPP_FMT_COSMO && o.transform != 0 && o.transform != 1) return SPP_ERR_INVALID_ARG;
    if (o.raw_segments != 0 && o.raw_segments != 1) return SPP_ERR_INVALID_ARG;
    if (n == 0) return SPP_OK;
    if (!d_src || !d_dst) return SPP_ERR_INVALID_ARG;
    if ((reinterpret_cast<uintptr_t>(d_dst) & 15) != 0) return SPP_ERR_INVALID_ARG;
    const size_t need = spp_decode_workspace_size(fmt, n, opts);
    if (need && (!o.workspace || o.workspace_size < need)) return SPP_ERR_BUFFER_TOO_SMALL;
    if ((reinterpret_cast<uintptr_t>(o.workspace) & 255) != 0) return SPP_ERR_INVALID_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    if (fmt == SPP_FMT_COSMO) return cosmo_decode(d_src, n, d_dst, o, st);
    return deepcam_decode(d_src, n, d_dst, o, st);
}

spp_status spp_decode_labels(int kind, const void *const *d_src, const uint64_t *src_bytes, int n, void *d_dst,
                             int H, int W, uint32_t *status, spp_stream_t stream) {
    if (n < 0 || (kind != SPP_LABEL_MASK && kind != SPP_LABEL_VECTOR)) return SPP_ERR_INVALID_ARG;
    if (H < 1 || W < 1 || H > 65535 || W > 65535 || (kind == SPP_LABEL_VECTOR && H != 1)) return SPP_ERR_INVALID_ARG;
    if (n == 0) return SPP_OK;
    if (!d_src || !d_dst) return SPP_ERR_INVALID_ARG;
    if (kind == SPP_LABEL_VECTOR && (reinterpret_cast<uintptr_t>(d_dst) & 3) != 0) return SPP_ERR_INVALID_ARG;
    return labels_decode(kind, d_src, src_bytes, n, d_dst, H, W, status, reinterpret_cast<cudaStream_t>(stream));
}

spp_status spp_stream_info(spp_format fmt, const void *src, size_t src_bytes, int64_t info[4]) {
    if (!src || !info) return SPP_ERR_INVALID_ARG;
    const uint8_t *b = static_cast<const uint8_t *>(src);
    if (src_bytes < (size_t)kHeaderBytes) return SPP_ERR_CORRUPT;
    auto r16 = [&](size_t o) { uint16_t v; memcpy(&v, b + o, 2); return v; };
    auto r32 = [&](size_t o) { uint32_t v; memcpy(&v, b + o, 4); return v; };
    auto r64 = [&](size_t o) { uint64_t v; memcpy(&v, b + o, 8); return v; };
    if (fmt == SPP_FMT_COSMO) {
        if (r32(0) != kCosmoMagic || r16(4) != kVersion) return SPP_ERR_CORRUPT;
        const uint32_t nU = r32(cosmo::kNU), T = r32(cosmo::kNSlab);
        const uint64_t slab_off = r64(cosmo::kSlabOff);
        if (T < 1 || slab_off > src_bytes || 32ull * T > src_bytes - slab_off) return SPP_ERR_CORRUPT;
        info[0] = nU;
        info[1] = T;
        info[2] = r32(slab_off + 8);
        info[3] = b[slab_off + 12];
        return SPP_OK;
    }
    if (fmt == SPP_FMT_DEEPCAM) {
        if (r32(0) != kDeepcamMagic || r16(4) != kVersion) return SPP_ERR_CORRUPT;
        const uint32_t L = r32(deepcam::kL);
        const uint64_t dir_off = r64(deepcam::kDirOff), pay = r64(deepcam::kPayloadOff);
        if (dir_off > src_bytes || 4ull * (L + 1) > src_bytes - dir_off || pay > src_bytes) return SPP_ERR_CORRUPT;
        int64_t raw = 0, seg = 0, segs = 0, dbytes = 0;
        for (uint32_t l = 0; l < L; l++) {
            const uint64_t a = r32(dir_off + 4ull * l), e = r32(dir_off + 4ull * l + 4);
            if (e > src_bytes - pay || e < a + 16) return SPP_ERR_CORRUPT;
            const uint8_t *p = b + pay + a;
            if (p[0] == deepcam::kModeRaw || p[0] == deepcam::kModeRaw16) { raw++; continue; }
            seg++;
            uint16_t ns;
            memcpy(&ns, p + 2, 2);
            segs += ns;
            if (4ull + 8ull * ns > e - a) return SPP_ERR_CORRUPT;
            for (int s = 0; s < ns; s++) {
                uint16_t len;
                memcpy(&len, p + 4 + 4 * s, 2);
                if (p[4 + 4 * s + 2] == deepcam::kDiff && len > 0) dbytes += len - 1;
            }
        }
        info[0] = raw;
        info[1] = seg;
        info[2] = segs;
        info[3] = dbytes;
        return SPP_OK;
    }
    return SPP_ERR_INVALID_ARG;
}

const char *spp_status_string(spp_status s) {
    switch (s) {
        case SPP_OK: return "ok";
        case SPP_ERR_INVALID_ARG: return "invalid argument";
        case SPP_ERR_BUFFER_TOO_SMALL: return "buffer too small";
        case SPP_ERR_CORRUPT: return "corrupt stream";
        case SPP_ERR_UNSUPPORTED: return "unsupported by the GPU path";
        case SPP_ERR_CUDA: return "CUDA error";
    }
    return "unknown status";
}

const char *spp_version(void) { return "spp 0.1.0 sm_100a"; }

}  // extern "C"
