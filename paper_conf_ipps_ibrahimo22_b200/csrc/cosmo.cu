// cosmo.cu — CosmoFlow decode + log-preprocess on sm_100a (FORMAT.md 1.2).
//
// PAPER.md §V.B and §VI: a sample is a per-sample lookup
// table of 4-groups (8-byte values of four 16-bit indices into the unique
// count set U) plus one 1- or 2-byte key per voxel.  The log transform is
// applied to U only, before expansion, and the four redshift planes
// are written directly in the training layout (fused transpose).
//
// Two kernels per batch:
//   KC0  kc0_prologue   one CTA per sample: validate header + slab table,
//                        fU[i] = RN_fp32(log1p(U[i])) (or the identity) into
//                        the workspace.  |U| is hundreds, so this is ~10^3
//                        transcendental evaluations per 8M outputs.
//   KC   kc_expand      persistent CTAs over (sample, voxel chunk) items,
//                        contiguous per CTA.  Each CTA stages the hottest
//                        groups of the current slab (keys are frequency-ordered
//                        by the encoder) as ready-to-store output tuples
//                        T[g] = (f(U[e0]),..,f(U[e3])) in shared memory; cold
//                        keys rebuild the tuple from the L1/L2-resident LUT.
//                        Each thread handles 8 consecutive voxels: one 16-B key
//                        load, 8 smem gathers, four 16-B (fp16) streaming
//                        stores, one per redshift plane.  One producer warp
//                        streams the key tiles of every segment the CTA will
//                        expand through a 5-stage TMA ring (kc_produce); the
//                        768 consumer threads classify cold keys one tile
//                        ahead and fetch their LUT rows by cp.async.
//   KC (ESC instance, opts.escape_keys) also decodes FORMAT.md 1.5 escaped
//                        1-byte keys: the producer stages each tile's low
//                        bytes, escape-block index and escape entries; the
//                        consumers resolve keys once per tile (warp scan of
//                        escape counts) into a buffer carved from the hot region.
// HBM traffic per sample = keys + LUT + U + outputs; everything else is
// on-chip or L2.
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include <algorithm>

#include "common.cuh"
#include "spp_format.h"
#include "spp_internal.h"

namespace spp {
namespace {

using namespace spp::cosmo;

struct CosmoMeta {  // written by KC0, read by KC
    uint32_t valid;
    uint32_t nU;
    uint32_t nslab;
    uint32_t pad;
};

constexpr size_t kFuStride = kMaxU;  // floats per sample in the workspace
#ifndef SPP_KC_THREADS
#define SPP_KC_THREADS 768
#endif
#ifndef SPP_KC_HOT_KB
#define SPP_KC_HOT_KB 132
#endif
#ifndef SPP_KC_PRODUCER
#define SPP_KC_PRODUCER 1
#endif
constexpr int kConsumers = SPP_KC_THREADS;  // threads that expand voxels (8 per tile)
constexpr bool kProducerWarp = SPP_KC_PRODUCER;  // one extra warp refills the key ring
constexpr int kThreads = kConsumers + (kProducerWarp ? 32 : 0);
constexpr int kPrologueThreads = 256;
constexpr int kMinBlocks = kThreads <= 288 ? 3 : (kThreads <= 416 ? 2 : 1);  // CTAs per SM the registers target
constexpr int kHotBytes = SPP_KC_HOT_KB * 1024;  // shared-memory hot prefix of T per CTA
constexpr int kUCap = 2048;           // part of the region nominally for f(U) (8 KB)
constexpr int kRegionBytes = kHotBytes + kUCap * 4;  // f(U) first, then the hot tuples
#ifndef SPP_KC_STAGES
#define SPP_KC_STAGES 5
#endif
constexpr int kKeyStages = SPP_KC_STAGES;  // TMA ring of key tiles
#ifndef SPP_KC_DIAG_LDG  // timing diagnostic only (wrong output): cold keys = one global 8-B load, no slots
#define SPP_KC_DIAG_LDG 0
#endif
#ifndef SPP_KC_DIAG_NOCOLD
#define SPP_KC_DIAG_NOCOLD 0
#endif
#ifndef SPP_KC_PREFETCH_TAIL
#define SPP_KC_PREFETCH_TAIL 1
#endif
// key tiles are read once: their TMA loads carry an L2 evict_first hint so they do
// not displace the LUT tails (evict_last) and cold rows (r2: C2 0.817 -> 0.834,
// dense C5 rows +1-3 points; profiles/r02a3_*, r02a5_*)
#ifndef SPP_KC_BAD_MAX
#define SPP_KC_BAD_MAX 1
#endif
#ifndef SPP_KC_KEY_EF
#define SPP_KC_KEY_EF 1
#endif
constexpr int kTileVox = kConsumers * 8;  // voxels per CTA iteration (8 per consumer thread)
constexpr int kStageBytes = kTileVox * 2;
#ifndef SPP_KC_LA
#define SPP_KC_LA 1
#endif
constexpr int kColdLA = SPP_KC_LA;                        // tiles of cold-row lookahead
#ifndef SPP_KC_ESC_IMPL
#define SPP_KC_ESC_IMPL 1  // escaped-key resolution: 0 predicated generic loads, 1 shared loads + PRMT, 2 loop
#endif
#ifndef SPP_KC_ESC_PREFETCH
#define SPP_KC_ESC_PREFETCH 2
#endif
// escaped tiles: 0 = keys resolved at expansion, cold rows fetched there; 1 = resolved at
// classify (to prefetch cold rows) and again at expansion; 2 = resolved once, at classify,
// into a buffer carved from the end of the hot region, cold rows prefetched
constexpr int kEscPrefetch = SPP_KC_ESC_PREFETCH;
constexpr uint32_t kRkBytes = (kColdLA + 1) * kConsumers * 16;  // resolved keys, 16 B per thread per tile
#ifndef SPP_KC_ALL_LANES_RELEASE
#define SPP_KC_ALL_LANES_RELEASE 1
#endif
constexpr bool kAllLanesRelease = SPP_KC_ALL_LANES_RELEASE;  // every consumer lane arrives on a stage's empty barrier
#ifndef SPP_KC_COLD_SLOTS
#define SPP_KC_COLD_SLOTS 2
#endif
constexpr int kColdSlots = SPP_KC_COLD_SLOTS;             // LUT rows per thread per tile fetched ahead
constexpr int kColdSlotBytes = (kColdLA + 1) * kConsumers * kColdSlots * 8;
constexpr int kSmemBytes = kHotBytes + kUCap * 4 + kKeyStages * kStageBytes + kColdSlotBytes + 2 * kKeyStages * 8;

size_t meta_offset(int n) { return round_up16((size_t)n * kFuStride * sizeof(float)); }

// --------------------------------------------------------------------------
// KC0: header/slab validation and the unique-value transform
__global__ void __launch_bounds__(kPrologueThreads) kc0_prologue(const void *const *__restrict__ src,
                                                         const uint64_t *__restrict__ src_bytes, int transform,
                                                         int D, int H, int W, float *__restrict__ fU_ws,
                                                         CosmoMeta *__restrict__ meta,
                                                         uint32_t *__restrict__ status, int esc_ok) {
    const int s = blockIdx.x;
    const uint8_t *b = static_cast<const uint8_t *>(src[s]);
    __shared__ uint32_t sh_ok, sh_nU;
    __shared__ uint64_t sh_Uoff;
    if (threadIdx.x == 0) {
        uint32_t ok = b != nullptr && (reinterpret_cast<uintptr_t>(b) & 15) == 0, unsupported = 0;
        uint64_t limit = src_bytes ? src_bytes[s] : ~0ull;
        uint32_t nU = 0, T = 0;
        uint64_t U_off = 0;
        if (ok && limit < (uint64_t)kHeaderBytes) ok = 0;
        if (ok) {
            ok = ld_le32(b) == kCosmoMagic && ld_le16(b + 4) == kVersion && ld_le16(b + kC) == 4 &&
                 ld_le16(b + kD) == D && ld_le16(b + kH) == H && ld_le16(b + kW) == W;
        }
        if (ok) {
            nU = ld_le32(b + kNU);
            T = ld_le32(b + kNSlab);
            U_off = ld_le64(b + kUOff);
            const uint64_t slab_off = ld_le64(b + kSlabOff), total = ld_le64(b + kTotal);
            // every range checked as off <= total && len <= total - off: stream-supplied
            // 64-bit offsets never wrap an addition
            auto in_range = [&](uint64_t off, uint64_t len) { return off <= total && len <= total - off; };
            ok = total <= limit && nU >= 1 && nU <= (uint32_t)kMaxU && T >= 1 && T <= (uint32_t)D &&
                 in_range(U_off, 2ull * nU) && in_range(slab_off, (uint64_t)kSlabBytes * T) &&
                 (slab_off & 15) == 0 && (U_off & 1) == 0;
            const uint64_t plane = (uint64_t)H * W;
            uint32_t zexp = 0;
            for (uint32_t t = 0; ok && t < T; t++) {
                const uint8_t *sl = b + slab_off + (uint64_t)kSlabBytes * t;
                const uint32_t z0 = ld_le32(sl), z1 = ld_le32(sl + 4), G = ld_le32(sl + 8);
                const int kw = sl[12];
                const uint64_t lut_off = ld_le64(sl + 16), keys_off = ld_le64(sl + 24);
                ok = z0 == zexp && z1 > z0 && z1 <= (uint32_t)D;
                const uint64_t Nt = (uint64_t)(z1 - z0) * plane;
                if (kw == 0) ok = ok && G == 1;
                else if (kw == 1) ok = ok && G >= 1 && G <= (uint32_t)kMaxG1;
                else if (kw == 2) ok = ok && G >= 1 && G <= (uint32_t)kMaxG2;
                else if (kw == kEscaped) {
                    if (!esc_ok) unsupported = 1;
                    ok = ok && G >= 1 && G <= (uint32_t)kMaxG2;
                }
                else if (kw == kRawSlab) ok = ok && G == 0;
                else ok = 0;
                if (kw != kRawSlab) ok = ok && (lut_off & 15) == 0 && in_range(lut_off, 8ull * G);
                if (kw == kEscaped) {  // FORMAT.md 1.5: eidx[0] = 0, the escape list inside the stream
                    const uint64_t nb = (Nt + kEscBlock - 1) / kEscBlock;
                    const uint64_t head = ((4 * (nb + 1) + 15) & ~15ull) + ((Nt + 15) & ~15ull);
                    ok = ok && (keys_off & 15) == 0 && in_range(keys_off, head);
                    const uint64_t esc_off = ok ? keys_off + head : 0;
                    ok = ok && ld_le32(b + keys_off) == 0 && in_range(esc_off, 2ull * ld_le32(b + keys_off + 4 * nb));
                } else if (kw != 0) {
                    ok = ok && (keys_off & 15) == 0 && in_range(keys_off, (uint64_t)(kw == kRawSlab ? 8 : kw) * Nt);
                }
                zexp = z1;
            }
            ok = ok && zexp == (uint32_t)D;
        }
        if (!ok) report(status, SPP_ERR_CORRUPT, s);
        else if (unsupported) report(status, SPP_ERR_UNSUPPORTED, s);  // needs opts.escape_keys
        ok = ok && !unsupported;
        sh_ok = ok;
        sh_nU = nU;
        sh_Uoff = U_off;
        meta[s] = CosmoMeta{ok, nU, T, 0};
    }
    __syncthreads();
    if (!sh_ok) return;
    const uint8_t *U = b + sh_Uoff;
    float *fU = fU_ws + (size_t)s * kFuStride;
    for (uint32_t i = threadIdx.x; i < sh_nU; i += blockDim.x) {
        const int c = (int16_t)ld_le16(U + 2 * i);
        // fp64 log1p rounded once to fp32 (FORMAT.md 1.2, reading S2)
        fU[i] = transform ? (float)log1p((double)c) : (float)c;
    }
}

// --------------------------------------------------------------------------
// KC: fused LUT expansion + transpose
template <int OUT>
struct Entry;
template <>
struct Entry<SPP_OUT_F16> { using T = uint2; };
template <>
struct Entry<SPP_OUT_I16> { using T = uint2; };
template <>
struct Entry<SPP_OUT_F32> { using T = uint4; };

template <int OUT>
__device__ __forceinline__ uint32_t cvt_lane(float f);
template <>
__device__ __forceinline__ uint32_t cvt_lane<SPP_OUT_F16>(float f) {
    return (uint32_t)__half_as_ushort(__float2half_rn(f));
}
template <>
__device__ __forceinline__ uint32_t cvt_lane<SPP_OUT_I16>(float f) {
    return (uint32_t)(uint16_t)(int16_t)__float2int_rn(f);
}

template <int OUT>
__device__ __forceinline__ typename Entry<OUT>::T pack_entry(const float (&f)[4]) {
    if constexpr (OUT == SPP_OUT_F32) {
        return make_uint4(__float_as_uint(f[0]), __float_as_uint(f[1]), __float_as_uint(f[2]), __float_as_uint(f[3]));
    } else {
        return make_uint2(cvt_lane<OUT>(f[0]) | (cvt_lane<OUT>(f[1]) << 16),
                          cvt_lane<OUT>(f[2]) | (cvt_lane<OUT>(f[3]) << 16));
    }
}

// Where f(U) lives for the current sample: shared memory (|U| <= kUCap, the
// normal case: hundreds of values) or the global workspace.
struct FuView {
    uint32_t smem;        // shared address of fU_s
    const float *global;  // workspace copy
    uint32_t nU;
    bool in_smem;
};

// output 4-tuple of LUT entry `e` (four 16-bit U indices); an index >= nU
// (corrupt stream) is clamped and flagged in `bad` (reported once per item)
template <int OUT, bool SMEM>
__device__ __forceinline__ typename Entry<OUT>::T make_entry(uint2 e, const FuView &fu, uint32_t &bad) {
    uint32_t idx[4] = {e.x & 0xFFFFu, e.x >> 16, e.y & 0xFFFFu, e.y >> 16};
    float f[4];
#if SPP_KC_BAD_MAX  // one compare of the largest index instead of four
    bad |= max(max(idx[0], idx[1]), max(idx[2], idx[3])) >= fu.nU;
#endif
#pragma unroll
    for (int c = 0; c < 4; c++) {
#if !SPP_KC_BAD_MAX
        bad |= idx[c] >= fu.nU;
#endif
        const uint32_t i = min(idx[c], fu.nU - 1);
        if constexpr (SMEM) f[c] = lds_f32(fu.smem + 4 * i);
        else f[c] = ld_ro_f32(fu.global + i);
    }
    return pack_entry<OUT>(f);
}

template <int OUT>
__device__ __forceinline__ typename Entry<OUT>::T lds_entry(uint32_t addr) {
    if constexpr (OUT == SPP_OUT_F32) return lds_u4(addr);
    else return lds_u2(addr);
}
template <int OUT>
__device__ __forceinline__ void sts_entry(uint32_t addr, typename Entry<OUT>::T v) {
    if constexpr (OUT == SPP_OUT_F32) sts_u4(addr, v);
    else sts_u2(addr, v);
}

struct SlabView {
    uint32_t z0, z1, G;
    int kw;
    const uint8_t *lut;
    const uint8_t *keys;
};

// slab table entry t (32 B, 16-B aligned and bounds-checked by KC0; the
// stream is little-endian like the device): two 16-B read-only loads
__device__ __forceinline__ SlabView read_slab(const uint8_t *b, uint64_t slab_off, int t) {
    const uint8_t *sl = b + slab_off + (uint64_t)kSlabBytes * t;
    const uint4 w0 = ld_ro_u4(sl), w1 = ld_ro_u4(sl + 16);
    SlabView v;
    v.z0 = w0.x;
    v.z1 = w0.y;
    v.G = w0.z;
    v.kw = (int)(w0.w & 0xFFu);
    v.lut = b + ((uint64_t)w1.y << 32 | w1.x);
    v.keys = b + ((uint64_t)w1.w << 32 | w1.z);
    return v;
}

__host__ __device__ __forceinline__ uint64_t up16(uint64_t x) { return (x + 15) & ~uint64_t(15); }

// FORMAT.md 1.5 escaped-key slab of Nt voxels: eidx u32[nb+1] at keys, then
// the low bytes, then the u16 escape list (each section 16-B aligned)
struct EscView {
    const uint32_t *eidx;
    const uint8_t *low;
    const uint16_t *esc;
    uint32_t nb, n_esc;
};
__device__ __forceinline__ EscView esc_view(const SlabView &sv, uint64_t Nt) {
    EscView e;
    e.nb = (uint32_t)((Nt + kEscBlock - 1) / kEscBlock);
    e.eidx = reinterpret_cast<const uint32_t *>(sv.keys);
    e.low = sv.keys + up16(4ull * (e.nb + 1));
    e.esc = reinterpret_cast<const uint16_t *>(e.low + up16(Nt));
    e.n_esc = ld_le32(sv.keys + 4ull * e.nb);
    return e;
}
// key of voxel `rel` of an escaped-key slab, sequentially (scalar path)
__device__ __forceinline__ uint32_t esc_key_scalar(const EscView &ev, uint64_t rel) {
    const uint32_t lo = ev.low[rel];
    if (lo != 255u) return lo;
    const uint64_t b0 = rel / kEscBlock * kEscBlock;
    uint32_t r = ev.eidx[rel / kEscBlock];
    for (uint64_t v = b0; v < rel; v++) r += ev.low[v] == 255u;
    return ev.n_esc ? ev.esc[min(r, ev.n_esc - 1)] : 0xFFFFFFFFu;
}
// eidx[blk + 1] - eidx[blk] equals the escapes in block blk (scalar-path check)
__device__ __forceinline__ bool esc_block_ok(const EscView &ev, uint64_t blk, uint64_t Nt) {
    uint32_t c = 0;
    const uint64_t v1 = min(Nt, (blk + 1) * kEscBlock);
    for (uint64_t v = blk * kEscBlock; v < v1; v++) c += ev.low[v] == 255u;
    return ev.eidx[blk + 1] - ev.eidx[blk] == c;
}

// Key stage layout of an escaped-key tile (FORMAT.md 1.5 staged by the producer):
// low bytes at 0, the tile's eidx entries from entry (b0 & ~3) at kIdxOff, and its
// escape entries from entry (e0 & ~7) at kEscOff when they fit kEscCap
constexpr uint32_t kIdxOff = kTileVox;          // after the low bytes (1 per voxel)
constexpr uint32_t kEscOff = kIdxOff + 160;      // eidx slice: <= 4 * (kTileVox / 256 + 4) bytes
constexpr uint32_t kEscCap = kStageBytes - kEscOff;
static_assert(4 * (kTileVox / kEscBlock + 4) <= 160 && kEscCap >= 1024, "escaped-key stage layout");
__device__ __forceinline__ uint32_t esc_copy_bytes(uint32_t e0, uint32_t e1) {
    return ((2u * e1 + 15u) & ~15u) - ((2u * e0) & ~15u);
}

// store the 4 planes of 8 consecutive voxels (vector path): plane c of voxel v
// is out_s[(c*N + v)]; one 16-B (fp16/int16) or 32-B (fp32) store per plane
template <int OUT>
__device__ __forceinline__ void store8(uint8_t *out_s, uint64_t N, uint64_t v, const typename Entry<OUT>::T (&e)[8]) {
    if constexpr (OUT == SPP_OUT_F32) {
#pragma unroll
        for (int c = 0; c < 4; c++) {
            float f[8];
#pragma unroll
            for (int j = 0; j < 8; j++) f[j] = __uint_as_float(c == 0 ? e[j].x : c == 1 ? e[j].y : c == 2 ? e[j].z : e[j].w);
            st_stream_f8(out_s + ((uint64_t)c * N + v) * 4, f);
        }
    } else {
        // entry = (c0 | c1 << 16, c2 | c3 << 16): plane c takes 16-bit lane c of each entry
        uint4 p0, p1, p2, p3;
        p0.x = __byte_perm(e[0].x, e[1].x, 0x5410); p1.x = __byte_perm(e[0].x, e[1].x, 0x7632);
        p2.x = __byte_perm(e[0].y, e[1].y, 0x5410); p3.x = __byte_perm(e[0].y, e[1].y, 0x7632);
        p0.y = __byte_perm(e[2].x, e[3].x, 0x5410); p1.y = __byte_perm(e[2].x, e[3].x, 0x7632);
        p2.y = __byte_perm(e[2].y, e[3].y, 0x5410); p3.y = __byte_perm(e[2].y, e[3].y, 0x7632);
        p0.z = __byte_perm(e[4].x, e[5].x, 0x5410); p1.z = __byte_perm(e[4].x, e[5].x, 0x7632);
        p2.z = __byte_perm(e[4].y, e[5].y, 0x5410); p3.z = __byte_perm(e[4].y, e[5].y, 0x7632);
        p0.w = __byte_perm(e[6].x, e[7].x, 0x5410); p1.w = __byte_perm(e[6].x, e[7].x, 0x7632);
        p2.w = __byte_perm(e[6].y, e[7].y, 0x5410); p3.w = __byte_perm(e[6].y, e[7].y, 0x7632);
        uint8_t *o = out_s + v * 2;
        st_stream_u4(o, p0);
        st_stream_u4(o + N * 2, p1);
        st_stream_u4(o + N * 4, p2);
        st_stream_u4(o + N * 6, p3);
    }
}

template <int OUT>
__device__ __forceinline__ void store1(uint8_t *out_s, uint64_t N, uint64_t v, typename Entry<OUT>::T e) {
    if constexpr (OUT == SPP_OUT_F32) {
        float *o = reinterpret_cast<float *>(out_s);
        o[v] = __uint_as_float(e.x); o[N + v] = __uint_as_float(e.y);
        o[2 * N + v] = __uint_as_float(e.z); o[3 * N + v] = __uint_as_float(e.w);
    } else {
        uint16_t *o = reinterpret_cast<uint16_t *>(out_s);
        o[v] = (uint16_t)(e.x & 0xFFFF); o[N + v] = (uint16_t)(e.x >> 16);
        o[2 * N + v] = (uint16_t)(e.y & 0xFFFF); o[3 * N + v] = (uint16_t)(e.y >> 16);
    }
}

// 8 keys of one group as eight 16-bit lanes of a uint4 (kw = 1 keys are widened
// after the shared-memory load, so one code path serves both key widths)
struct Keys8 {
    uint4 v;
    __device__ __forceinline__ uint32_t get(int j) const {  // j compile-time
        const uint32_t w = j < 2 ? v.x : j < 4 ? v.y : j < 6 ? v.z : v.w;
        return (j & 1) ? (w >> 16) : (w & 0xFFFFu);
    }
    __device__ __forceinline__ uint32_t get_dyn(uint32_t j) const {  // j runtime (rare cold path)
        const uint32_t w = (j & 4) ? ((j & 2) ? v.w : v.z) : ((j & 2) ? v.y : v.x);
        return (j & 1) ? (w >> 16) : (w & 0xFFFFu);
    }
    __device__ __forceinline__ void set_dyn(uint32_t j, uint32_t key) {  // j runtime, key < 2^16
        const uint32_t sel = (j & 1) ? 0x5410u : 0x3254u, w = j >> 1;
        v.x = w == 0 ? __byte_perm(v.x, key, sel) : v.x;
        v.y = w == 1 ? __byte_perm(v.y, key, sel) : v.y;
        v.z = w == 2 ? __byte_perm(v.z, key, sel) : v.z;
        v.w = w == 3 ? __byte_perm(v.w, key, sel) : v.w;
    }
};

// The key stream of the CTA's current range is staged into shared memory by
// 1-D TMA bulk copies (cp.async.bulk + mbarrier): a ring of kKeyStages tiles of
// 2048 voxels, refilled by thread 0 as soon as all 8 warps have released a
// stage (per-stage "empty" mbarriers, one arrival per warp: no CTA barrier),
// so many KB of key reads are in flight per SM without spending registers.
// Tile indices are CTA-global (`count` = tiles consumed so far) and select the
// stage and both mbarrier phases.
struct KeyRing {
    uint8_t *buf;      // kKeyStages * kStageBytes
    uint64_t *full;    // kKeyStages, completed by the TMA transaction count
    uint64_t *empty;   // kKeyStages, one arrival per warp
    uint32_t count;
    uint32_t cold;     // shared address of the per-thread cold-row slots
};

__device__ __forceinline__ Keys8 keys_from_smem(const uint8_t *stage, uint32_t kwb) {
    Keys8 k;
    const uint32_t ka = smem_u32(stage) + threadIdx.x * 8u * kwb;
    if (kwb == 2) {
        k.v = lds_u4(ka);
    } else {
        const uint2 t = lds_u2(ka);
        k.v.x = __byte_perm(t.x, 0u, 0x4140);
        k.v.y = __byte_perm(t.x, 0u, 0x4342);
        k.v.z = __byte_perm(t.y, 0u, 0x4140);
        k.v.w = __byte_perm(t.y, 0u, 0x4342);
    }
    return k;
}

// Voxels [a, b) of one slab (relative indices, multiples of 16), 8 consecutive
// voxels per thread per tile (a warp writes 512 contiguous bytes per plane
// store).  Hot tuples come from the shared-memory prefix.  Cold keys (the
// power-law tail beyond the prefix) are looked up one tile ahead: while
// tile t is expanded, each thread has already classified its keys of tile t+1
// and requested their LUT rows (up to two per thread; more are fetched in
// place, rarely), so every group is stored once, complete, and no warp waits
// on an L2 round trip.  A key >= G (corrupt) can only be cold: clamped, flagged.
template <int OUT, bool ESC>
__device__ __forceinline__ void expand_keys_vec(const SlabView &sv, uint64_t slab_v0, uint64_t a, uint64_t b,
                                                uint32_t hot_base, uint32_t n_hot, const FuView &fu, uint8_t *out_s,
                                                uint64_t N, uint32_t &bad, KeyRing &ring, uint64_t Nt,
                                                uint32_t rk_base) {
    using E = typename Entry<OUT>::T;
    constexpr uint32_t EB = sizeof(E);
    const bool escd = ESC && sv.kw == kEscaped;     // FORMAT.md 1.5 tile (staged by kc_produce)
    const uint32_t kwb = escd ? 1u : (uint32_t)sv.kw;  // key bytes per voxel in the stage
    EscView ev{};
    if (escd) ev = esc_view(sv, Nt);
    const uint32_t Gm1 = sv.G - 1;
    const uint32_t ntiles = (uint32_t)((b - a + kTileVox - 1) / kTileVox);
    const uint32_t lane = threadIdx.x & 31;
    const uint64_t pol = l2_policy_evict_last();  // keep this sample's LUT in L2 against the output stream
    // kw = 3 (FORMAT.md 1.5) tile t: where this warp's escaped keys are.  The stage
    // holds the tile's eidx entries (from entry b0 & ~3) and, when they fit, its
    // escape entries (from entry e0 & ~7); otherwise they are read from global
    // memory.  Returns esp with esp[i] = esc[e0 + i], and the warp's escape offset.
    struct EscTile {
        const uint16_t *esp;
        uint32_t n;      // escapes of the tile (esp[0..n) valid)
        uint32_t wbase;  // this warp's first escape, relative to e0
        uint32_t wcnt;   // this warp's escapes per the index
        bool wact;       // the warp has voxels in the tile
        bool staged;     // esp is in shared memory (at ssh)
        uint32_t ssh;
    };
    auto esc_tile = [&](uint32_t t) {
        const uint8_t *stage = ring.buf + ((ring.count + t) % kKeyStages) * kStageBytes;
        const uint64_t st = a + (uint64_t)t * kTileVox;
        const uint64_t rem = b - st;
        const uint32_t nvox = rem < (uint64_t)kTileVox ? (uint32_t)rem : (uint32_t)kTileVox;
        const uint32_t b0 = (uint32_t)(st / kEscBlock), b1 = (uint32_t)((st + nvox + kEscBlock - 1) / kEscBlock);
        const uint32_t bw = min(b0 + (threadIdx.x >> 5), b1 - 1);
        const uint32_t *ix = reinterpret_cast<const uint32_t *>(stage + kIdxOff) - (b0 & ~3u);  // ix[b] = eidx[b]
        const uint32_t e0 = ix[b0], e1 = ix[b1];
        EscTile et;
        et.wact = b0 + (threadIdx.x >> 5) < b1;
        const bool sane = e1 >= e0 && ix[bw] >= e0 && ix[bw + 1] >= ix[bw] && ix[bw + 1] <= e1;
        et.n = sane ? e1 - e0 : 0u;
        et.wbase = sane ? ix[bw] - e0 : 0u;
        et.wcnt = sane ? ix[bw + 1] - ix[bw] : 0xFFFFFFFFu;
        const bool staged = sane && esc_copy_bytes(e0, e1) <= kEscCap;
        if (!staged) et.n = sane ? min(et.n, ev.n_esc > e0 ? ev.n_esc - e0 : 0u) : 0u;
        et.esp = staged ? reinterpret_cast<const uint16_t *>(stage + kEscOff) + (e0 & 7u) : ev.esc + min(e0, ev.n_esc);
        et.staged = staged;
        et.ssh = smem_u32(stage + kEscOff) + 2u * (e0 & 7u);  // shared address of esp[0] when staged
        return et;
    };
    // 8-bit mask of the escaped voxels (low byte 255) among a thread's 8 low bytes
    auto esc_mask8 = [](uint2 raw) {
        const uint32_t a0 = __vcmpeq4(raw.x, 0xFFFFFFFFu) & 0x01010101u, a1 = __vcmpeq4(raw.y, 0xFFFFFFFFu) & 0x01010101u;
        return ((a0 * 0x01020408u) >> 24) | (((a1 * 0x01020408u) >> 24) << 4);
    };
    // the keys of a thread's 8 voxels: low bytes widened, escaped ones from esp
    auto esc_keys = [&](uint2 raw, uint32_t m, uint32_t r0, const EscTile &et) {
        Keys8 k;
        k.v.x = __byte_perm(raw.x, 0u, 0x4140);
        k.v.y = __byte_perm(raw.x, 0u, 0x4342);
        k.v.z = __byte_perm(raw.y, 0u, 0x4140);
        k.v.w = __byte_perm(raw.y, 0u, 0x4342);
#if SPP_KC_ESC_IMPL == 0
#pragma unroll
        for (int j = 0; j < 8; j++) {
            if ((m >> j) & 1u) {
                const uint32_t i = r0 + __popc(m & ((1u << j) - 1u));
                const uint32_t key = i < et.n ? (uint32_t)et.esp[i] : 0xFFFFu;  // past the list: corrupt
                uint32_t &w = j < 2 ? k.v.x : j < 4 ? k.v.y : j < 6 ? k.v.z : k.v.w;
                w = (j & 1) ? (w & 0xFFFFu) | (key << 16) : (w & 0xFFFF0000u) | key;
            }
        }
#elif SPP_KC_ESC_IMPL == 1
        // the warp's escapes are staged (the common case): shared loads; one PRMT per insert
        if (et.staged) {
#pragma unroll
            for (int j = 0; j < 8; j++) {
                if ((m >> j) & 1u) {
                    const uint32_t i = r0 + __popc(m & ((1u << j) - 1u));
                    const uint32_t key = i < et.n ? lds_u16(et.ssh + 2u * i) : 0xFFFFu;  // past the list: corrupt
                    uint32_t &w = j < 2 ? k.v.x : j < 4 ? k.v.y : j < 6 ? k.v.z : k.v.w;
                    w = __byte_perm(w, key, (j & 1) ? 0x5410u : 0x3254u);
                }
            }
        } else {
#pragma unroll
            for (int j = 0; j < 8; j++) {
                if ((m >> j) & 1u) {
                    const uint32_t i = r0 + __popc(m & ((1u << j) - 1u));
                    const uint32_t key = i < et.n ? (uint32_t)__ldg(et.esp + i) : 0xFFFFu;
                    uint32_t &w = j < 2 ? k.v.x : j < 4 ? k.v.y : j < 6 ? k.v.z : k.v.w;
                    w = __byte_perm(w, key, (j & 1) ? 0x5410u : 0x3254u);
                }
            }
        }
#else
        // a loop over this lane's escapes only (consecutive in the list)
        uint32_t i = r0;
#pragma unroll 1
        while (m) {
            const uint32_t j = __ffs(m) - 1;
            m &= m - 1;
            const uint32_t key = i < et.n ? (et.staged ? lds_u16(et.ssh + 2u * i) : (uint32_t)__ldg(et.esp + i)) : 0xFFFFu;
            k.set_dyn(j, key);
            i++;
        }
#endif
        return k;
    };
    auto issue = [&](uint32_t t) {  // thread 0: bulk copy of tile t's keys once its stage is free
        const uint32_t gt = ring.count + t;
        const uint32_t stg = gt % kKeyStages;
        if (gt >= (uint32_t)kKeyStages) mbar_wait(&ring.empty[stg], ((gt / kKeyStages) - 1) & 1u);
        const uint64_t st = a + (uint64_t)t * kTileVox;
        const uint64_t rem = b - st;
        const uint32_t nvox = rem < (uint64_t)kTileVox ? (uint32_t)rem : (uint32_t)kTileVox;
        const uint32_t bytes = (nvox * kwb + 15u) & ~15u;
        fence_proxy_async_smem();
        mbar_arrive_expect_tx(&ring.full[stg], bytes);
        bulk_g2s(ring.buf + stg * kStageBytes, sv.keys + st * kwb, bytes, &ring.full[stg]);
    };
    auto wait_full = [&](uint32_t t) {
        const uint32_t gt = ring.count + t;
        mbar_wait(&ring.full[gt % kKeyStages], (gt / kKeyStages) & 1u);
        return ring.buf + (gt % kKeyStages) * kStageBytes;
    };
    // Cold rows: while tile t is expanded, the thread classifies its keys of
    // tile t + kColdLA and starts LDGSTS copies (cp.async) of its first
    // kColdSlots cold LUT rows into its own shared-memory slots; one copy group
    // per tile, so the rows of tile t are waited for (per thread, no barrier)
    // kColdLA tiles later.  cj[] = the 8-bit cold mask of each tile in flight;
    // the i-th cold position of a tile reads slot i (i < kColdSlots).
    uint32_t cj[kColdLA + 1];
#pragma unroll
    for (int i = 0; i <= kColdLA; i++) cj[i] = 0u;
    auto slot_addr = [&](uint32_t t, uint32_t k) {  // slot k of this thread for tile t
        return ring.cold + ((((ring.count + t) % (kColdLA + 1)) * kConsumers + threadIdx.x) * kColdSlots + k) * 8;
    };
    auto classify = [&](uint32_t t) -> uint32_t {  // tile t's keys are in smem (full barrier passed)
        const uint64_t q = a + (uint64_t)t * kTileVox + 8u * threadIdx.x;
        uint32_t cold = 0;
        Keys8 kres;
        uint32_t escw = 0;  // escaped tile: escape mask << 8 | first escape (tile-relative) << 16
        if (escd) {         // warp-collective (scan): inactive lanes take part with no keys
            const uint8_t *stage = ring.buf + ((ring.count + t) % kKeyStages) * kStageBytes;
            const uint2 raw = q < b ? lds_u2(smem_u32(stage) + threadIdx.x * 8u) : make_uint2(0u, 0u);
            const uint32_t m = q < b ? esc_mask8(raw) : 0u;
            const uint32_t c = __popc(m);
            const uint32_t incl = warp_incl_scan(c, (int)lane);
            const EscTile et = esc_tile(t);
            const uint32_t wtot = __shfl_sync(0xffffffffu, incl, 31);
            if (lane == 0 && et.wact && wtot != et.wcnt) bad = 1u;  // the index disagrees with the low bytes
            const uint32_t r0 = et.wbase + incl - c;
            escw = (m << 8) | (min(r0, 0xFFFFu) << 16);
            if constexpr (kEscPrefetch == 0) {  // cold rows of escaped tiles are fetched at expansion
                cp_async_commit();
                return escw;
            }
            kres = esc_keys(raw, m, r0, et);
            if constexpr (kEscPrefetch == 2) {  // the expansion reads these resolved keys back
                if (q < b) sts_u4(rk_base + (((ring.count + t) % (kColdLA + 1)) * kConsumers + threadIdx.x) * 16u, kres.v);
            }
        }
        if (q < b) {
            const uint8_t *stage = ring.buf + ((ring.count + t) % kKeyStages) * kStageBytes;
            const Keys8 k = escd ? kres : keys_from_smem(stage, kwb);
#pragma unroll
            for (int j = 0; j < 8; j++) cold |= (k.get(j) >= n_hot ? 1u : 0u) << j;
#if SPP_KC_DIAG_NOCOLD || SPP_KC_DIAG_LDG
            cold = 0;
#endif
            uint32_t m = cold;
#pragma unroll
            for (int i = 0; i < kColdSlots; i++) {
                if (m) {
                    const uint32_t j = __ffs(m) - 1;
                    cp_async8(slot_addr(t, i), sv.lut + 8ull * min(k.get_dyn(j), Gm1));
                    m &= m - 1;
                }
            }
        }
        cp_async_commit();
        return cold | escw;
    };
    // (with kProducerWarp the key tiles are issued by kc_produce, which runs
    // ahead of the consumers across segments, items and samples)
    if (!kProducerWarp && threadIdx.x == 0) {
        for (uint32_t t = 0; t < ntiles && t < (uint32_t)(kKeyStages - 1); t++) issue(t);
    }
#pragma unroll
    for (int i = 0; i < kColdLA; i++) {
        if ((uint32_t)i < ntiles) {
            wait_full(i);
            cj[i] = classify(i);
        } else {
            cp_async_commit();
        }
    }
#pragma unroll 1
    for (uint32_t t = 0; t < ntiles; t++) {
        if (!kProducerWarp && threadIdx.x == 0 && t + kKeyStages - 1 < ntiles) issue(t + kKeyStages - 1);
        if (t + kColdLA < ntiles) {
            wait_full(t + kColdLA);
            cj[kColdLA] = classify(t + kColdLA);
        } else {
            cp_async_commit();  // keep one group per iteration
        }
        cp_async_wait<kColdLA>();  // the copies of tile t have landed (this thread's)
        const uint32_t cmask_all = cj[0], cmask = cmask_all & 0xFFu;  // cold mask (+ escapes, kw = 3)
#pragma unroll
        for (int i = 0; i < kColdLA; i++) cj[i] = cj[i + 1];  // rotate (compile-time indices)
        const uint8_t *stage = ring.buf + ((ring.count + t) % kKeyStages) * kStageBytes;
        const uint64_t q = a + (uint64_t)t * kTileVox + 8u * threadIdx.x;
        if (q < b) {
            Keys8 k0;
            if (escd) {  // the escapes located at classify time (mask, first index) from cj
                if constexpr (kEscPrefetch == 2) {
                    k0.v = lds_u4(rk_base + (((ring.count + t) % (kColdLA + 1)) * kConsumers + threadIdx.x) * 16u);
                } else {
                    const EscTile et = esc_tile(t);
                    k0 = esc_keys(lds_u2(smem_u32(stage) + threadIdx.x * 8u), (cmask_all >> 8) & 0xFFu,
                                  cmask_all >> 16, et);
                }
            } else {
                k0 = keys_from_smem(stage, kwb);
            }
            E e[8];
#if SPP_KC_DIAG_LDG
            if constexpr (OUT == SPP_OUT_F16 && !ESC) {
#pragma unroll
                for (int j = 0; j < 8; j++) {
                    const uint32_t g = k0.get(j);
                    e[j] = g < n_hot ? lds_entry<OUT>(hot_base + g * EB) : ld_ro_u2(sv.lut + 8ull * min(g, Gm1));
                }
                store8<OUT>(out_s, N, slab_v0 + q, e);
                __syncwarp();
                if (kAllLanesRelease || lane == 0) mbar_arrive(&ring.empty[(ring.count + t) % kKeyStages]);
                continue;
            }
#endif
#pragma unroll
            for (int j = 0; j < 8; j++) {
#if SPP_KC_DIAG_NOCOLD  // timing diagnostic only (wrong output): every key treated as hot
                const uint32_t g = k0.get(j) % n_hot;
#else
                const uint32_t g = k0.get(j);
#endif
                if (g < n_hot) {
                    e[j] = lds_entry<OUT>(hot_base + g * EB);
                } else {
                    bad |= g > Gm1;
                    const uint32_t si = __popc(cmask & ((1u << j) - 1u));  // rank among the tile's cold keys
                    const bool pre = !ESC || kEscPrefetch != 0 || ((cmask >> j) & 1u);  // fetched ahead at classify
                    const uint2 lv = pre && si < (uint32_t)kColdSlots ? lds_u2(slot_addr(t, si))
                                                               : ld_ro_u2_keep(sv.lut + 8ull * min(g, Gm1), pol);  // rare
                    e[j] = make_entry<OUT, true>(lv, fu, bad);
                }
            }
            store8<OUT>(out_s, N, slab_v0 + q, e);
        }
        __syncwarp();
        // this warp is done with the stage: every lane releases its own reads (kAllLanesRelease), or
        // lane 0 for the warp after __syncwarp (bar.warp.sync orders the other lanes' reads)
        if (kAllLanesRelease || lane == 0) mbar_arrive(&ring.empty[(ring.count + t) % kKeyStages]);
    }
    cp_async_wait<0>();
    ring.count += ntiles;
}

// The producer warp's whole life (VEC kernel with kProducerWarp): walk the
// same (item, slab) segments as the consumers, in the same order, and stream
// every key tile they will expand through the ring, refilling a stage the
// moment the last consumer warp releases it.  It never waits on the consumers'
// hot-prefix rebuilds, so the next segment's first tiles are already in shared
// memory when the consumers get there (no ring drain between segments).
// (Inlined: as a __noinline__ call the kernel ran 13% slower on C2.)
template <bool ESC>
__device__ __forceinline__ void kc_produce(const void *const *__restrict__ src, const CosmoMeta *__restrict__ meta,
                                           KeyRing ring, uint64_t i0, uint64_t i1, uint32_t items_per_sample,
                                           uint64_t chunk, uint64_t N, uint64_t plane) {
    uint32_t gt = 0;  // CTA-global tile index, same sequence as the consumers' ring.count
#if SPP_KC_KEY_EF
    const uint64_t key_pol = l2_policy_evict_first();
#endif
#pragma unroll 1
    for (uint64_t it = i0; it < i1; it++) {
        const int s = (int)(it / items_per_sample);
        const uint64_t v0 = (it % items_per_sample) * chunk;
        const uint64_t v1 = min(N, v0 + chunk);
        const CosmoMeta m = meta[s];
        if (!m.valid || 4u * m.nU > (uint32_t)kRegionBytes / 2) continue;  // consumers take the scalar path
        const uint8_t *b = static_cast<const uint8_t *>(src[s]);
        const uint64_t slab_off = ld_le64(b + kSlabOff);
#pragma unroll 1
        for (uint32_t t = 0; t < m.nslab; t++) {
            const SlabView sv = read_slab(b, slab_off, t);
            const uint64_t sa = (uint64_t)sv.z0 * plane, sb = (uint64_t)sv.z1 * plane;
            const uint64_t a = max(v0, sa), e = min(v1, sb);
            const bool escd = ESC && sv.kw == kEscaped && plane % kEscBlock == 0;
            if (a >= e || (sv.kw != 1 && sv.kw != 2 && !escd)) continue;
            const uint32_t kwb = escd ? 1u : (uint32_t)sv.kw;
            EscView ev{};
            if (escd) ev = esc_view(sv, sb - sa);
            const uint64_t ra = a - sa, rb = e - sa;
            const uint32_t ntiles = (uint32_t)((rb - ra + kTileVox - 1) / kTileVox);
#pragma unroll 1
            for (uint32_t k = 0; k < ntiles; k++, gt++) {
                const uint32_t stg = gt % kKeyStages;
                if (gt >= (uint32_t)kKeyStages) mbar_wait(&ring.empty[stg], ((gt / kKeyStages) - 1) & 1u);
                const uint64_t st = ra + (uint64_t)k * kTileVox;
                const uint64_t rem = rb - st;
                const uint32_t nvox = rem < (uint64_t)kTileVox ? (uint32_t)rem : (uint32_t)kTileVox;
                const uint32_t bytes = (nvox * kwb + 15u) & ~15u;
                uint8_t *stage = ring.buf + stg * kStageBytes;
                if (!escd) {
                    fence_proxy_async_smem();
                    mbar_arrive_expect_tx(&ring.full[stg], bytes);
#if SPP_KC_KEY_EF
                    bulk_g2s_hint(stage, sv.keys + st * kwb, bytes, &ring.full[stg], key_pol);
#else
                    bulk_g2s(stage, sv.keys + st * kwb, bytes, &ring.full[stg]);
#endif
                    continue;
                }
                // FORMAT.md 1.5 tile: low bytes, the eidx entries of its blocks (from an
                // aligned entry b0 & ~3) and, when they fit, its escape entries
                const uint32_t b0 = (uint32_t)(st / kEscBlock), b1 = (uint32_t)((st + nvox + kEscBlock - 1) / kEscBlock);
                const uint32_t i_lo = 4u * (b0 & ~3u), i_hi = (4u * (b1 + 1) + 15u) & ~15u;
                const uint32_t e0r = __ldg(ev.eidx + b0), e1r = __ldg(ev.eidx + b1);
                const uint32_t e1 = min(e1r, ev.n_esc), e0 = min(e0r, e1);
                const uint32_t ebytes = e1r >= e0r && e1r <= ev.n_esc && e1 > e0 && esc_copy_bytes(e0, e1) <= kEscCap
                                            ? esc_copy_bytes(e0, e1) : 0u;
                fence_proxy_async_smem();
                mbar_arrive_expect_tx(&ring.full[stg], bytes + (i_hi - i_lo) + ebytes);
#if SPP_KC_KEY_EF
                bulk_g2s_hint(stage, ev.low + st, bytes, &ring.full[stg], key_pol);
#else
                bulk_g2s(stage, ev.low + st, bytes, &ring.full[stg]);
#endif
                bulk_g2s(stage + kIdxOff, reinterpret_cast<const uint8_t *>(ev.eidx) + i_lo, i_hi - i_lo, &ring.full[stg]);
                if (ebytes)
                    bulk_g2s(stage + kEscOff, reinterpret_cast<const uint8_t *>(ev.esc) + ((2u * e0) & ~15u), ebytes,
                             &ring.full[stg]);
            }
        }
    }
}

// CTA-wide barrier of the threads that run the item loop: all of them, or the
// consumer warps only when the producer warp has split off (named barrier 1)
template <bool SPLIT>
__device__ __forceinline__ void loop_sync() {
    if constexpr (SPLIT) asm volatile("bar.sync 1, %0;" ::"n"(kConsumers) : "memory");
    else __syncthreads();
}

template <int OUT, bool VEC, bool ESC>
__global__ void __launch_bounds__(kThreads, kMinBlocks) kc_expand(const void *const *__restrict__ src, int n,
                                                         const float *__restrict__ fU_ws,
                                                         const CosmoMeta *__restrict__ meta, uint8_t *__restrict__ dst,
                                                         int H, int W, uint64_t N, uint64_t chunk,
                                                         uint32_t items_per_sample, uint32_t hot_cap,
                                                         uint32_t *__restrict__ status) {
    using E = typename Entry<OUT>::T;
    constexpr uint32_t EB = sizeof(E);
    extern __shared__ __align__(16) uint8_t smem_raw[];
    const uint32_t region = smem_u32(smem_raw);
    const uint32_t fu_base = region;  // f(U) at the start of the region, hot tuples after it
    uint32_t hot_base = region;
    uint64_t *bars =
        reinterpret_cast<uint64_t *>(smem_raw + kHotBytes + kUCap * 4 + kKeyStages * kStageBytes + kColdSlotBytes);
    KeyRing ring{smem_raw + kHotBytes + kUCap * 4, bars, bars + kKeyStages, 0,
                 smem_u32(smem_raw + kHotBytes + kUCap * 4 + kKeyStages * kStageBytes)};
    if (VEC && threadIdx.x == 0) {
        for (int i = 0; i < kKeyStages; i++) {
            mbar_init(&ring.full[i], 1);
            mbar_init(&ring.empty[i], kAllLanesRelease ? kConsumers : kConsumers / kWarp);
        }
        fence_mbar_init();
    }
    __syncthreads();
    const uint64_t plane = (uint64_t)H * W;
    const uint64_t total_items = (uint64_t)n * items_per_sample;
    const uint64_t per = (total_items + gridDim.x - 1) / gridDim.x;
    const uint64_t i0 = (uint64_t)blockIdx.x * per;
    const uint64_t i1 = min(total_items, i0 + per);
    constexpr bool kSplit = VEC && kProducerWarp;        // producer warp streams keys, consumers expand
    constexpr uint32_t kLoopThreads = kSplit ? (uint32_t)kConsumers : (uint32_t)kThreads;
    if constexpr (kSplit) {
        if (threadIdx.x >= (uint32_t)kConsumers) {
            if (threadIdx.x == (uint32_t)kConsumers)
                kc_produce<ESC>(src, meta, ring, i0, i1, items_per_sample, chunk, N, plane);
            return;
        }
    }
    const size_t ob = OUT == SPP_OUT_F32 ? 4 : 2;
    int cached_s = -1, cached_t = -1;
    uint32_t n_hot = 0;
#pragma unroll 1
    for (uint64_t it = i0; it < i1; it++) {
        const int s = (int)(it / items_per_sample);
        const uint64_t v0 = (it % items_per_sample) * chunk;
        const uint64_t v1 = min(N, v0 + chunk);
        const CosmoMeta m = meta[s];
        if (!m.valid) continue;
        const uint8_t *b = static_cast<const uint8_t *>(src[s]);
        // f(U) lives in shared memory unless |U| would take more than half the region
        const FuView fu{fu_base, fU_ws + (size_t)s * kFuStride, m.nU, 4u * m.nU <= (uint32_t)kRegionBytes / 2};
        const FuView fu_g{fu_base, fu.global, m.nU, false};
        uint8_t *out_s = dst + (uint64_t)s * 4 * N * ob;
        uint32_t bad = 0;  // corrupt key / index seen by this thread in this item
        const uint64_t slab_off = ld_le64(b + kSlabOff);
#pragma unroll 1
        for (uint32_t t = 0; t < m.nslab; t++) {
            const SlabView sv = read_slab(b, slab_off, t);
            const uint64_t sa = (uint64_t)sv.z0 * plane, sb = (uint64_t)sv.z1 * plane;
            const uint64_t a = max(v0, sa), e = min(v1, sb);
            if (a >= e) continue;
            if (sv.kw == 1 || sv.kw == 2 || ((ESC || !VEC) && sv.kw == kEscaped)) {
                if (cached_s != s || cached_t != (int)t) {
                    // stage f(U) and the hottest groups (keys are frequency-ordered) as output tuples;
                    // the LUT tail (cold groups) is prefetched into L2 for the cold lookups
                    loop_sync<kSplit>();
#if SPP_KC_PREFETCH_TAIL
                    if (threadIdx.x == 0 && sv.G > hot_cap) {  // (hot_cap: nominal prefix size)
                        const uint64_t off = 8ull * hot_cap, end = 8ull * sv.G;
                        const uint64_t pol = l2_policy_evict_last();
                        for (uint64_t o = off & ~15ull; o < end; o += 65536) {
                            const uint64_t nb = end - o < 65536 ? ((end - o + 15) & ~15ull) : 65536;
                            prefetch_l2(sv.lut + o, (uint32_t)nb, pol);
                        }
                    }
#endif
                    if (cached_s != s && fu.in_smem)
                        for (uint32_t i = threadIdx.x; i < m.nU; i += kLoopThreads) sts_f32(fu_base + 4 * i, fu.global[i]);
                    loop_sync<kSplit>();
                    const uint32_t fu_bytes = fu.in_smem ? (4u * m.nU + 15u) & ~15u : 0u;
                    hot_base = region + fu_bytes;
                    // hot prefix: as many tuples as fit, but not more than this CTA's
                    // voxels of the slab can amortise (multi-slab samples)
                    const uint64_t cta_end = v0 + (i1 - it) * chunk;  // this CTA's remaining voxels of the sample
                    const uint64_t span = (sb < cta_end ? sb : cta_end) - a;
                    const uint32_t amort = span / 8 > 4096 ? (uint32_t)min(span / 8, (uint64_t)0xFFFFFFFFu) : 4096u;
                    // (an escaped slab on the staging instance keeps the region's last kRkBytes
                    // for its resolved keys)
                    const uint32_t rk = ESC && kEscPrefetch == 2 && sv.kw == kEscaped ? kRkBytes : 0u;
                    n_hot = min(min(sv.G, ((uint32_t)kRegionBytes - fu_bytes - rk) / EB), amort);
#pragma unroll 1
                    for (uint32_t g0 = threadIdx.x; g0 < n_hot; g0 += 4 * kLoopThreads) {
                        uint2 lv[4];
#pragma unroll
                        for (int u = 0; u < 4; u++) {
                            const uint32_t g = g0 + u * kLoopThreads;
                            if (g < n_hot) lv[u] = ld_ro_u2(sv.lut + 8ull * g);
                        }
#pragma unroll
                        for (int u = 0; u < 4; u++) {
                            const uint32_t g = g0 + u * kLoopThreads;
                            if (g < n_hot)
                                sts_entry<OUT>(hot_base + g * EB, fu.in_smem ? make_entry<OUT, true>(lv[u], fu, bad)
                                                                             : make_entry<OUT, false>(lv[u], fu, bad));
                        }
                    }
                    loop_sync<kSplit>();
                    cached_s = s;
                    cached_t = (int)t;
                }
                // escaped-key slabs (FORMAT.md 1.5) take the vector path in the ESC instance
                // (the caller's opts.escape_keys) when blocks align with planes, else the scalar one
                if (VEC && fu.in_smem && (sv.kw != kEscaped || (ESC && plane % kEscBlock == 0))) {
                    if constexpr (VEC)
                        expand_keys_vec<OUT, ESC>(sv, sa, a - sa, e - sa, hot_base, n_hot, fu, out_s, N, bad, ring,
                                                  sb - sa, region + (uint32_t)kRegionBytes - kRkBytes);
                } else if (sv.kw == kEscaped) {
                    // escaped keys off the vector path: scalar, each key resolved by counting the
                    // escapes before it in its block; the thread ending a block checks its eidx
                    if constexpr (ESC || !VEC) {
                        const EscView ev = esc_view(sv, sb - sa);
                        for (uint64_t v = a + threadIdx.x; v < e; v += kLoopThreads) {
                            const uint64_t rel = v - sa;
                            uint32_t g = esc_key_scalar(ev, rel);
                            if ((rel & (kEscBlock - 1)) == kEscBlock - 1 || rel + 1 == sb - sa)
                                bad |= !esc_block_ok(ev, rel / kEscBlock, sb - sa);
                            bad |= g >= sv.G;
                            g = g < sv.G ? g : 0u;
                            const E en = g < n_hot ? lds_entry<OUT>(hot_base + g * EB)
                                                   : make_entry<OUT, false>(ld_ro_u2(sv.lut + 8ull * g), fu_g, bad);
                            store1<OUT>(out_s, N, v, en);
                        }
                    }
                } else {  // scalar path: odd shapes, or |U| too large for shared memory
                    for (uint64_t v = a + threadIdx.x; v < e; v += kLoopThreads) {
                        const uint64_t rel = v - sa;
                        uint32_t g = sv.kw == 2 ? ld_le16(sv.keys + 2 * rel) : sv.keys[rel];
                        bad |= g >= sv.G;
                        g = g < sv.G ? g : 0u;
                        const E en = g < n_hot ? lds_entry<OUT>(hot_base + g * EB)
                                               : make_entry<OUT, false>(ld_ro_u2(sv.lut + 8ull * g), fu_g, bad);
                        store1<OUT>(out_s, N, v, en);
                    }
                }
            } else if (sv.kw == 0) {
                // broadcast of a constant 4-group
                const E en = make_entry<OUT, false>(ld_ro_u2(sv.lut), fu_g, bad);
                if constexpr (VEC) {
                    E e8[8];
#pragma unroll
                    for (int j = 0; j < 8; j++) e8[j] = en;
                    for (uint64_t q = a + (uint64_t)threadIdx.x * 8; q < e; q += (uint64_t)kLoopThreads * 8)
                        store8<OUT>(out_s, N, q, e8);
                } else {
                    for (uint64_t v = a + threadIdx.x; v < e; v += kLoopThreads) store1<OUT>(out_s, N, v, en);
                }
            } else if (VEC && fu.in_smem) {
                // RAW escape slab: four planes of U indices (FORMAT.md 1.1, kw = 8), 8 voxels per thread
                if (cached_s != s) {
                    loop_sync<kSplit>();
                    for (uint32_t i = threadIdx.x; i < m.nU; i += kLoopThreads) sts_f32(fu_base + 4 * i, fu.global[i]);
                    loop_sync<kSplit>();
                    cached_s = s;
                    cached_t = -1;
                }
                const uint64_t Nt = sb - sa;
                for (uint64_t q = a + (uint64_t)threadIdx.x * 8; q < e; q += (uint64_t)kLoopThreads * 8) {
                    const uint64_t rel = q - sa;
                    uint4 pc[4];
#pragma unroll
                    for (int c = 0; c < 4; c++) pc[c] = ld_stream_u4(sv.keys + 2 * ((uint64_t)c * Nt + rel));
                    E e8[8];
#pragma unroll
                    for (int j = 0; j < 8; j++) {
                        uint32_t w[4];
#pragma unroll
                        for (int c = 0; c < 4; c++) {
                            const uint32_t ww = (j >> 1) == 0 ? pc[c].x : (j >> 1) == 1 ? pc[c].y : (j >> 1) == 2 ? pc[c].z : pc[c].w;
                            w[c] = (j & 1) ? ww >> 16 : ww & 0xFFFFu;
                        }
                        e8[j] = make_entry<OUT, true>(make_uint2(w[0] | (w[1] << 16), w[2] | (w[3] << 16)), fu, bad);
                    }
                    store8<OUT>(out_s, N, q, e8);
                }
            } else {
                // RAW escape slab: four planes of U indices (FORMAT.md 1.1, kw = 8)
                const uint64_t Nt = sb - sa;
                for (uint64_t v = a + threadIdx.x; v < e; v += kLoopThreads) {
                    const uint64_t rel = v - sa;
                    uint2 ent;
                    ent.x = (uint32_t)ld_le16(sv.keys + 2 * rel) | ((uint32_t)ld_le16(sv.keys + 2 * (Nt + rel)) << 16);
                    ent.y = (uint32_t)ld_le16(sv.keys + 2 * (2 * Nt + rel)) |
                            ((uint32_t)ld_le16(sv.keys + 2 * (3 * Nt + rel)) << 16);
                    store1<OUT>(out_s, N, v, make_entry<OUT, false>(ent, fu_g, bad));
                }
            }
        }
        if (bad) report(status, SPP_ERR_CORRUPT, s);
    }
}

template <int OUT, bool VEC, bool ESC = false>
spp_status launch_expand(const void *const *d_src, int n, const float *fU, const CosmoMeta *meta, uint8_t *dst,
                         const spp_decode_opts &o, uint64_t N, cudaStream_t stream, const DeviceProps &dp) {
    auto kern = kc_expand<OUT, VEC, ESC>;
    const int entry_bytes = OUT == SPP_OUT_F32 ? 16 : 8;
    const int smem = kSmemBytes;
    if (set_smem_attr<kc_expand<OUT, VEC, ESC>>(smem, dp) != SPP_OK) return SPP_ERR_CUDA;  // per device
    int occ = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kThreads, smem) != cudaSuccess || occ < 1)
        return SPP_ERR_CUDA;
    const int ctas = dp.sms * occ;
    // chunk: multiple of 2*8*kThreads voxels, at least ~8 items per CTA slot
    uint64_t chunk = 4096;
    const uint64_t want_items = (uint64_t)ctas * 8;
    while (chunk < (1u << 18) && (uint64_t)n * ((N + chunk * 2 - 1) / (chunk * 2)) >= want_items) chunk *= 2;
    if (!VEC) chunk = std::max<uint64_t>(1, std::min<uint64_t>(chunk, N));
    const uint32_t ips = (uint32_t)((N + chunk - 1) / chunk);
    const uint64_t items = (uint64_t)n * ips;
    const int grid = (int)std::min<uint64_t>(items, (uint64_t)ctas);
    kern<<<grid, kThreads, smem, stream>>>(d_src, n, fU, meta, dst, o.H, o.W, N, chunk, ips,
                                           (uint32_t)(kHotBytes / entry_bytes), o.status);
    return cudaGetLastError() == cudaSuccess ? SPP_OK : SPP_ERR_CUDA;
}

}  // namespace

static spp_status cosmo_expand(const void *const *d_src, int n, void *d_dst, const spp_decode_opts &o,
                               cudaStream_t stream, const DeviceProps &dp, float *fU, CosmoMeta *meta);

size_t cosmo_workspace_bytes(int n) {
    if (n <= 0) return 0;
    return meta_offset(n) + round_up16((size_t)n * sizeof(CosmoMeta));
}

spp_status cosmo_decode(const void *const *d_src, int n, void *d_dst, const spp_decode_opts &o,
                        cudaStream_t stream) {
    DeviceProps dp;
    spp_status st = current_device_props(&dp);
    if (st != SPP_OK) return st;
    uint8_t *ws = static_cast<uint8_t *>(o.workspace);
    float *fU = reinterpret_cast<float *>(ws);
    CosmoMeta *meta = reinterpret_cast<CosmoMeta *>(ws + meta_offset(n));
    cudaEvent_t const *ev = reinterpret_cast<cudaEvent_t const *>(o.timing_events);
    if (ev && cudaEventRecord(ev[0], stream) != cudaSuccess) return SPP_ERR_CUDA;
    // escaped-key slabs (FORMAT.md 1.5) decode on the instance selected by opts.escape_keys or on
    // the scalar kernel (shapes off the vector path); the paper-format vector kernel never sees them
    const uint64_t plane = (uint64_t)o.H * o.W;
    const size_t align = o.out == SPP_OUT_F32 ? 32 : 16;
    const bool vec = plane % 16 == 0 && (reinterpret_cast<uintptr_t>(d_dst) % align) == 0;
    const int esc_ok = !vec || o.escape_keys;
    kc0_prologue<<<n, kPrologueThreads, 0, stream>>>(d_src, o.src_bytes, o.transform, o.D, o.H, o.W, fU, meta, o.status,
                                                     esc_ok);
    if (cudaGetLastError() != cudaSuccess) return SPP_ERR_CUDA;
    if (ev && cudaEventRecord(ev[1], stream) != cudaSuccess) return SPP_ERR_CUDA;
    spp_status r = cosmo_expand(d_src, n, d_dst, o, stream, dp, fU, meta);
    if (r == SPP_OK && ev && cudaEventRecord(ev[2], stream) != cudaSuccess) return SPP_ERR_CUDA;
    return r;
}

static spp_status cosmo_expand(const void *const *d_src, int n, void *d_dst, const spp_decode_opts &o,
                               cudaStream_t stream, const DeviceProps &dp, float *fU, CosmoMeta *meta) {
    const uint64_t N = (uint64_t)o.D * o.H * o.W;
    const uint64_t plane = (uint64_t)o.H * o.W;
    const size_t align = o.out == SPP_OUT_F32 ? 32 : 16;
    const bool vec = plane % 16 == 0 && (reinterpret_cast<uintptr_t>(d_dst) % align) == 0;  // 16-B key tiles
    uint8_t *dst = static_cast<uint8_t *>(d_dst);
    // opts.escape_keys selects the instance that stages FORMAT.md 1.5 escaped keys
    const bool esc = vec && o.escape_keys && kProducerWarp;
    switch (o.out) {
        case SPP_OUT_F16:
            return esc   ? launch_expand<SPP_OUT_F16, true, true>(d_src, n, fU, meta, dst, o, N, stream, dp)
                   : vec ? launch_expand<SPP_OUT_F16, true>(d_src, n, fU, meta, dst, o, N, stream, dp)
                         : launch_expand<SPP_OUT_F16, false>(d_src, n, fU, meta, dst, o, N, stream, dp);
        case SPP_OUT_F32:
            return esc   ? launch_expand<SPP_OUT_F32, true, true>(d_src, n, fU, meta, dst, o, N, stream, dp)
                   : vec ? launch_expand<SPP_OUT_F32, true>(d_src, n, fU, meta, dst, o, N, stream, dp)
                         : launch_expand<SPP_OUT_F32, false>(d_src, n, fU, meta, dst, o, N, stream, dp);
        case SPP_OUT_I16:
            return esc   ? launch_expand<SPP_OUT_I16, true, true>(d_src, n, fU, meta, dst, o, N, stream, dp)
                   : vec ? launch_expand<SPP_OUT_I16, true>(d_src, n, fU, meta, dst, o, N, stream, dp)
                         : launch_expand<SPP_OUT_I16, false>(d_src, n, fU, meta, dst, o, N, stream, dp);
        default:
            return SPP_ERR_INVALID_ARG;
    }
}

}  // namespace spp
