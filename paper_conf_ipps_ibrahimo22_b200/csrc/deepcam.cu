// deepcam.cu — DeepCAM decode + per-channel normalisation on sm_100a
// (FORMAT.md 2.3).
//
// PAPER.md §V.A: lines along x are split into segments with a head
// value and 8-bit minifloat differences relative to a per-segment minimum
// exponent; abrupt lines are stored raw; constant runs are broadcast; per-line
// metadata makes every line independently decodable.  §VI: the
// loop-carried dependency is handled with hierarchical parallelism — here one
// warp per line, lanes cooperating on the inner loop.
//
//   KD0  kd0_parse     one thread per sample: validate header, publish the line
//                      directory / payload pointers.
//   KD   kd_decode_ws  persistent, warp-specialised: one producer warp per CTA
//                      streams each consumer warp's lines (line record by
//                      st.async + bytes by 1-D TMA) into a 3-slot ring in shared
//                      memory; each consumer warp decodes one line at a time.
//                      Line paths (all bit-identical, FORMAT.md 2.3):
//                      * one pass (W = 1152, A = 36, <= 32 segments): lane l owns
//                        positions [36l, 36l+36), codes -> exact fp16 pairs, two
//                        exact fp32 prefix chains, one warp scan; the row is
//                        staged in a per-warp row buffer and leaves by one TMA
//                        bulk store (decode_line_onepass);
//                      * aligned (A = positions per lane): block bitmap + scans
//                        (decode_line_aligned);
//                      * general (any A, RAW / RAW16 / mode-3 lines): start bitmap,
//                        prefix counts, segmented warp scan (decode_line);
//                      * global (a line longer than the ring, or W too large for
//                        the shared tables): decoded straight from HBM, segment
//                        by segment, with an exact int32 prefix scan
//                        (decode_line_global).  Every FORMAT-legal line decodes.
//                      The instance selected by opts.raw_segments also takes
//                      mode-3 lines (FORMAT.md 2.7) and RAW16 lines (2.6) in one
//                      pass.
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>

#include "common.cuh"
#include "spp_format.h"
#include "spp_internal.h"

namespace spp {
namespace {

using namespace spp::deepcam;

// L2 policy of the decoded rows' TMA bulk stores (written once): 1 = evict_first hint
// (r2: C4 0.844 -> 0.851 of the measured peak, 3 alternating runs, profiles/r02a8_*)
#ifndef SPP_KD_ROW_EF
#define SPP_KD_ROW_EF 1
#endif
constexpr uint64_t kRowEfBytes = 64ull << 20;  // launches writing more than this (half of L2) use evict_first
struct DcMeta {  // written by KD0, read by KD (32 B)
    const uint8_t *dir;
    const uint8_t *payload;
    uint64_t limit;  // bytes available from payload
    uint32_t valid;
    uint32_t align;  // declared segment alignment A (FORMAT.md 2.1)
};

// Lines of W > kSmemMaxW take the global path (the shared start-bitmap / prefix
// tables of the general path are sized by W); FORMAT.md allows W <= 65535.
constexpr uint32_t kSmemMaxW = 8192;

__global__ void kd0_parse(const void *const *__restrict__ src, const uint64_t *__restrict__ src_bytes, int n, int C,
                          int H, int W, DcMeta *__restrict__ meta, uint32_t *__restrict__ status) {
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= n) return;
    const uint8_t *b = static_cast<const uint8_t *>(src[s]);
    const uint64_t limit = src_bytes ? src_bytes[s] : ~0ull;
    bool ok = b != nullptr && (reinterpret_cast<uintptr_t>(b) & 15) == 0 && limit >= (uint64_t)kHeaderBytes;
    DcMeta m{nullptr, nullptr, 0, 0, 0};
    if (ok) {
        const uint64_t L = (uint64_t)C * H;
        ok = ld_le32(b) == kDeepcamMagic && ld_le16(b + 4) == kVersion && ld_le16(b + kC) == C &&
             ld_le16(b + kH) == H && ld_le16(b + kW) == W && ld_le32(b + kL) == L;
        const uint64_t dir_off = ld_le64(b + kDirOff), pay = ld_le64(b + kPayloadOff), total = ld_le64(b + kTotal);
        const uint32_t A = ld_le16(b + kAlign);
        // every range as off <= total && len <= total - off: stream-supplied 64-bit
        // offsets never wrap an addition
        ok = ok && total <= limit && (dir_off & 3) == 0 && dir_off <= total && 4 * (L + 1) <= total - dir_off &&
             (pay & 15) == 0 && pay <= total && A >= 1 && (uint32_t)W % A == 0;
        if (ok) m = DcMeta{b + dir_off, b + pay, total - pay, 1u, A};
    }
    if (!ok) report(status, SPP_ERR_CORRUPT, s);
    meta[s] = m;
}

// delta byte -> code value as an fp32 multiple of 2^-130 (exact; FORMAT.md 2.2):
// sign bit -> bit 31, the 7 exponent|mantissa bits -> bits 19..25, so that
// E = 0 lands on fp32 subnormals (M * 2^-130) and E >= 1 on (16+M) * 2^(E-131).
template <int K>
__device__ __forceinline__ float code_f(uint32_t w) {
    uint32_t r;
    if constexpr (K == 0) r = ((w << 24) & 0x80000000u) | ((w << 19) & 0x03F80000u);
    else if constexpr (K == 1) r = ((w << 16) & 0x80000000u) | ((w << 11) & 0x03F80000u);
    else if constexpr (K == 2) r = ((w << 8) & 0x80000000u) | ((w << 3) & 0x03F80000u);
    else r = (w & 0x80000000u) | ((w >> 5) & 0x03F80000u);
    return __uint_as_float(r);
}
// same value, arithmetic-shift form: byte K moved to the top, sign-extending
// shift by 5, then one mask keeps bit 31 (sign) and bits 19..25 (E|M)
template <int K>
__device__ __forceinline__ float code_f_sar(uint32_t w) {
    const int32_t t = (int32_t)(w << (24 - 8 * K));
    return __uint_as_float((uint32_t)(t >> 5) & 0x83F80000u);
}
// Two delta codes as an fp16 pair: the code's 7 E|M bits land on fp16 bits
// 6..12 and its sign on bit 15, so the half equals code * 2^-18 exactly (E = 0
// maps onto fp16 subnormals). prmt puts code byte `lo` in bits 8..15 with its
// sign replicated into bits 16..23 and code byte `hi` in bits 24..31; one
// arithmetic shift by 2 moves both E|M fields into place while copying each
// sign into bits 13..15 / 29..31, and one mask keeps sign + E|M.
template <uint32_t SEL>
__device__ __forceinline__ uint32_t codes_h2(uint32_t w) {
    uint32_t x;
    asm("prmt.b32 %0, %1, 0, %2;" : "=r"(x) : "r"(w), "n"(SEL));
    return (uint32_t)((int32_t)x >> 2) & 0x9FC09FC0u;
}
// RN(float(a) + c) with a an fp16 (mixed-precision add, sm_100: FHADD)
__device__ __forceinline__ float fadd_h(uint32_t h2, int hi, float c) {
    const uint16_t a = (uint16_t)(hi ? (h2 >> 16) : (h2 & 0xFFFFu));
    float d;
    asm("add.rn.f32.f16 %0, %1, %2;" : "=f"(d) : "h"(a), "f"(c));
    return d;
}
__device__ __forceinline__ float code_f_byte(uint32_t b) {
    return __uint_as_float(((b & 0x80u) << 24) | ((b & 0x7Fu) << 19));
}

// Inclusive warp scans whose shuffle also yields the "source lane in range"
// predicate (shfl.sync.up's second destination), so each step is SHFL + one
// predicated add (no separate lane >= d compare / select).
__device__ __forceinline__ uint32_t scan_incl_u32(uint32_t v) {
#pragma unroll
    for (int d = 1; d < kWarp; d <<= 1)
        asm("{\n.reg .u32 t;\n.reg .pred p;\nshfl.sync.up.b32 t|p, %0, %1, 0, 0xffffffff;\n@p add.u32 %0, %0, t;\n}\n"
            : "+r"(v)
            : "r"(d));
    return v;
}
__device__ __forceinline__ float scan_incl_f32(float v) {  // exact here: sums of codes (see callers)
#pragma unroll
    for (int d = 1; d < kWarp; d <<= 1)
        asm("{\n.reg .f32 t;\n.reg .pred p;\nshfl.sync.up.b32 t|p, %0, %1, 0, 0xffffffff;\n@p add.rn.f32 %0, %0, t;\n}\n"
            : "+f"(v)
            : "r"(d));
    return v;
}

// per-segment packed info written in place of the descriptor:
//   bits 0..21  byte base a + 2^21 (DIFF: the delta byte of position p is dl[a + p];
//               RAW segment: its value is the binary32 at dl + a + 4p), any W <= 65535
//   bits 22..23 kind (validated <= 2 before packing), bits 24..31 emin_b
constexpr int kBaseBias = 1 << 21;
__device__ __forceinline__ uint32_t pack_seg(int a, uint32_t kind, uint32_t eb) {
    return ((uint32_t)(a + kBaseBias) & 0x3FFFFFu) | ((kind & 3u) << 22) | (eb << 24);
}
struct SegInfo {
    float h;
    float sc;      // 2^(emin+130) (emin <= -3) or 2^(emin+30) (big)
    int a;
    uint32_t kind;
    uint32_t big;
};
__device__ __forceinline__ SegInfo seg_info(const uint32_t *desc, const float *heads, int s) {
    const uint32_t d = desc[s];
    SegInfo si;
    si.h = heads[s];
    si.a = (int)(d & 0x3FFFFFu) - kBaseBias;
    si.kind = (d >> 22) & 3u;
    const uint32_t eb = d >> 24;
    si.big = eb >= 148u;
    si.sc = __uint_as_float((si.big ? (eb + 7u) : (eb + 107u)) << 23);
    return si;
}

// binary32 at any byte address of shared memory (RAW segments, FORMAT.md 2.7)
__device__ __forceinline__ float lds_f32_any(uint32_t addr) {
    const uint32_t al = addr & ~3u, sh = (addr & 3u) * 8u;
    uint32_t w0, w1;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(w0) : "r"(al));
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(w1) : "r"(al + 4));
    return __uint_as_float(__funnelshift_r(w0, w1, sh));
}

template <int OUT>
__device__ __forceinline__ void emit8(uint8_t *row, uint32_t p0, uint32_t W, const float (&y)[8]) {
    if constexpr (OUT == SPP_OUT_F32) {
        st_stream_f8(row + 4ull * p0, y);
    } else {
        uint4 u;
        __half2 h0 = __floats2half2_rn(y[0], y[1]), h1 = __floats2half2_rn(y[2], y[3]);
        __half2 h2 = __floats2half2_rn(y[4], y[5]), h3 = __floats2half2_rn(y[6], y[7]);
        u.x = *reinterpret_cast<uint32_t *>(&h0);
        u.y = *reinterpret_cast<uint32_t *>(&h1);
        u.z = *reinterpret_cast<uint32_t *>(&h2);
        u.w = *reinterpret_cast<uint32_t *>(&h3);
        st_stream_u4(row + 2ull * p0, u);
    }
}
template <int OUT>
__device__ __forceinline__ void emit_scalar(uint8_t *row, uint32_t p0, uint32_t W, const float (&y)[8]) {
#pragma unroll
    for (int j = 0; j < 8; j++) {
        if (p0 + j < W) {
            if constexpr (OUT == SPP_OUT_F32) reinterpret_cast<float *>(row)[p0 + j] = y[j];
            else reinterpret_cast<__half *>(row)[p0 + j] = __float2half_rn(y[j]);
        }
    }
}

// Decode one staged line (warp-cooperative).  Returns false if malformed.
template <int OUT, bool VEC>
__device__ __forceinline__ bool decode_line(uint8_t *buf, uint32_t bytes, uint32_t W, uint32_t A, uint32_t *sbits,
                                            uint32_t *wpre, uint32_t nwords, float shv, float scv, uint8_t *row,
                                            int lane) {
    const uint32_t hdr = *reinterpret_cast<const uint32_t *>(buf);
    const uint32_t mode = hdr & 0xFFu;
    if (mode == kModeRaw) {
        if (16u + 4u * W > bytes) return false;
        const float *x = reinterpret_cast<const float *>(buf + 16);
        for (uint32_t c0 = 0; c0 < W; c0 += 256) {
            const uint32_t p0 = c0 + 8 * lane;
            if (p0 >= W) continue;
            float y[8];
            if constexpr (VEC) {
                const float4 a = *reinterpret_cast<const float4 *>(x + p0);
                const float4 b = *reinterpret_cast<const float4 *>(x + p0 + 4);
                const float xv[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
#pragma unroll
                for (int j = 0; j < 8; j++) y[j] = __fmul_rn(__fsub_rn(xv[j], shv), scv);
                emit8<OUT>(row, p0, W, y);
            } else {
#pragma unroll
                for (int j = 0; j < 8; j++) y[j] = p0 + j < W ? __fmul_rn(__fsub_rn(x[p0 + j], shv), scv) : 0.f;
                emit_scalar<OUT>(row, p0, W, y);
            }
        }
        return true;
    }
    if (mode == kModeRaw16) {  // FORMAT.md 2.6: binary16 values, widened exactly
        if (16u + 2u * W > bytes) return false;
        const __half *x = reinterpret_cast<const __half *>(buf + 16);
        for (uint32_t c0 = 0; c0 < W; c0 += 256) {
            const uint32_t p0 = c0 + 8 * lane;
            if (p0 >= W) continue;
            float y[8];
            if constexpr (VEC) {
                const uint4 v = *reinterpret_cast<const uint4 *>(x + p0);
                const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
                for (int j = 0; j < 8; j++) {
                    const float xv = __half2float(__ushort_as_half((unsigned short)((w[j >> 1] >> (16 * (j & 1))) & 0xFFFFu)));
                    y[j] = __fmul_rn(__fsub_rn(xv, shv), scv);
                }
                emit8<OUT>(row, p0, W, y);
            } else {
#pragma unroll
                for (int j = 0; j < 8; j++)
                    y[j] = p0 + j < W ? __fmul_rn(__fsub_rn(__half2float(x[p0 + j]), shv), scv) : 0.f;
                emit_scalar<OUT>(row, p0, W, y);
            }
        }
        return true;
    }
    if (mode != kModeSeg && mode != kModeSegRaw) return false;
    const uint32_t max_kind = mode == kModeSegRaw ? kRawSeg : kDiff;  // RAW segments: FORMAT.md 2.7
    const uint32_t nseg = hdr >> 16;
    if (nseg < 1 || nseg > W || 4u + 8u * nseg > bytes) return false;
    uint32_t *desc = reinterpret_cast<uint32_t *>(buf + 4);
    const float *heads = reinterpret_cast<const float *>(buf + 4 + 4 * nseg);
    const uint8_t *dl = buf + 4 + 8 * nseg;

    // 1. segment table: starts (bitmap), byte bases (in place), validation
    for (uint32_t w = lane; w < nwords; w += kWarp) sbits[w] = 0;
    __syncwarp();
    uint32_t cl = 0, cd = 0;
    bool bad = false;
    for (uint32_t b0 = 0; b0 < nseg; b0 += kWarp) {
        const uint32_t s = b0 + lane;
        uint32_t len = 0, kind = 0, eb = 0;
        if (s < nseg) {
            const uint32_t d = desc[s];
            len = d & 0xFFFFu;
            kind = (d >> 16) & 0xFFu;
            eb = d >> 24;
        }
        const uint32_t dlen = (kind == kDiff && len > 0) ? len - 1 : (kind == kRawSeg ? 4u * len : 0u);
        const uint32_t il = warp_incl_scan(len, lane), id = warp_incl_scan(dlen, lane);
        const uint32_t st = cl + il - len, db = cd + id - dlen;
        if (s < nseg) {
            bad |= len == 0 || kind > max_kind ||
                   (kind == kDiff && (eb < (uint32_t)kEminBMin || eb > (uint32_t)kEminBMax)) || st + len > W ||
                   st % A != 0;
            if (st < W) atomicOr(&sbits[st >> 5], 1u << (st & 31));
            // DIFF: the code of position p is byte a + p; RAW: its value is at bytes a + 4p
            const int a = kind == kRawSeg ? (int)db - 4 * (int)st : (int)db - (int)st - 1;
            desc[s] = pack_seg(a, kind, eb);
        }
        cl += __shfl_sync(0xffffffffu, il, 31);
        cd += __shfl_sync(0xffffffffu, id, 31);
    }
    bad = __any_sync(0xffffffffu, bad) || cl != W || 4u + 8u * nseg + cd > bytes;
    if (bad) return false;
    __syncwarp();
    // starts in the bitmap words before word w (segment index of a position =
    // starts before it + starts at or below it in its word - 1)
    {
        uint32_t carry_w = 0;
        for (uint32_t w0 = 0; w0 < nwords; w0 += kWarp) {
            const uint32_t w = w0 + lane;
            const uint32_t c = w < nwords ? __popc(sbits[w]) : 0u;
            const uint32_t ic = warp_incl_scan(c, lane);
            if (w < nwords) wpre[w] = carry_w + ic - c;
            carry_w += __shfl_sync(0xffffffffu, ic, 31);
        }
    }
    __syncwarp();

    // 2. chunks of 256 positions, lane owns [p0, p0 + 8).  All code sums are
    // fp32 multiples of 2^-130 below 2^-106 in magnitude: exact in any order.
    const uint32_t dl_s = smem_u32(dl);
    float carry_P = 0.f;     // line prefix of codes before this chunk
    float carry_base = 0.f;  // line prefix before the head of the segment open at the chunk start
    const uint32_t below_mask = (1u << lane) - 1u;
    for (uint32_t c0 = 0; c0 < W; c0 += 256) {
        const uint32_t p0 = c0 + 8 * lane;
        const bool act = p0 < W;
        uint32_t sb = 0, valid = 0, nbefore = 0;
        if (act) {
            const uint32_t word = sbits[p0 >> 5];
            sb = (word >> (p0 & 31)) & 0xFFu;
            valid = W - p0 >= 8 ? 0xFFu : ((1u << (W - p0)) - 1u);
            sb &= valid;
            nbefore = wpre[p0 >> 5] + __popc(word & ((1u << (p0 & 31)) - 1u));
        }
        const int s_prev = (int)nbefore - 1;  // segment of position p0 - 1

        // local sums: r[j] = codes since the last head in the lane (or since p0),
        // pl = plain lane total, lv = plain prefix before the lane's last head
        float r[8], hj[8], scj[8];
        uint32_t started = 0, keep = 0, bigm = 0;
        float pl = 0.f, lv = 0.f;
        if (!__any_sync(0xffffffffu, (sb >> 1) != 0)) {
            // fast path: every lane's 8 positions lie in one segment (head allowed at p0)
            const int s = act ? s_prev + (int)(sb & 1u) : 0;
            const SegInfo si = seg_info(desc, heads, s);
            float f[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
            if (act && si.kind == kDiff) {
                const uint32_t addr = dl_s + (uint32_t)(si.a + (int)p0);
                const uint32_t al = addr & ~3u, shb = (addr & 3u) * 8u;
                uint32_t w0, w1, w2;
                asm volatile("ld.shared.u32 %0, [%1];" : "=r"(w0) : "r"(al));
                asm volatile("ld.shared.u32 %0, [%1];" : "=r"(w1) : "r"(al + 4));
                asm volatile("ld.shared.u32 %0, [%1];" : "=r"(w2) : "r"(al + 8));
                uint32_t lo = __funnelshift_r(w0, w1, shb), hi = __funnelshift_r(w1, w2, shb);
                if (sb & 1u) lo &= 0xFFFFFF00u;  // the head has no delta byte
                if (valid != 0xFFu) {           // positions past the line end
                    const uint64_t m = (1ull << (8 * __popc(valid))) - 1ull;
                    lo &= (uint32_t)m;
                    hi &= (uint32_t)(m >> 32);
                }
                f[0] = code_f<0>(lo); f[1] = code_f<1>(lo); f[2] = code_f<2>(lo); f[3] = code_f<3>(lo);
                f[4] = code_f<0>(hi); f[5] = code_f<1>(hi); f[6] = code_f<2>(hi); f[7] = code_f<3>(hi);
            }
            r[0] = f[0];
#pragma unroll
            for (int j = 1; j < 8; j++) r[j] = r[j - 1] + f[j];
            pl = r[7];
#pragma unroll
            for (int j = 0; j < 8; j++) { hj[j] = si.h; scj[j] = si.sc; }
            started = (sb & 1u) ? 0xFFu : 0u;
            keep = si.kind == kRepeat ? 0xFFu : (sb & 1u);
            if (act && si.kind == kRawSeg) {  // RAW segment: every position is its stored value
#pragma unroll
                for (int j = 0; j < 8; j++)
                    if ((valid >> j) & 1u) hj[j] = lds_f32_any(dl_s + (uint32_t)(si.a + 4 * (int)(p0 + j)));
                keep = 0xFFu;
            }
            bigm = si.big ? 0xFFu : 0u;
        } else {
            // general path: segment heads inside the lane's 8 positions
            int s = s_prev;
            SegInfo si = seg_info(desc, heads, s < 0 ? 0 : s);
            float run = 0.f;
#pragma unroll
            for (int j = 0; j < 8; j++) {
                const uint32_t p = p0 + j;
                float hraw = 0.f;
                bool israw = false;
                if ((sb >> j) & 1u) {
                    s++;
                    si = seg_info(desc, heads, s);
                    lv = pl;  // plain prefix before this head
                    run = 0.f;
                    started |= 0xFFu << j;
                    keep |= 1u << j;
                    israw = si.kind == kRawSeg;
                } else if ((valid >> j) & 1u) {
                    if (si.kind == kRepeat) {
                        keep |= 1u << j;
                    } else if (si.kind == kRawSeg) {
                        keep |= 1u << j;
                        israw = true;
                    } else {
                        const float f = code_f_byte(dl[si.a + (int)p]);
                        run += f;
                        pl += f;
                    }
                }
                if (israw) hraw = lds_f32_any(dl_s + (uint32_t)(si.a + 4 * (int)p));
                r[j] = run;
                hj[j] = israw ? hraw : si.h;
                scj[j] = si.sc;
                if (si.big) bigm |= 1u << j;
            }
            started &= 0xFFu;
        }
        // plain inclusive warp scan of the lane totals
        float P = pl;
#pragma unroll
        for (int d = 1; d < kWarp; d <<= 1) {
            const float y = __shfl_up_sync(0xffffffffu, P, d);
            if (lane >= d) P += y;
        }
        const float P_excl = carry_P + (P - pl);      // line prefix before p0
        const float lastbase = P_excl + lv;           // prefix before this lane's last head
        const uint32_t smask = __ballot_sync(0xffffffffu, sb != 0);
        const uint32_t below = smask & below_mask;
        const int src = below ? 31 - __clz(below) : lane;
        const float gotb = __shfl_sync(0xffffffffu, lastbase, src);
        const float B_in = below ? gotb : carry_base;  // prefix before the head of the segment open at p0
        const float dlt = P_excl - B_in;
        carry_P += __shfl_sync(0xffffffffu, P, 31);
        const float topb = __shfl_sync(0xffffffffu, lastbase, smask ? 31 - __clz(smask) : 0);
        if (smask) carry_base = topb;
        if (!act) continue;
        float y[8];
#pragma unroll
        for (int j = 0; j < 8; j++) {
            float S = ((started >> j) & 1u) ? r[j] : r[j] + dlt;  // exact
            if ((bigm >> j) & 1u) S *= 0x1p100f;                   // keep the scale representable
            const float xh = ((keep >> j) & 1u) ? hj[j] : __fmaf_rn(S, scj[j], hj[j]);
            y[j] = __fmul_rn(__fsub_rn(xh, shv), scv);
        }
        if constexpr (VEC) emit8<OUT>(row, p0, W, y);
        else emit_scalar<OUT>(row, p0, W, y);
    }
    return true;
}

// ---------------------------------------------------------------------------
// Aligned fast path: the sample declares segment alignment A == VPL, so each
// lane's VPL positions lie in exactly one segment and a segment head can only
// sit at a lane's first position.  One bitmap word per 32*VPL-position chunk
// (bit = "a segment starts at this lane's p0") gives every lane its segment
// index with one shared load and a popc.
template <int VPL>
struct Bytes {  // VPL delta bytes starting at an arbitrary shared address, as VPL/4 words
    static constexpr int NW = VPL / 4;
    uint32_t w[NW];
    __device__ __forceinline__ void load(uint32_t addr) {
        const uint32_t al = addr & ~3u, sh = (addr & 3u) * 8u;
        uint32_t v[NW + 1];
#pragma unroll
        for (int k = 0; k <= NW; k++) asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v[k]) : "r"(al + 4 * k));
#pragma unroll
        for (int k = 0; k < NW; k++) w[k] = __funnelshift_r(v[k], v[k + 1], sh);
    }
};

template <int OUT, int VPL>
__device__ __forceinline__ void emit_vpl(uint8_t *row, uint32_t p0, const float (&y)[VPL]) {
    static_assert(VPL == 8, "direct stores: 16-B lanes");
    emit8<OUT>(row, p0, 0, y);
}

// one-pass lines (VPL = 36): the warp's output row is staged in shared memory
// (lane l writes its VPL values at l*VPL) and leaves with one TMA bulk store
template <int OUT, int VPL>
__device__ __forceinline__ void stage_vpl(uint32_t sdst, const float (&y)[VPL]) {
    if constexpr (OUT == SPP_OUT_F32) {
#pragma unroll
        for (int k = 0; k < VPL / 4; k++)
            sts_u4(sdst + 16 * k, make_uint4(__float_as_uint(y[4 * k]), __float_as_uint(y[4 * k + 1]),
                                             __float_as_uint(y[4 * k + 2]), __float_as_uint(y[4 * k + 3])));
    } else {
#pragma unroll
        for (int k = 0; k < VPL / 4; k++) {
            __half2 a = __floats2half2_rn(y[4 * k], y[4 * k + 1]);
            __half2 b = __floats2half2_rn(y[4 * k + 2], y[4 * k + 3]);
            sts_u2(sdst + 8 * k, make_uint2(*reinterpret_cast<uint32_t *>(&a), *reinterpret_cast<uint32_t *>(&b)));
        }
    }
}

// The one-pass instances stage each output row in a per-warp row buffer (not
// in the line's input slot, which the producer refills by TMA): acquire waits
// until the previous row's bulk store has finished reading the buffer, release
// hands the staged row to the TMA engine.  The input slot is only ever read by
// the consumer's generic loads, so its release/refill needs no proxy fence.
__device__ __forceinline__ void row_buffer_acquire(int lane) {
    if (lane == 0) bulk_wait_read_all();
    __syncwarp();
}
template <int OUT>
__device__ __forceinline__ void row_buffer_release(uint8_t *row, uint8_t *rowbuf, uint32_t W, int lane, uint64_t rpol) {
    fence_proxy_async_smem();  // this lane's row writes -> visible to the async proxy
    __syncwarp();
    if (lane == 0) bulk_s2g_hint(row, rowbuf, W * (OUT == SPP_OUT_F32 ? 4u : 2u), rpol);
}

template <int OUT, int VPL>
__device__ __forceinline__ bool decode_line_aligned(uint8_t *buf, uint32_t bytes, uint32_t W, uint32_t *bbits,
                                                    uint32_t nbw, float shv, float scv, uint8_t *row, uint8_t *rowbuf,
                                                    int lane, uint64_t rpol) {
    constexpr bool STAGED = VPL == 36;  // one pass per line (W = 32 * VPL): row staged in rowbuf, one TMA bulk store
    const uint32_t hdr = *reinterpret_cast<const uint32_t *>(buf);
    const uint32_t nseg = hdr >> 16;
    if (nseg < 1 || nseg > W || 4u + 8u * nseg > bytes) return false;
    uint32_t *desc = reinterpret_cast<uint32_t *>(buf + 4);
    const float *heads = reinterpret_cast<const float *>(buf + 4 + 4 * nseg);
    const uint32_t dl_s = smem_u32(buf + 4 + 8 * nseg);

    // segment table: one packed scan of (len | delta-bytes << 16) gives starts
    // and byte bases; starts go to the block bitmap, byte bases in place
    if ((uint32_t)lane < nbw) bbits[lane] = 0;
    __syncwarp();
    uint32_t cacc = 0;
    bool bad = false;
    for (uint32_t b0 = 0; b0 < nseg; b0 += kWarp) {
        const uint32_t s = b0 + lane;
        uint32_t len = 0, kind = 0, eb = 0;
        if (s < nseg) {
            const uint32_t d = desc[s];
            len = d & 0xFFFFu;
            kind = (d >> 16) & 0xFFu;
            eb = d >> 24;
        }
        const uint32_t dlen = (kind == kDiff && len > 0) ? len - 1 : 0;
        const uint32_t pk = len | (dlen << 16);  // both sums stay below 2^16 (W <= 16383)
        const uint32_t inc = warp_incl_scan(pk, lane);
        const uint32_t ex = cacc + inc - pk;
        const uint32_t st = ex & 0xFFFFu, db = ex >> 16;
        if (s < nseg) {
            const uint32_t blk = st / VPL;
            bad |= len == 0 || kind > kDiff || (kind == kDiff && (eb < (uint32_t)kEminBMin || eb > (uint32_t)kEminBMax)) ||
                   st + len > W || blk * VPL != st;
            if (st < W) atomicOr(&bbits[blk >> 5], 1u << (blk & 31));
            desc[s] = pack_seg((int)db - (int)st - 1, kind, eb);
        }
        cacc += __shfl_sync(0xffffffffu, inc, 31);
    }
    bad = __any_sync(0xffffffffu, bad) || (cacc & 0xFFFFu) != W || 4u + 8u * nseg + (cacc >> 16) > bytes;
    if (bad) return false;
    __syncwarp();

    const uint32_t below = (1u << lane) - 1u;
    const uint32_t le_mask = 0xFFFFFFFFu >> (31 - lane);
    float carry_P = 0.f, carry_base = 0.f;
    uint32_t carry_seg = 0;
    for (uint32_t c = 0, c0 = 0; c0 < W; c++, c0 += 32 * VPL) {
        const uint32_t p0 = c0 + VPL * lane;
        const bool act = p0 < W;
        const uint32_t word = bbits[c];
        const uint32_t flag = act ? (word >> lane) & 1u : 0u;  // a segment starts at p0
        const int s = act ? (int)(carry_seg + __popc(word & below) + flag) - 1 : 0;
        carry_seg += __popc(word);
        const SegInfo si = seg_info(desc, heads, s);
        // Every lane runs the same straight-line code.  Signed zeros make the
        // special cases exact without branches: a REPEAT lane decodes delta
        // bytes 0x80 (code -0) and uses dlt = -0, so S = -0 there and
        // fma(-0, sc, h) == h bit for bit (also for h = +-0); a head lane's
        // position 0 takes S = -0 the same way, while its other positions
        // sum from dlt = +0 like the definition's running sum (a code -0 after
        // the head must give S = +0, not -0).
        const bool rep = si.kind == kRepeat || !act;
        Bytes<VPL> bt;
        bt.load(dl_s + (uint32_t)(rep ? 0 : si.a + (int)p0));
        if (rep) {
#pragma unroll
            for (int k = 0; k < VPL / 4; k++) bt.w[k] = 0x80808080u;
        }
        if (flag) bt.w[0] = (bt.w[0] & 0xFFFFFF00u) | 0x80u;  // the head has no delta byte
        if constexpr (VPL == 8) {
            if (act && W - p0 < 8) {  // positions past the line end (W % 256 != 0)
                const uint64_t m = (1ull << (8 * (W - p0))) - 1ull;
                bt.w[0] &= (uint32_t)m;
                bt.w[1] &= (uint32_t)(m >> 32);
            }
        }
        float pl[VPL];
        {
            float run = 0.f;
#pragma unroll
            for (int k = 0; k < VPL / 4; k++) {
                run = (k == 0 ? code_f<0>(bt.w[k]) : run + code_f<0>(bt.w[k])); pl[4 * k + 0] = run;
                run += code_f<1>(bt.w[k]); pl[4 * k + 1] = run;
                run += code_f<2>(bt.w[k]); pl[4 * k + 2] = run;
                run += code_f<3>(bt.w[k]); pl[4 * k + 3] = run;
            }
        }
        // plain inclusive scan of lane totals; base = prefix before the head of
        // this lane's segment (its head lane in this chunk, else carried)
        const float tot = pl[VPL - 1];
        float P = tot;
#pragma unroll
        for (int d = 1; d < kWarp; d <<= 1) {
            const float y = __shfl_up_sync(0xffffffffu, P, d);
            if (lane >= d) P += y;
        }
        const float P_excl = carry_P + (P - tot);
        const uint32_t smask = __ballot_sync(0xffffffffu, flag != 0);
        const uint32_t mle = smask & le_mask;
        const float gotb = __shfl_sync(0xffffffffu, P_excl, mle ? 31 - __clz(mle) : lane);
        const float base = mle ? gotb : carry_base;
        const float dlt = rep ? -0.0f : (flag ? 0.0f : P_excl - base);
        if constexpr (!STAGED) {
            carry_P += __shfl_sync(0xffffffffu, P, 31);
            const float topb = __shfl_sync(0xffffffffu, P_excl, smask ? 31 - __clz(smask) : 0);
            if (smask) carry_base = topb;
        }
        if (!act) continue;
        float y[VPL];
        if (!si.big) {
#pragma unroll
            for (int j = 0; j < VPL; j++) {
                const float S = (j == 0 && flag) ? -0.0f : pl[j] + dlt;  // exact
                const float xh = __fmaf_rn(S, si.sc, si.h);              // RN(h + S * 2^emin)
                y[j] = __fmul_rn(__fsub_rn(xh, shv), scv);
            }
        } else {
#pragma unroll
            for (int j = 0; j < VPL; j++) {
                const float S = (j == 0 && flag) ? -0.0f : (pl[j] + dlt) * 0x1p100f;  // 2^(emin+30) scale
                const float xh = __fmaf_rn(S, si.sc, si.h);
                y[j] = __fmul_rn(__fsub_rn(xh, shv), scv);
            }
        }
        if constexpr (STAGED) {
            row_buffer_acquire(lane);
            stage_vpl<OUT, VPL>(smem_u32(rowbuf) + p0 * (uint32_t)(OUT == SPP_OUT_F32 ? 4 : 2), y);
        } else {
            emit_vpl<OUT, VPL>(row, p0, y);
        }
    }
    if constexpr (STAGED) row_buffer_release<OUT>(row, rowbuf, W, lane, rpol);
    return true;
}

// One-pass decode of a W = 32*36 line with at most 32 segments (the common
// case): lane s holds segment s's table entry in registers; the head lanes form
// one bitmap word (one warp OR-reduction) and every lane fetches its segment's
// parameters by shuffle.  Falls back to the shared-memory tables otherwise.
template <int OUT, bool RAWSEG>  // RAWSEG: a mode-3 line (FORMAT.md 2.7); mode-1 lines run without its code
__device__ __forceinline__ bool decode_line_onepass(uint8_t *buf, uint32_t buf_s, uint32_t hdr, uint32_t bytes,
                                                    uint32_t W, uint32_t *bbits, uint32_t nbw, float shv, float scv,
                                                    uint8_t *row, uint8_t *rowbuf, uint32_t rowbuf_s, uint32_t rep_s,
                                                    int lane, uint64_t rpol) {
    constexpr int VPL = 36;
    const uint32_t nseg = hdr >> 16;
    // mode 3 (FORMAT.md 2.7) also allows RAW segments; with A = 36 and W = 1152
    // it never has more than 32 segments, so the fallback sees only mode 1
    constexpr uint32_t max_kind = RAWSEG ? kRawSeg : kDiff;
    if (nseg > (uint32_t)kWarp)
        return decode_line_aligned<OUT, VPL>(buf, bytes, W, bbits, nbw, shv, scv, row, rowbuf, lane, rpol);
    if (nseg < 1 || 4u + 8u * nseg > bytes) return false;
    const uint32_t dl_s = buf_s + 4 + 8 * nseg;
    const bool have = (uint32_t)lane < nseg;
    // lanes past nseg read the (in-slot) neighbouring words and discard them
    const uint32_t dw = lds_u32(buf_s + 4 + 4 * (uint32_t)lane);
    const float hs = lds_f32(buf_s + 4 + 4 * nseg + 4 * (uint32_t)lane);
    const uint32_t len = have ? dw & 0xFFFFu : 0u, kind = have ? (dw >> 16) & 0xFFu : 0u, eb = dw >> 24;
    // delta bytes: len - 1 for DIFF, 4 len for a RAW segment (mode 3 only), none for REPEAT (selects, no branches)
    const uint32_t dlen = (kind == kDiff ? len - (uint32_t)(len > 0) : 0u) + ((RAWSEG && kind == kRawSeg) ? 4u * len : 0u);
    const uint32_t pk = len | (dlen << 16);
    const uint32_t inc = scan_incl_u32(pk);
    const uint32_t ex = inc - pk;
    const uint32_t st = ex & 0xFFFFu, db = ex >> 16;
    const uint32_t blk = st / VPL;
    // validation without short-circuit branches (FORMAT.md 2.1 / 2.7 rules)
    const uint32_t bad_lane = (uint32_t)have & ((uint32_t)(len == 0) | (uint32_t)(kind > max_kind) |
                                                ((uint32_t)(kind == kDiff) & ((uint32_t)(eb < (uint32_t)kEminBMin) |
                                                                              (uint32_t)(eb > (uint32_t)kEminBMax))) |
                                                (uint32_t)(st + len > W) | (uint32_t)(blk * VPL != st));
    const uint32_t tot = __shfl_sync(0xffffffffu, inc, 31);
    if (__any_sync(0xffffffffu, bad_lane) | ((tot & 0xFFFFu) != W) | (4u + 8u * nseg + (tot >> 16) > bytes)) return false;
    const uint32_t word = __reduce_or_sync(0xffffffffu, have ? 1u << blk : 0u);  // head lanes
    // DIFF: the code of position p is delta byte a + p; RAW: its value is at bytes a + 4p
    const int a_s = kind == kRawSeg ? (int)db - 4 * (int)st : (int)db - (int)st - 1;
    const uint32_t info = pack_seg(a_s, kind, eb);

    const uint32_t le_mask = 0xFFFFFFFFu >> (31 - lane);
    const uint32_t p0 = VPL * lane;
    const uint32_t flag = (word >> lane) & 1u;
    const int s = __popc(word & le_mask) - 1;  // segment of this lane (position 0 is always a head)
    const uint32_t d = __shfl_sync(0xffffffffu, info, s);
    const float h = __shfl_sync(0xffffffffu, hs, s);
    const int a = (int)(d & 0x3FFFFFu) - kBaseBias;
    const uint32_t skind = (d >> 22) & 3u, seb = d >> 24;
    const bool raw = RAWSEG && skind == kRawSeg;
    const bool rep = skind == kRepeat || raw;  // RAW lanes run the chain on zero codes, then take their values
    // a REPEAT / RAW lane reads a constant block of 0x80 bytes (code -0: S = -0
    // keeps h exact) instead of the delta area: same loads, no selects
    Bytes<VPL> bt;
    bt.load(rep ? rep_s : dl_s + (uint32_t)(a + (int)p0));
    if (flag) bt.w[0] = (bt.w[0] & 0xFFFFFF00u) | 0x80u;  // the head has no delta byte
    // codes of the lane's 36 positions as fp16 pairs (value = code * 2^-18),
    // then two exact fp32 prefix chains (positions 0..17 and 18..35) fed by
    // mixed-precision adds
    constexpr int HALF = VPL / 2;
    uint32_t hv[VPL / 2];
#pragma unroll
    for (int k = 0; k < VPL / 4; k++) {
        hv[2 * k] = codes_h2<0x1800u>(bt.w[k]);      // positions 4k, 4k+1
        hv[2 * k + 1] = codes_h2<0x3A20u>(bt.w[k]);  // positions 4k+2, 4k+3
    }
    float2 pp[HALF];
    pp[0] = make_float2(fadd_h(hv[0], 0, -0.0f), fadd_h(hv[HALF / 2], HALF & 1, -0.0f));
#pragma unroll
    for (int i = 1; i < HALF; i++)
        pp[i] = make_float2(fadd_h(hv[i >> 1], i & 1, pp[i - 1].x),
                            fadd_h(hv[(HALF + i) >> 1], (HALF + i) & 1, pp[i - 1].y));
    const float totA = pp[HALF - 1].x;
    const float lt = totA + pp[HALF - 1].y;  // lane total
    const float P = scan_incl_f32(lt);        // exact: multiples of 2^-18 far below 2^6
    const float P_excl = P - lt;
    const uint32_t mle = word & le_mask;
    const float base = __shfl_sync(0xffffffffu, P_excl, 31 - __clz(mle));
    // REPEAT lane: every S = -0 (x̂ = h exactly); head lane: S = -0 at the
    // head only, the rest sums from +0 like the definition's running sum
    const float dlt = rep ? -0.0f : (flag ? 0.0f : P_excl - base);
    // x̂ = RN(h + S * 2^emin) with S in code * 2^-18 units: the multiplier is
    // 2^(emin + 18) = 2^(emin_b - 132), a normal float for emin_b >= 6 and an
    // exact subnormal below; y = RN(RN(x̂ - shift) * scale). Two values per
    // instruction (FADD2/FFMA2/FMUL2 round exactly like the scalar forms).
    const float sc = __uint_as_float(seb >= 6u ? (seb - 5u) << 23 : 1u << (seb + 17u));
    const float2 dl2 = make_float2(dlt, dlt + totA), h2 = make_float2(h, h), nsh2 = make_float2(-shv, -shv),
                 scv2 = make_float2(scv, scv), sc2 = make_float2(sc, sc);
    float y[VPL];
#pragma unroll
    for (int i = 0; i < HALF; i++) {
        float2 S = fadd2_rn(pp[i], dl2);  // exact (positions i and i + 18)
        if (i == 0 && flag) S.x = -0.0f;  // the head: x̂ = h exactly
        const float2 y2 = fmul2_rn(fadd2_rn(ffma2_rn(S, sc2, h2), nsh2), scv2);
        y[i] = y2.x;
        y[HALF + i] = y2.y;
    }
    if (raw) {  // RAW segment lane: x̂ is the stored binary32 value, y = RN(RN(x̂ - shift) * scale)
        const uint32_t va = dl_s + (uint32_t)(a + 4 * (int)p0);
#pragma unroll
        for (int i = 0; i < VPL; i++) y[i] = __fmul_rn(__fadd_rn(lds_f32_any(va + 4u * i), -shv), scv);
    }
    row_buffer_acquire(lane);
    stage_vpl<OUT, VPL>(rowbuf_s + p0 * (uint32_t)(OUT == SPP_OUT_F32 ? 4 : 2), y);
    row_buffer_release<OUT>(row, rowbuf, W, lane, rpol);
    return true;
}

// mode-3 lines out of line: the mode-1 loop keeps its code footprint
// One-pass RAW16 line (FORMAT.md 2.6) of W = 32*36 values, on the instance
// opts.raw_segments selects: lane l widens its 36 binary16 values (72 B at
// 16 + 72 l, 8-B aligned) exactly, y = RN(RN(x - shift) * scale), and the row
// leaves like a one-pass SEG row (staged in the slot, one TMA bulk store).
template <int OUT>
__device__ __forceinline__ bool decode_line_raw16_onepass(uint8_t *buf, uint32_t bytes, uint32_t W, float shv,
                                                          float scv, uint8_t *row, uint8_t *rowbuf, int lane,
                                                          uint64_t rpol) {
    constexpr int VPL = 36;
    if (16u + 2u * W > bytes) return false;
    const uint32_t src = smem_u32(buf + 16) + 2u * VPL * (uint32_t)lane;
    uint32_t w[VPL / 2];
#pragma unroll
    for (int k = 0; k < VPL / 4; k++) {
        const uint2 v = lds_u2(src + 8u * k);
        w[2 * k] = v.x;
        w[2 * k + 1] = v.y;
    }
    float y[VPL];
#pragma unroll
    for (int j = 0; j < VPL; j++) {
        const float xv = __half2float(__ushort_as_half((unsigned short)((w[j >> 1] >> (16 * (j & 1))) & 0xFFFFu)));
        y[j] = __fmul_rn(__fsub_rn(xv, shv), scv);
    }
    row_buffer_acquire(lane);
    stage_vpl<OUT, VPL>(smem_u32(rowbuf) + VPL * (uint32_t)lane * (uint32_t)(OUT == SPP_OUT_F32 ? 4 : 2), y);
    row_buffer_release<OUT>(row, rowbuf, W, lane, rpol);
    return true;
}

// ---------------------------------------------------------------------------
// Global-memory line path: any FORMAT-legal line the shared-memory ring cannot
// hold (a SEG line longer than the ring, e.g. W = 1152 at A = 1 with ~1,150
// segments, or a mode-3 line with many short RAW segments) and every line of a
// sample whose W exceeds kSmemMaxW.  The warp walks the segments in order
// (32 descriptors per step: scans of len / delta-byte counts, validated before
// any byte of those segments is read) and decodes each segment with all lanes:
// REPEAT broadcasts the head, a RAW segment copies its binary32 values, a DIFF
// segment takes an exact int32 inclusive scan of its codes (S_j, |S_j| < 2^24 in
// a valid stream, FORMAT.md 2.3) and x̂ = RN(h + S_j * 2^emin) as one fma of exact
// operands (reading S13).  Rows are written with per-lane scalar stores (rare
// path: correctness, not bandwidth).  Out of line so the hot loop keeps its
// registers.
__device__ __forceinline__ int code_int(uint32_t b) {  // FORMAT.md 2.2
    const int E = (b >> 4) & 7, M = b & 15;
    const int mag = E == 0 ? M : (16 + M) << (E - 1);
    return (b & 0x80u) ? -mag : mag;
}
__device__ __forceinline__ float pow2_emin(uint32_t eb) {  // 2^(eb - 150), eb in [1, 246]: exact
    const int e = (int)eb - 150;
    return e >= -126 ? __uint_as_float((uint32_t)(e + 127) << 23) : __uint_as_float(1u << (e + 149));
}
__device__ __forceinline__ uint32_t ldg_u8(const uint8_t *p) {
    uint32_t v;
    asm volatile("ld.global.nc.u8 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}
template <int OUT>
__device__ __forceinline__ void emit1(uint8_t *row, uint32_t p, float xh, float shv, float scv) {
    const float y = __fmul_rn(__fsub_rn(xh, shv), scv);
    if constexpr (OUT == SPP_OUT_F32) reinterpret_cast<float *>(row)[p] = y;
    else reinterpret_cast<__half *>(row)[p] = __float2half_rn(y);
}
template <int OUT>
__device__ __noinline__ bool decode_line_global(const uint8_t *__restrict__ p, uint32_t bytes, uint32_t W, uint32_t A,
                                                float shv, float scv, uint8_t *__restrict__ row, int lane) {
    const uint32_t mode = ldg_u8(p);
    if (mode == kModeRaw) {  // 16-B aligned line: aligned binary32 loads
        if (16ull + 4ull * W > bytes) return false;
        const float *x = reinterpret_cast<const float *>(p + 16);
        for (uint32_t q = lane; q < W; q += kWarp) emit1<OUT>(row, q, __ldg(x + q), shv, scv);
        return true;
    }
    if (mode == kModeRaw16) {
        if (16ull + 2ull * W > bytes) return false;
        const __half *x = reinterpret_cast<const __half *>(p + 16);
        for (uint32_t q = lane; q < W; q += kWarp) emit1<OUT>(row, q, __half2float(__ldg(x + q)), shv, scv);
        return true;
    }
    if (mode != kModeSeg && mode != kModeSegRaw) return false;
    const uint32_t max_kind = mode == kModeSegRaw ? kRawSeg : kDiff;
    const uint32_t nseg = ldg_u8(p + 2) | (ldg_u8(p + 3) << 8);
    if (nseg < 1 || nseg > W || 4ull + 8ull * nseg > bytes) return false;
    const uint32_t *desc = reinterpret_cast<const uint32_t *>(p + 4);
    const float *heads = reinterpret_cast<const float *>(p + 4 + 4 * nseg);
    const uint8_t *dl = p + 4 + 8 * nseg;
    const uint64_t dl_cap = bytes - (4ull + 8ull * nseg);  // delta area bytes available
    uint32_t cl = 0;
    uint64_t cd = 0;
    for (uint32_t b0 = 0; b0 < nseg; b0 += kWarp) {
        const uint32_t s = b0 + lane;
        uint32_t len = 0, kind = 0, eb = 0;
        float h = 0.f;
        if (s < nseg) {
            const uint32_t d = __ldg(desc + s);
            len = d & 0xFFFFu;
            kind = (d >> 16) & 0xFFu;
            eb = d >> 24;
            h = __ldg(heads + s);
        }
        const uint32_t dlen = (kind == kDiff && len > 0) ? len - 1 : (kind == kRawSeg ? 4u * len : 0u);
        const uint32_t il = warp_incl_scan(len, lane), id = warp_incl_scan(dlen, lane);  // < 2^18 each
        const uint32_t st = cl + il - len;
        const uint64_t db = cd + id - dlen;
        const bool bad = s < nseg && (len == 0 || kind > max_kind ||
                                      (kind == kDiff && (eb < (uint32_t)kEminBMin || eb > (uint32_t)kEminBMax)) ||
                                      (uint64_t)st + len > W || st % A != 0);
        cl += __shfl_sync(0xffffffffu, il, 31);
        cd += __shfl_sync(0xffffffffu, id, 31);
        if (__any_sync(0xffffffffu, bad) || cd > dl_cap) return false;  // this step's bytes lie inside the line
        const uint32_t cnt = min((uint32_t)kWarp, nseg - b0);
        for (uint32_t k = 0; k < cnt; k++) {
            const uint32_t kst = __shfl_sync(0xffffffffu, st, k), klen = __shfl_sync(0xffffffffu, len, k);
            const uint32_t kkind = __shfl_sync(0xffffffffu, kind, k), keb = __shfl_sync(0xffffffffu, eb, k);
            const uint64_t kdb = __shfl_sync(0xffffffffu, db, k);
            const float kh = __shfl_sync(0xffffffffu, h, k);
            if (kkind == kRepeat) {
                for (uint32_t j = lane; j < klen; j += kWarp) emit1<OUT>(row, kst + j, kh, shv, scv);
            } else if (kkind == kRawSeg) {  // FORMAT.md 2.7: the values are binary32 at the byte base
                for (uint32_t j = lane; j < klen; j += kWarp) {
                    const uint8_t *v = dl + kdb + 4ull * j;
                    const uint32_t bits = ldg_u8(v) | (ldg_u8(v + 1) << 8) | (ldg_u8(v + 2) << 16) | (ldg_u8(v + 3) << 24);
                    emit1<OUT>(row, kst + j, __uint_as_float(bits), shv, scv);
                }
            } else {  // DIFF: S_j = code(d_0) + ... + code(d_{j-1}) for the position j of the segment
                const float unit = pow2_emin(keb);
                int carry = 0;
                for (uint32_t j0 = 0; j0 < klen; j0 += kWarp) {
                    const uint32_t j = j0 + lane;
                    const int c = (j >= 1 && j < klen) ? code_int(ldg_u8(dl + kdb + (j - 1))) : 0;
                    const int S = warp_incl_scan(c, lane) + carry;
                    carry = __shfl_sync(0xffffffffu, S, 31);
                    if (j < klen) emit1<OUT>(row, kst + j, j == 0 ? kh : __fmaf_rn((float)S, unit, kh), shv, scv);
                }
            }
        }
    }
    return cl == W;
}

// ---------------------------------------------------------------------------
// Warp-specialised KD: the last warp of each CTA is a producer whose lane k
// streams the lines of consumer warp k into that warp's ring of input slots
// (directory read + validation, channel constants, 1-D TMA bulk copy,
// full/empty mbarriers per slot), so the decoding warps spend their issue
// slots on decoding only.  A consumer waits for its slot, decodes the line
// and releases the slot as soon as it has read it (one-pass rows are staged in
// the warp's own row buffer, never in the input slot).  A line longer than one
// slot takes the whole ring; a line longer than the ring (or any line when W
// exceeds the shared tables) is handed over as a record only and decoded from
// HBM by decode_line_global.
#ifndef SPP_KD_WS_WPC
#define SPP_KD_WS_WPC 11  // consumer warps per CTA (+1 producer warp)
#endif
#ifndef SPP_KD_WS_MINB
#define SPP_KD_WS_MINB 2
#endif
constexpr int kWsWarps = SPP_KD_WS_WPC + 1;
#ifndef SPP_KD_PROD_SLEEP_NS
#define SPP_KD_PROD_SLEEP_NS 100  // producer back-off when no slot was free this round
#endif
#ifndef SPP_KD_PROD_SERIAL
#define SPP_KD_PROD_SERIAL 0
#endif
#ifndef SPP_KD_PROD_REACQUIRE
#define SPP_KD_PROD_REACQUIRE 0  // measured -3% on C4 and racecheck still flags the refills (profiles/r02b)
#endif
#ifndef SPP_KD_WS_NS
#define SPP_KD_WS_NS 3  // input slots per consumer warp (a ring)
#endif
#ifndef SPP_KD_WS_SLOT
#define SPP_KD_WS_SLOT 2048  // target slot bytes; longer lines take the whole ring, longer still the global path
#endif
constexpr uint32_t kWsNs = SPP_KD_WS_NS;
static_assert(kWsNs >= 2 && kWsNs <= 8, "slot ring");
constexpr uint32_t kWsCtl = 32 * kWsNs;  // per consumer: full[NS], empty[NS] mbarriers + info[NS] (16 B each)
constexpr uint32_t kFlagBig = 1u, kFlagGlobal = 2u;  // line record flags (bits 16.. = alignment A)

template <int OUT, bool VEC, int VPL, bool RAWSEG>  // RAWSEG: opts.raw_segments (mode-3 lines in one pass)
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kWsWarps * kWarp, SPP_KD_WS_MINB) kd_decode_ws(
    const DcMeta *__restrict__ meta, int n, uint32_t L, uint32_t H, uint32_t W, const float *__restrict__ shift,
    const float *__restrict__ scale, uint8_t *__restrict__ dst, uint32_t cap, uint32_t rowb, uint32_t nwords,
    uint32_t warp_bytes, uint32_t *__restrict__ status, uint32_t row_ef) {
    extern __shared__ __align__(16) uint8_t smem_raw[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int wpc = (int)(blockDim.x >> 5) - 1;  // consumer warps; warp wpc produces
    const size_t ob = OUT == SPP_OUT_F32 ? 4 : 2;
    const uint32_t cap_data = cap - 16;         // one slot; the last 16 B are read slack
    const uint32_t big_cap = kWsNs * cap - 16;  // the whole ring
    const uint64_t T = (uint64_t)n * L;
    const uint64_t NW = (uint64_t)gridDim.x * wpc;
    const uint32_t ctl_off = (kWsNs * cap + rowb + 4 * nwords + 15u) & ~15u;  // 16-B aligned: info[] is read as uint4
    auto ctl = [&](int w) { return reinterpret_cast<uint64_t *>(smem_raw + (size_t)w * warp_bytes + ctl_off); };

    if (warp == wpc && lane < 12)  // 48 B of 0x80 after the warps' regions: REPEAT lanes' code bytes
        reinterpret_cast<uint32_t *>(smem_raw + (size_t)wpc * warp_bytes)[lane] = 0x80808080u;
    if (warp == wpc && lane < wpc) {
        uint64_t *c = ctl(lane);
        for (uint32_t i = 0; i < kWsNs; i++) {
            mbar_init(&c[i], 1);              // full[i]: the producer lane's arrival + the TMA bytes
            mbar_init(&c[kWsNs + i], kWarp);  // empty[i]: every consumer lane (each has read the slot)
        }
        fence_mbar_init();
    }
    __syncthreads();

    if (warp == wpc) {
        // ------------------------------------------------------------ producer
        // Lane k streams consumer k's lines.  The directory is read one line
        // ahead of need (dn = dir[lk + 2]), so the entry of the next line is
        // ready, from registers, the moment its slot is released.
        const int k = lane;
        bool active = k < wpc;
        uint64_t g = 0, ge = 0;
        if (active) {
            const uint64_t gw = (uint64_t)blockIdx.x * wpc + k;
            g = gw * T / NW;
            ge = (gw + 1) * T / NW;
            active = g < ge;
        }
        uint8_t *rb = smem_raw + (size_t)(active ? k : 0) * warp_bytes;
        uint64_t *full = ctl(active ? k : 0), *empty = full + kWsNs;
        uint4 *info = reinterpret_cast<uint4 *>(full + 2 * kWsNs);
        uint32_t sk = 0, lk = 0, ck = 0, yk = 0, da = 0, db = 0, dn = 0, s = 0;
        uint32_t used = 0, par = 0;  // bit i: slot i filled before / parity of its next release
        DcMeta m{nullptr, nullptr, 0, 0, 0};
        float shv = 0.f, scv = 1.f;
        uint32_t e_bytes = 0, e_flags = 0;
        const uint8_t *e_src = nullptr;
        auto dir_at = [&](uint32_t i) { return __ldg(reinterpret_cast<const uint32_t *>(m.dir) + i); };
        auto start_sample = [&]() {  // line lk of sample sk (synchronous: once per sample)
            m = meta[sk];
            if (m.valid) {
                da = dir_at(lk);
                db = dir_at(lk + 1);
                dn = lk + 2 <= L ? dir_at(lk + 2) : 0u;
            }
        };
        auto load_consts = [&]() {
            shv = shift ? __ldg(shift + ck) : 0.f;
            scv = scale ? __ldg(scale + ck) : 1.f;
        };
        auto compute_entry = [&]() {  // line g from (da, db), validated once
            e_bytes = 0;
            e_flags = 0;
            if (m.valid) {
                const bool ok = db >= da && ((da | db) & 15u) == 0 && (uint64_t)db <= m.limit && db - da >= 16;
                if (!ok) {
                    report(status, SPP_ERR_CORRUPT, (int64_t)sk);
                } else {
                    e_bytes = db - da;
                    e_src = m.payload + da;
                    // too long for the ring, or W beyond the shared tables: decoded from HBM
                    e_flags = (nwords == 0 || e_bytes > big_cap ? kFlagGlobal : (e_bytes > cap_data ? kFlagBig : 0u)) |
                              (m.align << 16);
                }
            }
        };
        if (active) {
            sk = (uint32_t)(g / L);
            lk = (uint32_t)(g - (uint64_t)sk * L);
            ck = lk / H;
            yk = lk - ck * H;
            start_sample();
            load_consts();
            compute_entry();
        }
        while (__any_sync(0xffffffffu, active)) {
            bool did = false;
            if (active) {
                const bool big = e_flags & kFlagBig;
                const bool glob = e_flags & kFlagGlobal;
                bool ready = false;
                auto test_slots = [&]() {
                    if (!big) {
                        ready = !((used >> s) & 1u) || mbar_test(&empty[s], (par >> s) & 1u);
                    } else {  // an oversize line takes the whole ring: every slot must be free
                        ready = true;
                        for (uint32_t i = 0; i < kWsNs; i++)
                            ready = ready && (!((used >> i) & 1u) || mbar_test(&empty[i], (par >> i) & 1u));
                    }
                };
                if constexpr (SPP_KD_PROD_SERIAL) {
                    // one lane at a time: compute-sanitizer's racecheck does not see the
                    // acquire of an mbarrier test issued by several lanes of a warp on
                    // different barriers (scripts/racecheck_repro.cu variants 4 vs 3/7)
                    for (int kk = 0; kk < wpc; kk++)
                        if (kk == k) test_slots();
                } else {
                    test_slots();
                }
                if (ready && SPP_KD_PROD_REACQUIRE) {
                    // the phases just found complete by test_wait are taken again with
                    // try_wait (returns at once): same acquire semantics, but the form
                    // compute-sanitizer's racecheck models, so it sees the consumer's
                    // reads of the slot ordered before this refill
                    for (uint32_t i = 0; i < kWsNs; i++)
                        if ((((big ? (1u << kWsNs) - 1u : 1u << s) & used) >> i) & 1u)
                            mbar_wait(&empty[i], (par >> i) & 1u);
                }
                if (ready) {
                    // the line record (16 B, st.async) and its bytes (TMA) both count on
                    // full[s]; a zero-byte line delivers only the record, a global line
                    // its record with the source address in place of the channel constants
                    const uint32_t tx = glob ? 0u : e_bytes;
                    mbar_arrive_expect_tx(&full[s], tx + 16u);
                    const uint64_t sa = reinterpret_cast<uint64_t>(e_src);
                    st_async_u4(smem_u32(&info[s]),
                                glob ? make_uint4(e_bytes, e_flags, (uint32_t)sa, (uint32_t)(sa >> 32))
                                     : make_uint4(e_bytes, e_flags, __float_as_uint(shv), __float_as_uint(scv)),
                                &full[s]);
                    if (tx) bulk_g2s(big ? rb : rb + s * cap, e_src, tx, &full[s]);
                    const uint32_t took = big ? (1u << kWsNs) - 1u : 1u << s;
                    par ^= took & used;
                    used |= took;
                    s = s + 1 == kWsNs ? 0u : s + 1;
                    g++;
                    did = true;
                    active = g < ge;
                    if (active) {  // advance to line g and prepare its entry
                        if (++yk == H) {
                            yk = 0;
                            ck++;
                        }
                        if (++lk == L) {
                            lk = 0;
                            ck = 0;
                            yk = 0;
                            sk++;
                            start_sample();
                        } else {
                            da = db;
                            db = dn;
                            if (m.valid && lk + 2 <= L) dn = dir_at(lk + 2);  // used one line from now
                        }
                        if (yk == 0) load_consts();
                        compute_entry();
                    }
                }
            }
            if (!__any_sync(0xffffffffu, did) && SPP_KD_PROD_SLEEP_NS) __nanosleep(SPP_KD_PROD_SLEEP_NS);
        }
        return;
    }

    // ---------------------------------------------------------------- consumer
    const uint64_t gw = (uint64_t)blockIdx.x * wpc + warp;
    const uint64_t g_begin = gw * T / NW, g_end = (gw + 1) * T / NW;
    uint8_t *base = smem_raw + (size_t)warp * warp_bytes;
    uint8_t *rowbuf = base + kWsNs * cap;  // one-pass instances: the staged output row
    uint32_t *sbits = reinterpret_cast<uint32_t *>(base + kWsNs * cap + rowb);
    uint32_t *wpre = sbits + nwords / 2;
    uint64_t *full = ctl(warp), *empty = full + kWsNs;
    const uint32_t info_s = smem_u32(full + 2 * kWsNs);
    const uint32_t nbw = (W / VPL + 31) / 32;
    const uint32_t nsb = nwords / 2;  // words of the start bitmap (and of its prefix counts)
    const uint32_t rep_s = smem_u32(smem_raw + (size_t)wpc * warp_bytes);  // 48 B of 0x80 (producer-filled)
    const uint32_t base_s = smem_u32(base), rowbuf_s = smem_u32(rowbuf);      // shared addresses, hoisted
    // L2 policy of the row stores: evict_first when the launch writes far more than
    // L2 holds (batches: C4 +0.8%, profiles/r02a8_*), normal otherwise (a single
    // sample's output stays L2-resident for its consumer)
    uint64_t rpol;
    if (row_ef) asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(rpol));
    else asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(rpol));
    uint32_t fph = 0;  // bit s: parity of slot s's next full phase
    uint32_t s = 0;
    const uint32_t nlines = (uint32_t)(g_end - g_begin);  // < 2^32: lines of one warp
    const uint64_t row_bytes = (uint64_t)W * ob;
    uint8_t *row = dst + g_begin * row_bytes;
    for (uint32_t it = 0; it < nlines; it++, row += row_bytes, s = s + 1 == kWsNs ? 0u : s + 1) {
        mbar_wait(&full[s], (fph >> s) & 1u);
        fph ^= 1u << s;
        const uint4 inf = lds_u4(info_s + 16u * s);
        const uint32_t bytes = inf.x, flags = inf.y, al = flags >> 16;
        if (flags & kFlagGlobal) {
            // record only: release the slot at once, decode the line from HBM
            mbar_arrive(&empty[s]);
            const uint64_t g = g_begin + it;
            const uint8_t *src = reinterpret_cast<const uint8_t *>((uint64_t)inf.w << 32 | inf.z);
            const uint32_t c = (uint32_t)(g % L) / H;
            const float shv = shift ? __ldg(shift + c) : 0.f, scv = scale ? __ldg(scale + c) : 1.f;
            const bool ok = decode_line_global<OUT>(src, bytes, W, al, shv, scv, row, lane);
            if (!ok && lane == 0) report(status, SPP_ERR_CORRUPT, (int64_t)(g / L));
            continue;
        }
        if (bytes) {
            const uint32_t boff = (flags & kFlagBig) ? 0u : s * cap;
            uint8_t *buf = base + boff;
            const uint32_t buf_s = base_s + boff;
            const float shv = __uint_as_float(inf.z), scv = __uint_as_float(inf.w);
            const uint32_t hdr = lds_u32(buf_s);  // mode (byte 0) and nseg (bytes 2-3)
            const uint32_t mode = hdr & 0xFFu;
            bool ok;
            if (RAWSEG && mode == kModeRaw16) {
                if constexpr (RAWSEG && VPL == 36)
                    ok = decode_line_raw16_onepass<OUT>(buf, bytes, W, shv, scv, row, rowbuf, lane, rpol);
            } else if (VEC && al == (uint32_t)VPL && (mode == kModeSeg || (RAWSEG && mode == kModeSegRaw))) {
                if constexpr (VPL == 36) {
                    if (!RAWSEG || mode == kModeSeg)
                        ok = decode_line_onepass<OUT, false>(buf, buf_s, hdr, bytes, W, sbits, nbw, shv, scv, row,
                                                             rowbuf, rowbuf_s, rep_s, lane, rpol);
                    else
                        ok = decode_line_onepass<OUT, true>(buf, buf_s, hdr, bytes, W, sbits, nbw, shv, scv, row,
                                                            rowbuf, rowbuf_s, rep_s, lane, rpol);
                }
                else ok = decode_line_aligned<OUT, VPL>(buf, bytes, W, sbits, nbw, shv, scv, row, rowbuf, lane, rpol);
            } else {
                ok = decode_line<OUT, VEC>(buf, bytes, W, al, sbits, wpre, nsb, shv, scv, row, lane);
            }
            if (!ok && lane == 0) report(status, SPP_ERR_CORRUPT, (int64_t)((g_begin + it) / L));
        }
        __syncwarp();
        // every lane releases: its own reads of the slot and of info[s] precede its arrival
        if (__builtin_expect(flags & kFlagBig, 0)) {
            for (uint32_t i = 0; i < kWsNs; i++) mbar_arrive(&empty[i]);  // the line took the whole ring
        } else {
            mbar_arrive(&empty[s]);
        }
    }
    if constexpr (VPL == 36) {
        if (lane == 0) bulk_wait_all();  // shared memory must outlive the last row stores
    }
}

template <int OUT, bool VEC, int VPL, bool RAWSEG>
spp_status launch_kd_ws(const DcMeta *meta, int n, void *d_dst, const spp_decode_opts &o, cudaStream_t stream,
                        const DeviceProps &dp) {
    const uint32_t W = (uint32_t)o.W;
    const bool smem_tables = W <= kSmemMaxW;  // else every line takes the global path
    // slot: a typical SEG line (~1 B/value); a RAW line (or any longer line)
    // takes the whole ring; a line longer than the ring is decoded from HBM
    const uint32_t raw = (uint32_t)round_up16(16 + 4ull * W);
    uint32_t cap_in = 16;
    if (smem_tables) {
        cap_in = std::min<uint32_t>(raw, SPP_KD_WS_SLOT);
        cap_in = std::max<uint32_t>(cap_in, std::min<uint32_t>((uint32_t)round_up16((raw + kWsNs - 1) / kWsNs),
                                                               2 * SPP_KD_WS_SLOT));
    }
    const uint32_t cap = (uint32_t)round_up16(cap_in) + 16;
    const uint32_t rowb = VPL == 36 ? W * (OUT == SPP_OUT_F32 ? 4u : 2u) : 0u;  // one-pass row buffer
    const uint32_t nwords = smem_tables ? 2 * ((W + 31) / 32 + 1) : 0u;        // start bitmap + prefix counts
    const uint32_t warp_bytes = (uint32_t)round_up16(kWsNs * cap + rowb + 4 * nwords) + kWsCtl;
    // consumer warps per CTA: as many as fit two CTAs per SM (else one)
    int wpc = SPP_KD_WS_WPC;
    auto fits = [&](int w, int ctas) {
        return (size_t)w * warp_bytes + 64 <= (size_t)dp.smem_optin &&
               (size_t)ctas * ((size_t)w * warp_bytes + 64 + dp.smem_reserved) <= (size_t)dp.smem_per_sm;
    };
    while (wpc > 1 && !fits(wpc, 2)) wpc--;
    if (!fits(wpc, 2)) {
        wpc = SPP_KD_WS_WPC;
        while (wpc > 1 && !fits(wpc, 1)) wpc--;
    }
    if (!fits(wpc, 1)) return SPP_ERR_UNSUPPORTED;
    const int smem = wpc * (int)warp_bytes + 64;  // + the constant REPEAT code block
    auto kern = kd_decode_ws<OUT, VEC, VPL, RAWSEG>;
    if (set_smem_attr<kd_decode_ws<OUT, VEC, VPL, RAWSEG>>(smem, dp) != SPP_OK) return SPP_ERR_CUDA;
    int occ = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, (wpc + 1) * kWarp, smem) != cudaSuccess || occ < 1)
        return SPP_ERR_CUDA;
    const uint64_t lines = (uint64_t)n * o.C * o.H;
    const uint64_t max_ctas = (uint64_t)dp.sms * occ;
    // st.async needs a cluster of at least 2 CTAs (they never touch each other's memory): even grid
    int grid = (int)std::max<uint64_t>(1, std::min<uint64_t>(max_ctas, (lines + wpc - 1) / wpc));
    // row stores evict_first when the launch's output far exceeds L2 (SPP_KD_ROW_EF)
    const uint32_t row_ef = SPP_KD_ROW_EF && lines * W * (OUT == SPP_OUT_F32 ? 4u : 2u) > kRowEfBytes;
    grid += grid & 1;
    kern<<<grid, (wpc + 1) * kWarp, smem, stream>>>(meta, n, (uint32_t)(o.C * o.H), (uint32_t)o.H, W, o.shift,
                                                     o.scale, static_cast<uint8_t *>(d_dst), cap, rowb, nwords,
                                                     warp_bytes, o.status, row_ef);
    return cudaGetLastError() == cudaSuccess ? SPP_OK : SPP_ERR_CUDA;
}

}  // namespace

size_t deepcam_workspace_bytes(int n) { return n <= 0 ? 0 : round_up16((size_t)n * sizeof(DcMeta)); }

spp_status deepcam_decode(const void *const *d_src, int n, void *d_dst, const spp_decode_opts &o,
                          cudaStream_t stream) {
    DeviceProps dp;
    spp_status st = current_device_props(&dp);
    if (st != SPP_OK) return st;
    DcMeta *meta = static_cast<DcMeta *>(o.workspace);
    cudaEvent_t const *ev = reinterpret_cast<cudaEvent_t const *>(o.timing_events);
    if (ev && cudaEventRecord(ev[0], stream) != cudaSuccess) return SPP_ERR_CUDA;
    kd0_parse<<<(n + 127) / 128, 128, 0, stream>>>(d_src, o.src_bytes, n, o.C, o.H, o.W, meta, o.status);
    if (cudaGetLastError() != cudaSuccess) return SPP_ERR_CUDA;
    if (ev && cudaEventRecord(ev[1], stream) != cudaSuccess) return SPP_ERR_CUDA;
    const size_t align = o.out == SPP_OUT_F32 ? 32 : 16;
    const bool vec = o.W % 8 == 0 && (reinterpret_cast<uintptr_t>(d_dst) % align) == 0;
    const bool v36 = vec && o.W == 1152;  // the DeepCAM line: 32 lanes x 36 positions, one pass
    spp_status r = SPP_ERR_INVALID_ARG;
    // opts.raw_segments: the W = 1152 instance that also takes mode-3 lines
    // (FORMAT.md 2.7) in one pass; without it they take the general line path
    const bool rs = v36 && o.raw_segments;
#define SPP_LAUNCH_KD(OUT, VEC, VPL) launch_kd_ws<OUT, VEC, VPL, false>(meta, n, d_dst, o, stream, dp)
#define SPP_LAUNCH_KD_RS(OUT) launch_kd_ws<OUT, true, 36, true>(meta, n, d_dst, o, stream, dp)
    if (o.out == SPP_OUT_F32)
        r = rs ? SPP_LAUNCH_KD_RS(SPP_OUT_F32)
               : v36 ? SPP_LAUNCH_KD(SPP_OUT_F32, true, 36)
                     : vec ? SPP_LAUNCH_KD(SPP_OUT_F32, true, 8) : SPP_LAUNCH_KD(SPP_OUT_F32, false, 8);
    else if (o.out == SPP_OUT_F16)
        r = rs ? SPP_LAUNCH_KD_RS(SPP_OUT_F16)
               : v36 ? SPP_LAUNCH_KD(SPP_OUT_F16, true, 36)
                     : vec ? SPP_LAUNCH_KD(SPP_OUT_F16, true, 8) : SPP_LAUNCH_KD(SPP_OUT_F16, false, 8);
#undef SPP_LAUNCH_KD
#undef SPP_LAUNCH_KD_RS
    if (r == SPP_OK && ev && cudaEventRecord(ev[2], stream) != cudaSuccess) return SPP_ERR_CUDA;
    return r;
}

}  // namespace spp
